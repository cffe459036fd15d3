// TMA pipeline instantiated for STAGED plans (per-chunk flag handoffs between
// CTAs / GPUs): two CTAs per SM with 3 x 32 KiB rings keep more items in flight
// while some producers wait on flags (profiles/sweep_tma_r01.json).
#define ADAPCC_TMA_NS tma_staged
#define ADAPCC_TMA_STAGES 3
#define ADAPCC_TMA_STAGE_KB 32
#define ADAPCC_TMA_MINB 2
#include "engine_tma_impl.cuh"
