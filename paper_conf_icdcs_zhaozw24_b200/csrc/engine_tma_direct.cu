// TMA pipeline instantiated for DIRECT plans (loopback, zero-copy IPC): no
// flag waits on the data path, so one CTA per SM with a deep 3 x 64 KiB ring
// moves the most bytes (profiles/sweep_tma_r01.json: 1.008 of the copy peak).
#define ADAPCC_TMA_NS tma_direct
#define ADAPCC_TMA_STAGES 3
#define ADAPCC_TMA_STAGE_KB 64
#define ADAPCC_TMA_MINB 1
#include "engine_tma_impl.cuh"
