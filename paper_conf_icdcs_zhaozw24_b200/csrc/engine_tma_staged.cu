// TMA pipeline instantiated for STAGED plans (per-chunk flag handoffs between
// CTAs / GPUs): two CTAs per SM with 3 x 32 KiB rings keep more items in flight
// while some producers wait on flags (profiles/sweep_tma_r01.json).
#define ADAPCC_TMA_NS tma_staged
#define ADAPCC_TMA_STAGES 3
#define ADAPCC_TMA_STAGE_KB 32
#define ADAPCC_TMA_MINB 2
// 2 CTAs x 9 warps per SM leave 96 registers per thread (the register file is
// split over 4 SM sub-partitions: 5 warps x 96 x 32 <= 16 K each); the kernel
// fits them without spills since the rare accumulate-copy path stopped
// holding 8 vectors per thread in registers.  ADAPCC_STAGED_MAXNREG (tuning
// only) trades occupancy for registers: 104+ drops the ring to 1 CTA/SM.
#if defined(ADAPCC_STAGED_MAXNREG) && ADAPCC_STAGED_MAXNREG > 0
#define ADAPCC_TMA_MAXNREG ADAPCC_STAGED_MAXNREG
#endif
#include "engine_tma_impl.cuh"
