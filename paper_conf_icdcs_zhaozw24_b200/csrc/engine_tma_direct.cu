// TMA pipeline instantiated for DIRECT plans (loopback, zero-copy IPC): no
// flag waits on the data path, so one CTA per SM with a deep 3 x 64 KiB ring
// moves the most bytes (profiles/sweep_tma_r01.json: 1.008 of the copy peak).
// ADAPCC_DIRECT_* override the ring shape for tuning sweeps only.
#ifndef ADAPCC_DIRECT_STAGES
#define ADAPCC_DIRECT_STAGES 3
#endif
#ifndef ADAPCC_DIRECT_STAGE_KB
#define ADAPCC_DIRECT_STAGE_KB 64
#endif
#ifndef ADAPCC_DIRECT_MINB
#define ADAPCC_DIRECT_MINB 1
#endif
#define ADAPCC_TMA_NS tma_direct
#define ADAPCC_TMA_STAGES ADAPCC_DIRECT_STAGES
#define ADAPCC_TMA_STAGE_KB ADAPCC_DIRECT_STAGE_KB
#define ADAPCC_TMA_MINB ADAPCC_DIRECT_MINB
#include "engine_tma_impl.cuh"
