// Link probe kernel (NEXT-2: the paper's alpha-beta link profiling, P:L109-115,
// §IV-B): one "message" = `bytes` from a local buffer to each of up to 64
// destination buffers (peer GPUs' IPC-mapped arenas over NVLink, or local HBM
// in loopback), moved by TMA bulk copies: global -> shared -> destination, the
// store path the engine's zero-copy plans use.  The copy-engine variant of the
// probe is plain cudaMemcpyAsync (adapcc.cpp).
#include <cuda_runtime.h>

#include <cstdint>

#include "launch.hpp"

namespace adapcc {
namespace {

constexpr int kProbeStages = 4;
constexpr uint32_t kProbeTile = 8 * 1024;  // 4 x 8 KiB static shared memory per CTA, several CTAs per SM

struct ProbeParams {
  const char* src;
  uint64_t bytes;  // per destination (multiple of 16)
  int ndst;
  char* dst[kMaxRanksDev];
};

__device__ __forceinline__ uint32_t s32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// One elected thread per CTA: a ring of kProbeStages tiles; tile j's bulk
// store is issued as soon as its bulk load landed, and its buffer is reloaded
// (tile j + stages) once that store has read it.
__global__ void __launch_bounds__(32) probe_copy_kernel(const __grid_constant__ ProbeParams P) {
  __shared__ __align__(128) char buf[kProbeStages][kProbeTile];
  __shared__ __align__(8) uint64_t full[kProbeStages];
  if (threadIdx.x != 0) return;
  const uint64_t per = (P.bytes + kProbeTile - 1) / kProbeTile;
  const uint64_t ntiles = per * (uint64_t)P.ndst;
  for (int k = 0; k < kProbeStages; ++k)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&full[k])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  auto tile_of = [&](uint64_t i, const char** s, char** d, uint32_t* tb) {
    const uint64_t q = i / per, t = i - q * per;
    const uint64_t off = t * kProbeTile;
    *tb = (uint32_t)(P.bytes - off < kProbeTile ? P.bytes - off : kProbeTile);
    *s = P.src + off;
    *d = P.dst[q] + off;
  };
  auto load = [&](uint64_t i, int k) {
    const char* s;
    char* d;
    uint32_t tb;
    tile_of(i, &s, &d, &tb);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(&full[k])), "r"(tb) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     s32(buf[k])), "l"(s), "r"(tb), "r"(s32(&full[k]))
                 : "memory");
  };
  uint32_t phase = 0;  // bit k: parity of stage k's next completion
  uint64_t j = 0;
  for (uint64_t i = blockIdx.x; i < ntiles && j < kProbeStages; i += gridDim.x, ++j) load(i, (int)j);
  j = 0;
  for (uint64_t i = blockIdx.x; i < ntiles; i += gridDim.x, ++j) {
    const int k = (int)(j % kProbeStages);
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                   : "=r"(ok) : "r"(s32(&full[k])), "r"((phase >> k) & 1) : "memory");
    phase ^= 1u << k;
    const char* s;
    char* d;
    uint32_t tb;
    tile_of(i, &s, &d, &tb);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(d), "r"(s32(buf[k])), "r"(tb)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    const uint64_t nxt = i + (uint64_t)kProbeStages * gridDim.x;
    if (nxt < ntiles) {
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // buf[k] read by its store
      load(nxt, k);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

}  // namespace

cudaError_t probe_launch(const char* src, char* const* dst, int ndst, uint64_t bytes, int grid,
                         cudaStream_t stream) {
  if (ndst < 1 || ndst > kMaxRanksDev || (bytes & 15)) return cudaErrorInvalidValue;
  ProbeParams p{};
  p.src = src;
  p.bytes = bytes;
  p.ndst = ndst;
  for (int q = 0; q < ndst; ++q) p.dst[q] = dst[q];
  cudaGetLastError();
  probe_copy_kernel<<<grid, 32, 0, stream>>>(p);
  return cudaGetLastError();
}

}  // namespace adapcc
