// Does compute-sanitizer racecheck model mbarrier arrive / try_wait?
//
// A textbook single-slot handoff: warp 1 (producer) writes a shared word,
// every lane __syncwarp()s, lane 0 arrives on `full` (release.cta); warp 0
// (consumer) waits on `full` (acquire.cta) and reads the word, then arrives on
// `empty`; the producer waits on `empty` before rewriting.  Correct by the
// PTX memory model.  Variant B replaces the mbarriers with named barriers
// (bar.arrive / bar.sync), which racecheck does model.  If racecheck reports
// hazards for A only, reports on the TMA engine's mbarrier-synchronised item
// queue are the tool's limitation, not races.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -o probe racecheck_mbarrier_probe.cu
//   compute-sanitizer --tool racecheck ./probe A ; ... ./probe B
#include <cstdio>
#include <cstring>

__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, unsigned c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, unsigned parity) {
  unsigned ok = 0;
  while (!ok)
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                 : "=r"(ok) : "r"(su32(b)), "r"(parity) : "memory");
}

__global__ void probe_mbarrier(int iters, int* out) {
  __shared__ unsigned long long full, empty;
  __shared__ int slot[32];
  if (threadIdx.x == 0) {
    mbar_init(&full, 1);
    mbar_init(&empty, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  int acc = 0;
  for (int i = 0; i < iters; ++i) {
    const unsigned ph = i & 1;
    if (threadIdx.x >= 32) {               // producer warp
      if (i > 0) mbar_wait(&empty, ph ^ 1);
      slot[lane] = i * 32 + lane;
      __syncwarp();
      if (lane == 0) mbar_arrive(&full);
    } else {                                // consumer warp
      mbar_wait(&full, ph);
      acc += slot[(lane + 1) & 31];
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty);
    }
  }
  if (threadIdx.x < 32) out[threadIdx.x] = acc;
}

__global__ void probe_named(int iters, int* out) {
  __shared__ int slot[32];
  const int lane = threadIdx.x & 31;
  int acc = 0;
  for (int i = 0; i < iters; ++i) {
    if (threadIdx.x >= 32) {
      if (i > 0) asm volatile("bar.sync 2, 64;" ::: "memory");     // empty
      slot[lane] = i * 32 + lane;
      asm volatile("bar.arrive 1, 64;" ::: "memory");              // full
    } else {
      asm volatile("bar.sync 1, 64;" ::: "memory");
      acc += slot[(lane + 1) & 31];
      if (i + 1 < iters) asm volatile("bar.arrive 2, 64;" ::: "memory");
    }
  }
  if (threadIdx.x < 32) out[threadIdx.x] = acc;
}

int main(int argc, char** argv) {
  const bool named = argc > 1 && !strcmp(argv[1], "B");
  int* d;
  cudaMalloc(&d, 32 * sizeof(int));
  if (named) probe_named<<<1, 64>>>(8, d);
  else probe_mbarrier<<<1, 64>>>(8, d);
  int h[32];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  int exp = 0;
  for (int i = 0; i < 8; ++i) exp += i * 32 + 1;
  printf("%s handoff: lane0 sum %d (expected %d) %s\n", named ? "named-barrier" : "mbarrier", h[0], exp,
         cudaGetLastError() == cudaSuccess && h[0] == exp ? "ok" : "FAIL");
  return 0;
}
