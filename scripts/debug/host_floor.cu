// Host enqueue cost of one collective call through the C ABI, without Python
// (separates the library's own cost from ctypes / torch marshalling).
// Build + run (GPU box):  bash scripts/debug/host_floor.sh
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <vector>

#include "../../include/adapcc.h"

struct Big { char b[1792]; };
__global__ void empty_big(const __grid_constant__ Big p) { if (p.b[threadIdx.x & 1023] == 123) asm volatile("trap;"); }
__global__ void empty_small(int x) { if (x == 123) asm volatile("trap;"); }

__global__ void spin(long long cycles) {
  const long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}

int main() {
  const int n = 8;
  const size_t count = 256;  // 1 KiB fp32 per rank
  adapcc_comm_t c;
  if (adapcc_init_loopback(&c, n, 0, 0, ADAPCC_MODE_DIRECT)) return 1;
  std::vector<void*> x(n), y(n);
  for (int r = 0; r < n; ++r) {
    cudaMalloc(&x[r], count * 4);
    cudaMalloc(&y[r], count * 4);
  }
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  auto call = [&] {
    return adapcc_allreduce_lb(c, (const void* const*)x.data(), (void* const*)y.data(), count, ADAPCC_FLOAT32,
                               (1u << n) - 1, 0, s);
  };
  for (int i = 0; i < 200; ++i) call();
  cudaStreamSynchronize(s);
  const int K = 300;
  // (1) host-only: stream held by a long spin kernel, K enqueues
  spin<<<1, 1, 0, s>>>(4000000000LL);
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < K; ++i) call();
  auto t1 = std::chrono::steady_clock::now();
  cudaStreamSynchronize(s);
  printf("host enqueue only (stream blocked): %.3f us/call\n",
         std::chrono::duration<double, std::micro>(t1 - t0).count() / K);
  {  // host-only costs of the pieces: bookkeeping without a launch, raw launches
    auto spin_then = [&](auto f) {
      spin<<<1, 1, 0, s>>>(2000000000LL);
      auto a0 = std::chrono::steady_clock::now();
      for (int i = 0; i < K; ++i) f();
      auto a1 = std::chrono::steady_clock::now();
      cudaStreamSynchronize(s);
      return std::chrono::duration<double, std::micro>(a1 - a0).count() / K;
    };
    printf("adapcc_allreduce_lb count=0 (no launch): %.3f us\n", spin_then([&] {
      adapcc_allreduce_lb(c, (const void* const*)x.data(), (void* const*)y.data(), 0, ADAPCC_FLOAT32, (1u << n) - 1, 0, s);
    }));
    Big big{};
    for (int pdl = 0; pdl < 2; ++pdl) {
      cudaLaunchConfig_t cfg{};
      cfg.gridDim = dim3(148);
      cfg.blockDim = dim3(256);
      cfg.stream = s;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      at[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = at;
      cfg.numAttrs = pdl;
      printf("cudaLaunchKernelEx 1792-B param, pdl=%d: %.3f us\n", pdl,
             spin_then([&] { cudaLaunchKernelEx(&cfg, empty_big, big); }));
      printf("cudaLaunchKernelEx 4-B param, pdl=%d: %.3f us\n", pdl,
             spin_then([&] { cudaLaunchKernelEx(&cfg, empty_small, 1); }));
    }
  }
  // (2) back to back: wall time per call incl. device execution
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, s);
  t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < K; ++i) call();
  cudaEventRecord(b, s);
  cudaStreamSynchronize(s);
  t1 = std::chrono::steady_clock::now();
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  printf("back to back: %.3f us/call (device events), %.3f us/call (wall)\n", ms * 1e3 / K,
         std::chrono::duration<double, std::micro>(t1 - t0).count() / K);
  // (3) the same calls in one CUDA graph
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < 100; ++i) call();
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaGraphLaunch(ge, s);
  cudaStreamSynchronize(s);
  cudaEventRecord(a, s);
  for (int i = 0; i < 20; ++i) cudaGraphLaunch(ge, s);
  cudaEventRecord(b, s);
  cudaStreamSynchronize(s);
  cudaEventElapsedTime(&ms, a, b);
  printf("graph: %.3f us/call (device)\n", ms * 1e3 / 2000);
  printf("async error: %d\n", adapcc_get_async_error(c));
  adapcc_finalize(c);
  return 0;
}
