// Ceiling probe for phase-2 ACCUMULATE (recv_g += x_a + x_b for 8 recvbufs):
// plain kernels outside the engine, to tell the engine's per-launch overhead
// from what the memory system gives at 16-100 MiB per rank.
//   ldst:  per 16-byte vector: fold the sources, then load/add/store every recv
//   red:   fold, then red.global.add.v4.f32 into every recv (L2 atomics, no
//          load round trip in the SM)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC
//        -o acc_ceiling.so acc_ceiling.cu
#include <cuda_runtime.h>
#include <stdint.h>

struct Ptrs {
  const float4* src[2];
  float4* dst[8];
};

template <int U>
__global__ void __launch_bounds__(512) k_ldst(Ptrs p, uint64_t nvec) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nvec; v0 += stride * U) {
    float4 a[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t v = v0 + u * stride;
      if (v < nvec) {
        float4 x = __ldcs(p.src[0] + v), y = __ldcs(p.src[1] + v);
        a[u] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + y.w);
      }
    }
#pragma unroll
    for (int g = 0; g < 8; ++g) {
      float4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec) r[u] = p.dst[g][v];
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec)
          p.dst[g][v] = make_float4(r[u].x + a[u].x, r[u].y + a[u].y, r[u].z + a[u].z, r[u].w + a[u].w);
      }
    }
  }
}

__device__ __forceinline__ void red_v4(float4* p, float4 a) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(a.z), "f"(a.w)
               : "memory");
}

template <int U>
__global__ void __launch_bounds__(512) k_red(Ptrs p, uint64_t nvec) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nvec; v0 += stride * U) {
    float4 a[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t v = v0 + u * stride;
      if (v < nvec) {
        float4 x = __ldcs(p.src[0] + v), y = __ldcs(p.src[1] + v);
        a[u] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + y.w);
      }
    }
#pragma unroll
    for (int g = 0; g < 8; ++g)
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec) red_v4(p.dst[g] + v, a[u]);
      }
  }
}

// all 8 destinations' loads issued before the first store (one memory round
// trip per vector group instead of one per destination)
template <int U>
__global__ void __launch_bounds__(256) k_batch(Ptrs p, uint64_t nvec) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nvec; v0 += stride * U) {
    float4 a[U], r[8][U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t v = v0 + u * stride;
      if (v < nvec) {
        float4 x = __ldcs(p.src[0] + v), y = __ldcs(p.src[1] + v);
        a[u] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + y.w);
#pragma unroll
        for (int g = 0; g < 8; ++g) r[g][u] = p.dst[g][v];
      }
    }
#pragma unroll
    for (int g = 0; g < 8; ++g)
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec)
          p.dst[g][v] = make_float4(r[g][u].x + a[u].x, r[g][u].y + a[u].y, r[g][u].z + a[u].z, r[g][u].w + a[u].w);
      }
  }
}

// plain AllReduce shape: fold 8 sources, store the sum to 8 destinations
struct Ptrs8 {
  const float4* src[8];
  float4* dst[8];
};
template <int U>
__global__ void __launch_bounds__(256) k_ar(Ptrs8 p, uint64_t nvec) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nvec; v0 += stride * U) {
    float4 x[8][U];
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec) x[k][u] = __ldcs(p.src[k] + v);
      }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      float4 a = x[0][u];
#pragma unroll
      for (int k = 1; k < 8; ++k) a = make_float4(a.x + x[k][u].x, a.y + x[k][u].y, a.z + x[k][u].z, a.w + x[k][u].w);
      x[0][u] = a;
    }
#pragma unroll
    for (int g = 0; g < 8; ++g)
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + u * stride;
        if (v < nvec) p.dst[g][v] = x[0][u];
      }
  }
}

extern "C" int ar_launch(int unroll, void* const* src, void* const* dst, uint64_t nvec, int grid, int block,
                         cudaStream_t st) {
  Ptrs8 p;
  for (int g = 0; g < 8; ++g) {
    p.src[g] = (const float4*)src[g];
    p.dst[g] = (float4*)dst[g];
  }
  if (unroll == 1) k_ar<1><<<grid, block, 0, st>>>(p, nvec);
  else k_ar<2><<<grid, block, 0, st>>>(p, nvec);
  return (int)cudaGetLastError();
}

extern "C" int acc_launch(int kind, int unroll, const void* s0, const void* s1, void* const* dst, uint64_t nvec,
                          int grid, int block, cudaStream_t st) {
  Ptrs p;
  p.src[0] = (const float4*)s0;
  p.src[1] = (const float4*)s1;
  for (int g = 0; g < 8; ++g) p.dst[g] = (float4*)dst[g];
#define L(K, U) K<U><<<grid, block, 0, st>>>(p, nvec)
  if (kind == 0) {
    if (unroll == 1) L(k_ldst, 1); else if (unroll == 2) L(k_ldst, 2); else L(k_ldst, 4);
  } else if (kind == 2) {
    if (unroll == 1) L(k_batch, 1); else L(k_batch, 2);
  } else {
    if (unroll == 1) L(k_red, 1); else if (unroll == 2) L(k_red, 2); else L(k_red, 4);
  }
  return (int)cudaGetLastError();
}
