// AdapCC transfer engine: one persistent sm_100a kernel per collective call.
//
// Each CTA repeatedly claims the next work item (task, chunk) from a per-rank
// counter, waits for the chunk's input flags (system-scope acquire; the
// paper's cudaStreamWaitEvent per chunk), folds its K source
// streams left to right with 128-bit loads (the aggregation kernel, P:L154,
// P:L265), writes the result to its D destinations -- local HBM, or a peer
// GPU's IPC-mapped arena over NVLink -- and posts the chunk's output flags
// (system-scope release; the paper's cudaEventRecord after
// cudaMemcpyPeerAsync).  Reduce and broadcast stages of every tree
// run in the same launch and pipeline chunk by chunk.
//
// Arithmetic (DESIGN.md §3 Q6): fp32 adds in IEEE RNE (__fadd_rn, no FTZ, no
// contraction); bf16 widened to fp32, folded, rounded ONCE per task with RNE;
// int32 wraps.  A single-source task without accumulation copies bytes
// unchanged (relay forwarding, broadcast).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"
#include "launch.hpp"

namespace adapcc {
namespace {

constexpr int kThreads = 256;
#ifndef ADAPCC_UNROLL
#define ADAPCC_UNROLL 8   // 128-bit vectors in flight per thread per source
#endif
#ifndef ADAPCC_MINB
#define ADAPCC_MINB 2     // resident CTAs per SM the register budget is sized for
#endif

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// 128-bit load/store; .cg keeps in-kernel-produced data out of L1
__device__ __forceinline__ uint4 ld16(const char* p) { return __ldcg(reinterpret_cast<const uint4*>(p)); }
__device__ __forceinline__ void st16(char* p, uint4 v) { __stcg(reinterpret_cast<uint4*>(p), v); }

// ------------------------------------------------------------ dtype traits
template <int DT> struct Ops;

template <> struct Ops<kF32> {
  static constexpr int kEsize = 4;
  struct Acc { float v[4]; };
  __device__ static Acc widen(uint4 x) {
    return {{__uint_as_float(x.x), __uint_as_float(x.y), __uint_as_float(x.z), __uint_as_float(x.w)}};
  }
  __device__ static void add(Acc& a, uint4 x) {
    a.v[0] = __fadd_rn(a.v[0], __uint_as_float(x.x));
    a.v[1] = __fadd_rn(a.v[1], __uint_as_float(x.y));
    a.v[2] = __fadd_rn(a.v[2], __uint_as_float(x.z));
    a.v[3] = __fadd_rn(a.v[3], __uint_as_float(x.w));
  }
  __device__ static uint4 narrow(const Acc& a) {
    return make_uint4(__float_as_uint(a.v[0]), __float_as_uint(a.v[1]), __float_as_uint(a.v[2]),
                      __float_as_uint(a.v[3]));
  }
  // scalar element path (misaligned slots / ragged tail)
  using E = uint32_t;
  __device__ static float w1(E x) { return __uint_as_float(x); }
  __device__ static float a1(float a, E x) { return __fadd_rn(a, __uint_as_float(x)); }
  __device__ static E n1(float a) { return __float_as_uint(a); }
};

template <> struct Ops<kBF16> {
  static constexpr int kEsize = 2;
  struct Acc { float v[8]; };
  __device__ static void w2(uint32_t p, float& lo, float& hi) {
    lo = __uint_as_float(p << 16);
    hi = __uint_as_float(p & 0xFFFF0000u);
  }
  __device__ static Acc widen(uint4 x) {
    Acc a;
    w2(x.x, a.v[0], a.v[1]);
    w2(x.y, a.v[2], a.v[3]);
    w2(x.z, a.v[4], a.v[5]);
    w2(x.w, a.v[6], a.v[7]);
    return a;
  }
  __device__ static void add(Acc& a, uint4 x) {
    Acc b = widen(x);
#pragma unroll
    for (int i = 0; i < 8; ++i) a.v[i] = __fadd_rn(a.v[i], b.v[i]);
  }
  __device__ static uint32_t n2(float lo, float hi) {
    __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);  // cvt.rn.bf16x2.f32: RNE
    return *reinterpret_cast<uint32_t*>(&h);
  }
  __device__ static uint4 narrow(const Acc& a) {
    return make_uint4(n2(a.v[0], a.v[1]), n2(a.v[2], a.v[3]), n2(a.v[4], a.v[5]), n2(a.v[6], a.v[7]));
  }
  using E = uint16_t;
  __device__ static float w1(E x) { return __uint_as_float(uint32_t(x) << 16); }
  __device__ static float a1(float a, E x) { return __fadd_rn(a, w1(x)); }
  __device__ static E n1(float a) {
    __nv_bfloat16 h = __float2bfloat16_rn(a);
    return *reinterpret_cast<uint16_t*>(&h);
  }
};

template <> struct Ops<kI32> {
  static constexpr int kEsize = 4;
  struct Acc { uint32_t v[4]; };
  __device__ static Acc widen(uint4 x) { return {{x.x, x.y, x.z, x.w}}; }
  __device__ static void add(Acc& a, uint4 x) {
    a.v[0] += x.x;  // unsigned: wraps mod 2^32 (reading Q15)
    a.v[1] += x.y;
    a.v[2] += x.z;
    a.v[3] += x.w;
  }
  __device__ static uint4 narrow(const Acc& a) { return make_uint4(a.v[0], a.v[1], a.v[2], a.v[3]); }
  using E = uint32_t;
  __device__ static uint32_t w1(E x) { return x; }
  __device__ static uint32_t a1(uint32_t a, E x) { return a + x; }
  __device__ static E n1(uint32_t a) { return a; }
};

struct Shared {
  const char* src[kMaxFold];
  char* dst[kMaxDst];
  uint8_t acc[kMaxDst];
  uint32_t item;
  int bad_align;
  int abort;
  int any_acc;
};

// ---------------------------------------------------------- vector fold
// Sources are folded one at a time with U 128-bit loads in flight per thread
// (U=8: 8 x 16 B x 256 threads x 2 CTAs = 64 KB in flight per SM, enough to
// cover HBM / NVLink latency); the accumulator stays in registers.  Vector
// indices are 32-bit (a chunk is at most 2^31 bytes).
template <int U>
__device__ __forceinline__ void load_u(uint4 (&x)[U], const char* src, uint32_t base, uint32_t nvec,
                                       bool full) {
  if (full) {
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = ld16(src + (size_t)(base + u * kThreads) * 16);
  } else {
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (base + u * kThreads < nvec) x[u] = ld16(src + (size_t)(base + u * kThreads) * 16);
  }
}

template <int U>
__device__ __forceinline__ void store_u(char* dst, const uint4 (&x)[U], uint32_t base, uint32_t nvec,
                                        bool full) {
  if (full) {
#pragma unroll
    for (int u = 0; u < U; ++u) st16(dst + (size_t)(base + u * kThreads) * 16, x[u]);
  } else {
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (base + u * kThreads < nvec) st16(dst + (size_t)(base + u * kThreads) * 16, x[u]);
  }
}

template <int DT, int U>
__device__ __forceinline__ void fold_vec(const Shared& sh, int nsrc, int ndst, uint32_t nvec) {
  using O = Ops<DT>;
  for (uint32_t base = threadIdx.x; base < nvec; base += U * kThreads) {
    const bool full = base + (U - 1) * kThreads < nvec;
    uint4 x[U];
    load_u<U>(x, sh.src[0], base, nvec, full);
    if (nsrc > 1) {
      typename O::Acc a[U];
#pragma unroll
      for (int u = 0; u < U; ++u) a[u] = O::widen(x[u]);
      for (int k = 1; k < nsrc; ++k) {
        load_u<U>(x, sh.src[k], base, nvec, full);
#pragma unroll
        for (int u = 0; u < U; ++u) O::add(a[u], x[u]);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) x[u] = O::narrow(a[u]);  // one rounding per task
    }
    for (int d = 0; d < ndst; ++d) {
      char* dst = sh.dst[d];
      if (sh.acc[d]) {  // recv += result (phase 2): one vector at a time
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const uint32_t v = base + u * kThreads;
          if (v < nvec) {
            typename O::Acc q = O::widen(ld16(dst + (size_t)v * 16));
            O::add(q, x[u]);
            st16(dst + (size_t)v * 16, O::narrow(q));
          }
        }
      } else {
        store_u<U>(dst, x, base, nvec, full);  // bytes unchanged when nsrc == 1
      }
    }
  }
}

// element path: e in [e_begin, e_end) relative to the chunk start
template <int DT>
__device__ __noinline__ void fold_scalar(const Shared& sh, int nsrc, int ndst, uint64_t e_begin,
                                            uint64_t e_end) {
  using O = Ops<DT>;
  using E = typename O::E;
  for (uint64_t e = e_begin + threadIdx.x; e < e_end; e += kThreads) {
    E x0 = *reinterpret_cast<const volatile E*>(sh.src[0] + e * sizeof(E));
    E r;
    if (nsrc == 1) {
      r = x0;
    } else {
      auto a = O::w1(x0);
      for (int k = 1; k < nsrc; ++k)
        a = O::a1(a, *reinterpret_cast<const volatile E*>(sh.src[k] + e * sizeof(E)));
      r = O::n1(a);
    }
    for (int d = 0; d < ndst; ++d) {
      E* p = reinterpret_cast<E*>(sh.dst[d] + e * sizeof(E));
      if (sh.acc[d]) {
        auto a = O::w1(*reinterpret_cast<volatile E*>(p));
        *p = O::n1(O::a1(a, r));
      } else {
        *p = r;
      }
    }
  }
}

template <int DT>
__device__ void fold_chunk(const Shared& sh, int nsrc, int ndst, uint64_t n, int op) {
  using O = Ops<DT>;
  using E = typename O::E;
  if (op == kOpZero) {
    for (int d = 0; d < ndst; ++d)
      for (uint64_t e = threadIdx.x; e < n; e += kThreads)
        reinterpret_cast<E*>(sh.dst[d])[e] = E(0);
    return;
  }
  if (sh.bad_align) {
    fold_scalar<DT>(sh, nsrc, ndst, 0, n);
    return;
  }
  constexpr int VE = 16 / O::kEsize;
  const uint64_t nvec = n / VE;
  fold_vec<DT, ADAPCC_UNROLL>(sh, nsrc, ndst, (uint32_t)nvec);
  if (nvec * VE < n) fold_scalar<DT>(sh, nsrc, ndst, nvec * VE, n);
}

// spin until *flag >= target; false on watchdog timeout or abort
__device__ bool wait_flag(const uint64_t* flag, uint64_t target, const LaunchParams& P) {
  if (ld_acquire_sys(flag) >= target) return true;
  const uint64_t t0 = globaltimer();
  for (uint32_t spin = 1;; ++spin) {
    if (ld_acquire_sys(flag) >= target) return true;
    if ((spin & 63) == 0) {
      if (*reinterpret_cast<volatile unsigned*>(&P.counters[2])) return false;
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicExch(&P.counters[2], 1u);
        *reinterpret_cast<volatile int*>(P.err) = 7;  // ADAPCC_ERR_TIMEOUT
        __threadfence_system();
        return false;
      }
    }
  }
}

__device__ __forceinline__ char* base_of(const LaunchParams& P, uint8_t kind, int rank) {
  return kind == kBufSend ? P.send[rank] : kind == kBufRecv ? P.recv[rank] : P.arena[rank];
}

template <int DT>
__global__ void __launch_bounds__(kThreads, ADAPCC_MINB) engine_kernel(const __grid_constant__ LaunchParams P) {
  __shared__ Shared sh;
  if (threadIdx.x == 0) sh.abort = 0;
  __syncthreads();
  // multi-process: every peer must have finished the call that last used this
  // parity half of the arenas (epoch - 2) before we write into any arena
  if (P.ipc && P.epoch > 2) {
    const int r = threadIdx.x;
    if (r < P.nranks && r != P.my_rank) {
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[r]), P.epoch - 2, P)) sh.abort = 1;
    }
  }
  __syncthreads();
  constexpr int esize = Ops<DT>::kEsize;
  while (!sh.abort) {
    if (threadIdx.x == 0) sh.item = atomicAdd(&P.counters[0], 1u);
    __syncthreads();
    const uint32_t it = sh.item;
    if (it >= P.nitems) break;
    const Item item = P.items[it];
    const Task& t = P.tasks[item.task];
    const int nsrc = t.nsrc, ndst = t.ndst;
    const uint64_t e0 = t.lo + (uint64_t)item.chunk * t.chunk_elems + item.off;
    const uint64_t e1 = e0 + item.len;
    const bool dropped = (int)t.owner == P.drop_rank;
    if (threadIdx.x == 0) { sh.bad_align = 0; sh.any_acc = 0; }
    __syncthreads();
    if (!dropped) {
      // input flags, one waiter thread per flag
      if (threadIdx.x < t.nwait) {
        const FlagRef f = P.flags[t.flag0 + threadIdx.x];
        const uint64_t* fl = reinterpret_cast<const uint64_t*>(P.arena[f.rank] + f.off) + item.chunk;
        if (!wait_flag(fl, P.epoch, P)) sh.abort = 1;
      }
      // resolve stream pointers for this chunk
      if (threadIdx.x < nsrc + ndst) {
        const BufRef r = P.refs[t.ref0 + threadIdx.x];
        char* p = base_of(P, r.kind, r.rank) + r.bias + (int64_t)(e0 * esize);
        if (reinterpret_cast<uintptr_t>(p) & 15) atomicOr(&sh.bad_align, 1);
        if (threadIdx.x < nsrc) {
          sh.src[threadIdx.x] = p;
        } else {
          sh.dst[threadIdx.x - nsrc] = p;
          sh.acc[threadIdx.x - nsrc] = r.accum;
          if (r.accum) atomicOr(&sh.any_acc, 1);
        }
      }
    }
    __syncthreads();
    if (sh.abort) break;
    if (!dropped) {
      fold_chunk<DT>(sh, nsrc, ndst, e1 - e0, t.op);
      __syncthreads();
      if (threadIdx.x == 0 && t.npost) {
        __threadfence_system();  // chunk bytes (incl. remote NVLink stores) before the flag
        for (int i = 0; i < t.npost; ++i) {
          const FlagRef f = P.flags[t.flag0 + t.nwait + i];
          st_release_sys(reinterpret_cast<uint64_t*>(P.arena[f.rank] + f.off) + item.chunk, P.epoch);
        }
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    const unsigned done = atomicAdd(&P.counters[1], 1u);
    if (done == gridDim.x - 1) {
      // last CTA: re-arm the counters for the next launch on this stream and
      // publish "this rank finished epoch" to the peers
      P.counters[0] = 0;
      P.counters[1] = 0;
      if (P.ipc) {
        __threadfence_system();
        st_release_sys(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank]), P.epoch);
      }
    }
  }
}

}  // namespace

int engine_threads() { return kThreads; }

cudaError_t engine_occupancy(int dtype, int* blocks_per_sm) {
  switch (dtype) {
    case kF32: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kF32>, kThreads, 0);
    case kBF16: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kBF16>, kThreads, 0);
    default: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kI32>, kThreads, 0);
  }
}

cudaError_t engine_launch(const LaunchParams& p, int grid, cudaStream_t stream) {
  switch (p.dtype) {
    case kF32: engine_kernel<kF32><<<grid, kThreads, 0, stream>>>(p); break;
    case kBF16: engine_kernel<kBF16><<<grid, kThreads, 0, stream>>>(p); break;
    default: engine_kernel<kI32><<<grid, kThreads, 0, stream>>>(p); break;
  }
  return cudaGetLastError();
}

}  // namespace adapcc
