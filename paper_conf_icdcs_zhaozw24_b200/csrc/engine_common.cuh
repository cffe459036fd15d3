// Device helpers shared by the transfer-engine kernels (engine.cu: 128-bit
// LDG/STG fold; engine_tma.cu: TMA bulk-copy pipeline).  Internal header.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"
#include "launch.hpp"

namespace adapcc {
namespace dev {

__device__ __forceinline__ uint64_t ld_acquire(const uint64_t* p, bool sys) {
  uint64_t v;
  if (sys) asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  else asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint64_t* p, uint64_t v, bool sys) {
  if (sys) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence(bool sys) {
  if (sys) __threadfence_system();
  else __threadfence();
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Programmatic dependent launch (PDL): a launch with
// cudaLaunchAttributeProgrammaticStreamSerialization may start while the
// previous kernel on the stream is still running.  Everything before
// pdl_wait() may only touch immutable plan tables and shared memory;
// pdl_wait() returns once the previous grid has completed and its memory is
// visible (a no-op when the launch had no such dependency).  pdl_trigger()
// lets the next launch start its own prologue early.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// appends one trace record (tracing is a debug mode: one atomic per record)
template <class LP>
__device__ __forceinline__ void trace_put(const LP& P, uint32_t item, uint32_t task, uint64_t t0,
                                          uint64_t t1, uint64_t t2, uint64_t bytes) {
  const unsigned i = atomicAdd(P.trace_n, 1u);
  if (i < P.trace_cap) P.trace[i] = TraceRec{P.launch_seq, blockIdx.x, item, task, t0, t1, t2, bytes};
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


// spin until *flag >= target; false on watchdog timeout or abort
template <class LP>
static __device__ __noinline__ bool wait_flag(const uint64_t* flag, uint64_t target, const LP& P) {
  const bool sys = P.ipc;
  if (ld_acquire(flag, sys) >= target) return true;
  const uint64_t t0 = globaltimer();
  for (uint32_t spin = 1;; ++spin) {
    if (ld_acquire(flag, sys) >= target) return true;
    if ((spin & 63) == 0) {
      if (*reinterpret_cast<volatile unsigned*>(&P.state->abort)) return false;
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicExch(&P.state->abort, 1u);
        *reinterpret_cast<volatile int*>(P.err) = 7;  // ADAPCC_ERR_TIMEOUT
        __threadfence_system();
        return false;
      }
    }
  }
}


// Debug-mode call check (mismatched calls fail loudly instead of
// corrupting data or hanging).  Block 0 publishes this rank's call signature
// for `epoch` in its arena header (slot epoch & 3: peers run at most one epoch
// apart, the parity-half start check bounds them); every CTA then compares it
// with every live peer's signature for the same epoch before moving any byte.
// A mismatch latches ADAPCC_ERR_MISMATCH and raises the abort flag.  Returns
// false on mismatch or watchdog timeout.  Called by all threads of the CTA.
template <class LP>
static __device__ bool check_call_sig(const LP& P, uint64_t epoch) {
  const int slot = (int)(epoch & 3);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    char* me = P.hdr[P.my_rank];
    *reinterpret_cast<volatile uint64_t*>(me + ArenaHeader::kSig + 8 * slot) = P.sig;
    st_release(reinterpret_cast<uint64_t*>(me + ArenaHeader::kSigEpoch + 8 * slot), epoch, true);
  }
  int bad = 0;
  const int r = threadIdx.x;
  if (r < P.nranks && r != P.my_rank && ((P.members >> r) & 1)) {
    const char* peer = P.hdr[r];
    if (!wait_flag(reinterpret_cast<const uint64_t*>(peer + ArenaHeader::kSigEpoch + 8 * slot), epoch, P)) {
      bad = 1;
    } else if (*reinterpret_cast<const volatile uint64_t*>(peer + ArenaHeader::kSig + 8 * slot) != P.sig) {
      *reinterpret_cast<volatile int*>(P.err) = 8;  // ADAPCC_ERR_MISMATCH
      atomicExch(&P.state->abort, 1u);
      __threadfence_system();
      bad = 1;
    }
  }
  return __syncthreads_or(bad) == 0;
}

// Late join ("data chunks with the same offset ... join the ongoing
// aggregation"): which of a root task's nlate candidate ranks take part in
// work item `item`.  Mode 1 (phase 1): candidates whose ready word
// (arena header + 16) reached the call's ticket, recorded in late_bits[item];
// mode 2 (phase 2): the candidates NOT recorded (only they remain to add).
// Position of the next entry in the plan's phase-2 list for the phase-1
// launch of `epoch`: the first append of a new launch (gen differs) restarts
// the count at 0 with one compare-and-swap; every later append of the launch
// is a plain atomicAdd on the count half (no retry loop: a CAS per append
// serialised a phase 1 that lists hundreds of items, launch.hpp late_count).
template <class LP>
static __device__ __forceinline__ uint32_t late_append(const LP& P, uint64_t epoch) {
  const unsigned long long gen = (unsigned long long)(uint32_t)epoch;
  unsigned long long old = *reinterpret_cast<volatile unsigned long long*>(&P.late_count[0]);
  while ((old >> 32) != gen) {
    const unsigned long long prev = atomicCAS(&P.late_count[0], old, (gen << 32) | 1ull);
    if (prev == old) return 0u;   // this launch's first entry
    old = prev;                   // someone else moved it: retry only while the gen is stale
  }
  return (uint32_t)atomicAdd(&P.late_count[0], 1ull);
}

// Entries phase 2 runs: the list of the last completed phase 1, if any.
template <class LP>
static __device__ __forceinline__ uint32_t late_listed(const LP& P) {
  const unsigned long long w = *reinterpret_cast<volatile unsigned long long*>(&P.late_count[0]);
  const unsigned long long g = *reinterpret_cast<volatile unsigned long long*>(&P.late_count[1]);
  return g != ~0ull && (w >> 32) == (unsigned long long)(uint32_t)g ? (uint32_t)w : 0u;
}

template <class LP>
static __device__ __forceinline__ uint64_t late_select(const LP& P, const Task& t,
                                                       uint32_t item, uint64_t epoch) {
  uint64_t m = 0;
  if (P.late_mode == 1) {
    for (int j = 0; j < t.nlate; ++j) {
      const BufRef r = P.refs[t.ref0 + t.nsrc + t.ndst + j];
      if (ld_acquire(reinterpret_cast<const uint64_t*>(P.hdr[r.rank] + ArenaHeader::kReady), P.ipc) >=
          P.late_ticket)
        m |= 1ull << j;
    }
    P.late_bits[item] = m;
    const uint64_t all = t.nlate >= 64 ? ~0ull : ((1ull << t.nlate) - 1);
    if (all & ~m) P.late_list[late_append(P, epoch)] = item;  // phase 2 has something to add here
  } else if (P.late_mode == 2) {
    const uint64_t all = t.nlate >= 64 ? ~0ull : ((1ull << t.nlate) - 1);
    m = all & ~P.late_bits[item];
  }
  return m;
}

// late_select for a whole warp (the TMA kernel's producer): lane j checks
// candidate j (and j + 32, ...), so the ref and ready-word loads of all
// candidates are in flight together instead of one candidate after another.
// Same result and side effects as late_select; every lane returns the mask.
template <class LP>
static __device__ __forceinline__ uint64_t late_select_warp(const LP& P, const Task& t,
                                                            uint32_t item, int lane, uint64_t epoch) {
  const uint64_t all = t.nlate >= 64 ? ~0ull : ((1ull << t.nlate) - 1);
  if (P.late_mode == 2) return all & ~P.late_bits[item];
  if (P.late_mode != 1) return 0;
  uint64_t m = 0;
  for (int j0 = 0; j0 < t.nlate; j0 += 32) {
    const int j = j0 + lane;
    bool ok = false;
    if (j < t.nlate) {
      const BufRef r = P.refs[t.ref0 + t.nsrc + t.ndst + j];
      ok = ld_acquire(reinterpret_cast<const uint64_t*>(P.hdr[r.rank] + ArenaHeader::kReady), P.ipc) >=
           P.late_ticket;
    }
    m |= (uint64_t)__ballot_sync(0xffffffffu, ok) << j0;
  }
  if (lane == 0) {
    P.late_bits[item] = m;
    if (all & ~m) P.late_list[late_append(P, epoch)] = item;  // phase 2 has something to add here
  }
  return m;
}

// index (into the task's late refs) of the k-th set bit of m
static __device__ __forceinline__ int nth_bit(uint64_t m, int k) {
  for (int j = 0; j < 64; ++j)
    if ((m >> j) & 1) {
      if (k == 0) return j;
      --k;
    }
  return 0;
}

}  // namespace dev

// Kernel launch, optionally as a programmatic dependent launch (see pdl_wait).
template <typename Kernel, class LP>
inline cudaError_t launch_kernel(Kernel kernel, int grid, int threads, size_t smem, cudaStream_t stream,
                                 bool pdl, const LP& p) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3((unsigned)threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kernel, p);
}
}  // namespace adapcc
