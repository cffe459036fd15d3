// AdapCC transfer engine, flat variant: for plans in which no task waits for
// or posts a flag and none touches an arena (DIRECT plans -- loopback and
// zero-copy across processes -- where every fold reads its sources in place:
// the root of tree m folds slice m of every ready rank's input and writes the
// result to every rank's recvbuf).  Such tasks are
// independent, so there are no work items and no claim counter: the vectors
// of all tasks are concatenated into one index space that the whole grid
// strides through (thread g: vectors g, g + grid x 256, ...), every CTA
// holding every task's stream pointers in shared memory (resolved once, from
// a plan-time descriptor blob read in one round trip before the stream-order
// wait).  At any moment the grid works in one narrow window of the streams,
// and a small call still spreads its tasks over the whole grid.
//
// Per 16-byte vector the K sources are loaded KB at a time and folded left to
// right in the strategy's order (one rounding, DESIGN.md §3 Q6); then -- for
// accumulating destinations (phase 2, recv += result) -- the recv
// vectors of up to 8 destinations are loaded together before their adds and
// stores: one memory round trip per 8 destinations instead of one per
// destination (engine.cu write_dsts), which is what phase 2 at 16-100 MiB per
// rank is bound by (loads in flight per SM, scripts/debug/acc_ceiling.py).
//
// Same epoch / counter / multi-process protocol as engine.cu: the launch's
// epoch is the one the previous launch published + 1, block 0 re-arms the
// other parity's counters, the last CTA to finish publishes the epoch (and,
// across processes, its done word); zero-copy calls keep the entry / exit
// barriers on the peers' arena headers.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"
#include "engine_common.cuh"
#include "launch.hpp"

namespace adapcc {
namespace flat {
namespace {

using namespace dev;

constexpr int kThreads = 256;
constexpr int kMinBlocks = 2;  // 128 registers (the 8-destination batch needs 72-92 plus the loop state)
constexpr int kDB = 8;         // accumulating destinations loaded together

struct Shared {
  uint64_t epoch;
  uint64_t nvec;                  // vectors of the launch's vector space
  uint64_t t_entry, t_ready, t0;  // trace (kept here, not in registers)
  int abort;
};

// one task's streams, as the fold loops see them (pointer arrays in shared
// memory, re-read at every use: kept in registers across the loops they would
// cost 2 registers each)
struct View {
  char* const* p;         // sources, then destinations
  const uint8_t* acc;     // per destination
  int nsrc, ndst;
  __device__ __forceinline__ const char* src(int k) const { return const_cast<char* const volatile*>(p)[k]; }
  __device__ __forceinline__ char* dst(int k) const { return const_cast<char* const volatile*>(p)[nsrc + k]; }
  __device__ __forceinline__ bool is_acc(int k) const { return const_cast<const volatile uint8_t*>(acc)[k] != 0; }
};

// K sources folded KB at a time (KB vectors of loads in flight), one rounding
template <int DT, int KB>
__device__ __forceinline__ uint4 fold_sources(const View& w, size_t off) {
  using O = Ops<DT>;
  if (w.nsrc == 1) return ld16(w.src(0) + off);
  typename O::Acc a;
#pragma unroll 1
  for (int k0 = 0; k0 < w.nsrc; k0 += KB) {
    uint4 x[KB];
#pragma unroll
    for (int j = 0; j < KB; ++j)
      if (k0 + j < w.nsrc) x[j] = ld16(w.src(k0 + j) + off);
    if (k0 == 0) a = O::widen(x[0]);
    else O::add(a, x[0]);
#pragma unroll
    for (int j = 1; j < KB; ++j)
      if (k0 + j < w.nsrc) O::add(a, x[j]);
  }
  return O::narrow(a);
}

// one 16-byte vector (byte offset off) of one task
template <int DT>
__device__ __forceinline__ void fold_vector(const View& w, bool any_acc, size_t off) {
  using O = Ops<DT>;
  const uint4 r = fold_sources<DT, 4>(w, off);
  if (!any_acc) {
#pragma unroll 1
    for (int d = 0; d < w.ndst; ++d) st16(w.dst(d) + off, r);
    return;
  }
#pragma unroll 1
  for (int d0 = 0; d0 < w.ndst; d0 += kDB) {
    const int nb = min(kDB, w.ndst - d0);
    uint4 q[kDB];
#pragma unroll
    for (int j = 0; j < kDB; ++j)
      if (j < nb && w.is_acc(d0 + j)) q[j] = ld16(w.dst(d0 + j) + off);
#pragma unroll
    for (int j = 0; j < kDB; ++j) {
      if (j < nb) {
        uint4 o = r;
        if (w.is_acc(d0 + j)) {  // recv + result, rounded once (as engine.cu write_dsts)
          typename O::Acc b = O::widen(q[j]);
          O::add(b, r);
          o = O::narrow(b);
        }
        st16(w.dst(d0 + j) + off, o);
      }
    }
  }
}

// element path: misaligned streams and the sub-16-byte tail, e = e0, e0 + stride, ...
template <int DT>
__device__ void fold_scalar(const View& w, uint64_t e0, uint64_t e_end, uint64_t stride) {
  using O = Ops<DT>;
  using E = typename O::E;
  for (uint64_t e = e0; e < e_end; e += stride) {
    E r;
    const E x0 = *reinterpret_cast<const E*>(w.src(0) + e * sizeof(E));
    if (w.nsrc == 1) {
      r = x0;
    } else {
      auto a = O::w1(x0);
      for (int k = 1; k < w.nsrc; ++k) a = O::a1(a, *reinterpret_cast<const E*>(w.src(k) + e * sizeof(E)));
      r = O::n1(a);
    }
    for (int d = 0; d < w.ndst; ++d) {
      E* p = reinterpret_cast<E*>(w.dst(d) + e * sizeof(E));
      *p = w.is_acc(d) ? O::n1(O::a1(O::w1(*p), r)) : r;
    }
  }
}

// Dynamic shared memory (flat_smem_bytes): the descriptor blob (FlatTask x
// ntasks, then the BufRefs; P.first / P.first_words / P.ntasks), then one
// pointer per ref, then one accumulate flag per ref.
template <int DT, int NR>
__global__ void __launch_bounds__(kThreads, kMinBlocks) flat_kernel(const __grid_constant__ LaunchParamsT<NR> P) {
  __shared__ Shared sh;
  extern __shared__ __align__(16) unsigned char dsm[];
  uint4* words = reinterpret_cast<uint4*>(dsm);
  FlatTask* ft = reinterpret_cast<FlatTask*>(dsm);
  const uint32_t nrefs = flat_nrefs(P.first_words, P.ntasks);
  const BufRef* refs = reinterpret_cast<const BufRef*>(dsm + (size_t)P.ntasks * sizeof(FlatTask));
  char** ptrs = reinterpret_cast<char**>(dsm + (size_t)P.first_words * 16);
  uint8_t* accs = reinterpret_cast<uint8_t*>(ptrs + nrefs);
  constexpr int esize = Ops<DT>::kEsize;
  if (threadIdx.x == 0) {
    sh.abort = 0;
    sh.t_entry = P.trace ? globaltimer() : 0;
  }
  // plan descriptors: immutable, read (one round trip) and resolved before
  // the stream-order wait -- under PDL this overlaps the previous kernel
  for (uint32_t i = threadIdx.x; i < P.first_words; i += kThreads) words[i] = P.first[i];
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < nrefs; i += kThreads) {
    const BufRef r = refs[i];
    char* p = (r.kind == kBufSend ? P.send[r.rank] : P.recv[r.rank]) + r.bias;  // (bias includes the task's lo)
    ptrs[i] = p;
    accs[i] = r.accum;
    // (pad[0..1]: the ref's task; every thread that finds a misaligned stream writes the same 1)
    if (reinterpret_cast<uintptr_t>(p) & 15) ft[r.pad[0] | (r.pad[1] << 8)].bad = 1;
  }
  __syncthreads();
  if (threadIdx.x == 0) {  // the launch's vector space: folding, aligned tasks (len / VE vectors each)
    uint64_t n = 0;
    for (uint32_t i = 0; i < P.ntasks; ++i) {
      FlatTask& t = ft[i];
      const bool vec = (int)t.owner != P.drop_rank && t.op == kOpFold && !t.bad;
      t.vstart = n;
      if (vec) n += t.len / (16 / esize);
    }
    sh.nvec = n;
  }
  __syncthreads();
  pdl_trigger();
  pdl_wait();
  // The epoch, counters and user buffers belong to the stream order.  In
  // loopback the epoch only counts this launch done at the end, so its load
  // stays in flight during the fold (no round trip and barrier up front);
  // across processes the start checks below need it first.
  uint64_t e_lazy = 0;
  if (!P.ipc) {
    if (threadIdx.x == 0) e_lazy = *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) + 1;
  } else {
    if (threadIdx.x == 0) {
      const uint64_t e = *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) + 1;
      sh.epoch = e;
      if (blockIdx.x == 0) {  // re-arm the other parity's counters for the next launch
        P.state->work[(e + 1) & 1] = 0;
        P.state->done[(e + 1) & 1] = 0;
      }
    }
    __syncthreads();
  }
  const uint64_t epoch = P.ipc ? sh.epoch : 0;  // (loopback: e_lazy, thread 0, at the end)
  if (P.ipc && epoch > 2) {  // peers done with the call before last (same start check as the engines)
    const int r = threadIdx.x;
    if (r < P.nranks && r != P.my_rank && ((P.members >> r) & 1))
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[r]), epoch - 2, P)) sh.abort = 1;
    __syncthreads();
  }
  if (P.ipc && P.check_sig && !check_call_sig(P, epoch)) sh.abort = 1;  // before any byte moves
  if (P.ipc && P.zc) {  // zero-copy: peers read / write our user buffers directly
    if (blockIdx.x == 0 && threadIdx.x == 0)
      st_release(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank] + ArenaHeader::kEntered), epoch, true);
    if (threadIdx.x < P.nranks && threadIdx.x != P.my_rank && ((P.members >> threadIdx.x) & 1))
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[threadIdx.x] + ArenaHeader::kEntered), epoch, P))
        sh.abort = 1;
    __syncthreads();
  }
  if (P.trace && threadIdx.x == 0) sh.t_ready = globaltimer();
  const uint32_t gthreads = gridDim.x * kThreads;
  const uint32_t gtid = blockIdx.x * kThreads + threadIdx.x;
  using E = typename Ops<DT>::E;
  constexpr int VE = 16 / esize;
  if (!sh.abort) {
    // the vectors of all folding tasks, concatenated: thread g handles g,
    // g + grid x 256, ... -- consecutive threads, consecutive vectors, and a
    // small call still spreads its tasks over the whole grid
    uint32_t ti = 0;
#pragma unroll 1
    for (uint64_t v = gtid; v < sh.nvec; v += gthreads) {
      while (ti + 1 < P.ntasks && v >= ft[ti + 1].vstart) ++ti;  // (tasks without vectors: empty ranges)
      const FlatTask& t = ft[ti];
      const View w{ptrs + t.ref0, accs + t.ref0 + t.nsrc, (int)t.nsrc, (int)t.ndst};
      fold_vector<DT>(w, t.any_acc != 0, (size_t)(v - t.vstart) * 16);
    }
    // rare: zero tasks, misaligned streams, and the sub-16-byte tails
    for (uint32_t tj = 0; tj < P.ntasks; ++tj) {
      const FlatTask& t = ft[tj];
      if ((int)t.owner == P.drop_rank || t.op == kOpNone) continue;  // (test hook: a dropped rank's tasks)
      const View w{ptrs + t.ref0, accs + t.ref0 + t.nsrc, (int)t.nsrc, (int)t.ndst};
      if (t.op == kOpZero) {
        for (int d = 0; d < w.ndst; ++d)
          for (uint64_t e = gtid; e < t.len; e += gthreads) reinterpret_cast<E*>(w.dst(d))[e] = E(0);
      } else if (t.bad) {
        fold_scalar<DT>(w, gtid, t.len, gthreads);
      } else if (t.len % VE) {
        fold_scalar<DT>(w, t.len / VE * VE + gtid, t.len, gthreads);
      }
    }
  }
  __syncthreads();
  if (P.trace && threadIdx.x == 0) trace_put(P, kTraceCta, 0, sh.t_entry, sh.t_ready, globaltimer(), 0);
  if (threadIdx.x == 0) {
    // across processes the done word published to peers follows every CTA's
    // data; in loopback only the next launch reads anything, after this grid
    // has completed
    if (P.ipc) fence(true);
    const uint64_t ep = P.ipc ? epoch : e_lazy;
    if (!P.ipc && blockIdx.x == 0) {  // re-arm the other parity's counters for the next launch
      P.state->work[(ep + 1) & 1] = 0;
      P.state->done[(ep + 1) & 1] = 0;
    }
    const unsigned done = atomicAdd(&P.state->done[ep & 1], 1u);
    if (done == gridDim.x - 1) {
      *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) = ep;
      if (P.ipc) {
        __threadfence_system();
        st_release(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank]), epoch, true);
        if (P.zc)  // our buffers stay in use until every peer has finished this call
          for (int q = 0; q < P.nranks; ++q)
            if (q != P.my_rank && ((P.members >> q) & 1))
              wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[q]), epoch, P);
      }
    }
  }
}

template <int NR>
cudaError_t launch_nr(const LaunchParamsT<NR>& p, int grid, cudaStream_t stream, bool pdl) {
  const size_t smem = flat_smem_bytes(p.first_words, p.ntasks);
  switch (p.dtype) {
    case kF32: return launch_kernel(flat_kernel<kF32, NR>, grid, kThreads, smem, stream, pdl, p);
    case kBF16: return launch_kernel(flat_kernel<kBF16, NR>, grid, kThreads, smem, stream, pdl, p);
    default: return launch_kernel(flat_kernel<kI32, NR>, grid, kThreads, smem, stream, pdl, p);
  }
}

}  // namespace

cudaError_t launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl) {
  cudaGetLastError();
  if (p.nranks <= kNarrowRanks) return launch_nr(narrow(p), grid, stream, pdl);
  return launch_nr(p, grid, stream, pdl);
}

}  // namespace flat
}  // namespace adapcc
