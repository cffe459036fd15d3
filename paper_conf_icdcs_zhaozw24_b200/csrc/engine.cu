// AdapCC transfer engine: one persistent sm_100a kernel per collective call.
//
// Each CTA repeatedly claims the next work item (task, chunk, piece) from a
// per-rank counter, waits for the chunk's input flags (acquire; the paper's
// cudaStreamWaitEvent per chunk), folds its K source streams left
// to right with 128-bit loads (the aggregation kernel), writes
// the result to its D destinations -- local HBM, or a peer GPU's IPC-mapped
// arena over NVLink -- and posts the chunk's output flags (release; the
// paper's cudaEventRecord after cudaMemcpyPeerAsync).  Reduce and
// broadcast stages of every tree run in the same launch and pipeline chunk by
// chunk.
//
// Arithmetic (DESIGN.md §3 Q6): fp32 adds in IEEE RNE (__fadd_rn, no FTZ, no
// contraction); bf16 widened to fp32, folded, rounded ONCE per task with RNE;
// int32 wraps.  A single-source task without accumulation copies bytes
// unchanged (relay forwarding, broadcast).
//
// Epochs live on the device (DevState): every launch reads the epoch the
// previous launch on this communicator published, so captured CUDA graphs can
// be replayed any number of times.  Memory-model scope: .gpu in loopback (one
// device), .sys across processes / GPUs.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"
#include "engine_common.cuh"
#include "launch.hpp"

namespace adapcc {
namespace {

using namespace dev;

constexpr int kThreads = 256;
#ifndef ADAPCC_MINB
#define ADAPCC_MINB 2     // resident CTAs per SM the register budget is sized for
#endif
#ifndef ADAPCC_COPY_UNROLL
#define ADAPCC_COPY_UNROLL 4  // 128-bit vectors in flight per thread for 1-source tasks
#endif




struct Cur {  // header of the work item being executed (staged by thread 0)
  uint64_t e0;
  uint64_t late;            // late-join sources of this piece (bit j: late ref j)
  uint32_t ref0, flag0, chunk, len;
  uint16_t nsrc, ndst, nwait, npost, op;
  uint16_t tnsrc, nreg;     // task's own source count; regular sources used
  bool dropped, force_acc;
  int8_t blob;              // refs come from blob buffer `blob` in shared memory (-1: from P.refs)
  // STAGED late join (LateKind): decision words
  uint8_t lkind, decide;    // decide: sources / op are fixed after the waits (decision words)
  uint8_t dec_dst, dec_out; // write dec_out into the decision word of every arena destination
  uint16_t tnwait, wait0, tnlate;  // task's wait count; first wait used; late candidates
  uint64_t tlo;             // task range start and chunk count (decision-word addresses)
  uint32_t tnch;
};

struct Shared {
  uint64_t tr0, tr1;           // trace: item claimed / inputs ready
  uint4 blob[2][kFirstMaxWords];  // item blobs: Item | Task | refs (static schedule: double-buffered)
  Cur cur;
  const char* src[kMaxFold];
  char* dst[kMaxDst];
  uint8_t acc[kMaxDst];
  uint64_t epoch;
  uint32_t item;
  uint32_t claim;              // claim index of `item` (= item, or its position in the phase-2 list)
  uint32_t nclaim;             // claimable indices (nitems, or the phase-2 list length)
  int bad_align;
  int abort;
  int any_acc;
  int nvls_alias;              // the item touches the NVLS scratch (unicast and multicast aliases)
};

// 16-byte global -> shared copy that completes asynchronously (blob prefetch)
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// ---------------------------------------------------------------- vector fold
// Thread t handles vectors base, base + 256, ..., base + (U-1)*256 of a
// stride of U*256 vectors; addresses are one per-stream pointer plus
// immediate offsets (keeps the register count low).
template <int U>
__device__ __forceinline__ void load_u(uint4 (&x)[U], const char* p, uint32_t base, uint32_t nvec,
                                       bool full) {
#pragma unroll
  for (int u = 0; u < U; ++u)
    if (full || base + u * kThreads < nvec) x[u] = ld16(p + u * kThreads * 16);
}

template <int U>
__device__ __forceinline__ void store_u(char* p, const uint4 (&x)[U], uint32_t base, uint32_t nvec,
                                        bool full) {
#pragma unroll
  for (int u = 0; u < U; ++u)
    if (full || base + u * kThreads < nvec) st16(p + u * kThreads * 16, x[u]);
}

template <int DT, int U>
__device__ __forceinline__ void write_dsts(const Shared& sh, int ndst, const uint4 (&x)[U], uint32_t base,
                                           uint32_t nvec, bool full) {
  using O = Ops<DT>;
  const size_t off = (size_t)base * 16;
  for (int d = 0; d < ndst; ++d) {
    char* p = sh.dst[d] + off;
    if (sh.acc[d]) {  // recv += result (phase 2): one vector at a time
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (full || base + u * kThreads < nvec) {
          typename O::Acc q = O::widen(ld16(p + u * kThreads * 16));
          O::add(q, x[u]);
          st16(p + u * kThreads * 16, O::narrow(q));
        }
      }
    } else {
      store_u<U>(p, x, base, nvec, full);
    }
  }
}

// One source: bytes unchanged (relay forwarding, broadcast, AllGather,
// AlltoAll), U vectors in flight per thread.
template <int DT, int U>
__device__ __forceinline__ void copy_vec(const Shared& sh, int ndst, uint32_t nvec) {
  for (uint32_t base = threadIdx.x; base < nvec; base += U * kThreads) {
    const bool full = base + (U - 1) * kThreads < nvec;
    uint4 x[U];
    load_u<U>(x, sh.src[0] + (size_t)base * 16, base, nvec, full);
    write_dsts<DT, U>(sh, ndst, x, base, nvec, full);
  }
}

// K >= 2 sources: KB sources x U vectors of loads are issued before the first
// add (KB*U = 8 loads in flight per thread; a small chunk costs one memory
// round trip per KB sources instead of one per source).
template <int DT, int U, int KB>
__device__ __forceinline__ void fold_vec(const Shared& sh, int nsrc, int ndst, uint32_t nvec) {
  using O = Ops<DT>;
  for (uint32_t base = threadIdx.x; base < nvec; base += U * kThreads) {
    const bool full = base + (U - 1) * kThreads < nvec;
    const size_t off = (size_t)base * 16;
    typename O::Acc a[U];
    for (int k0 = 0; k0 < nsrc; k0 += KB) {
      uint4 x[KB][U];
#pragma unroll
      for (int j = 0; j < KB; ++j)
        if (k0 + j < nsrc) load_u<U>(x[j], sh.src[k0 + j] + off, base, nvec, full);
#pragma unroll
      for (int j = 0; j < KB; ++j) {
        if (k0 + j >= nsrc) break;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (k0 + j == 0) a[u] = O::widen(x[0][u]);
          else O::add(a[u], x[j][u]);
        }
      }
    }
    uint4 r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = O::narrow(a[u]);  // one rounding per task
    write_dsts<DT, U>(sh, ndst, r, base, nvec, full);
  }
}

// Items with accumulating destinations (phase 2, recv += result): one vector
// per thread per round; the sources are folded KB at a time as in fold_vec,
// then the recv vectors of DB destinations are loaded together before their
// adds and stores -- one memory round trip per DB destinations instead of one
// per destination (write_dsts), 8 loads in flight per thread.  Same
// arithmetic: fold rounded once, then recv + result rounded once.
template <int DT, int KB, int DB>
__device__ __forceinline__ void fold_acc_vec(const Shared& sh, int nsrc, int ndst, uint32_t nvec) {
  using O = Ops<DT>;
  for (uint32_t v = threadIdx.x; v < nvec; v += kThreads) {
    const size_t off = (size_t)v * 16;
    uint4 r;
    if (nsrc == 1) {
      r = ld16(sh.src[0] + off);
    } else {
      typename O::Acc a;
      for (int k0 = 0; k0 < nsrc; k0 += KB) {
        uint4 x[KB];
#pragma unroll
        for (int j = 0; j < KB; ++j)
          if (k0 + j < nsrc) x[j] = ld16(sh.src[k0 + j] + off);
#pragma unroll
        for (int j = 0; j < KB; ++j) {
          if (k0 + j >= nsrc) break;
          if (k0 + j == 0) a = O::widen(x[0]);
          else O::add(a, x[j]);
        }
      }
      r = O::narrow(a);  // one rounding per task
    }
    for (int d0 = 0; d0 < ndst; d0 += DB) {
      uint4 q[DB];
#pragma unroll
      for (int j = 0; j < DB; ++j)
        if (d0 + j < ndst && sh.acc[d0 + j]) q[j] = ld16(sh.dst[d0 + j] + off);
#pragma unroll
      for (int j = 0; j < DB; ++j) {
        if (d0 + j >= ndst) break;
        char* p = sh.dst[d0 + j] + off;
        if (sh.acc[d0 + j]) {
          typename O::Acc b = O::widen(q[j]);
          O::add(b, r);
          st16(p, O::narrow(b));
        } else {
          st16(p, r);
        }
      }
    }
  }
}

// NVLS (NEXT-2 switch reduction): every 16-byte vector of the multicast
// source is summed over all ranks' copies by the NVSwitch (multimem
// ld_reduce; fp32 adds in the switch's order, bf16 accumulated in fp32 and
// rounded once, int32 wrapping) and the sum is stored to every rank's copy of
// the multicast destination (multimem.st).
template <int DT>
__device__ __forceinline__ uint4 mm_ld_reduce(const char* p) {
  uint4 v;
  if constexpr (DT == kF32)
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  else if constexpr (DT == kBF16)
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.acc::f32.v4.bf16x2 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  else {
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.u32 %0, [%1];" : "=r"(v.x) : "l"(p) : "memory");
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.u32 %0, [%1];" : "=r"(v.y) : "l"(p + 4) : "memory");
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.u32 %0, [%1];" : "=r"(v.z) : "l"(p + 8) : "memory");
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.u32 %0, [%1];" : "=r"(v.w) : "l"(p + 12) : "memory");
  }
  return v;
}
__device__ __forceinline__ void mm_st(char* p, uint4 v) {
  asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w) : "memory");
}
template <int DT, class SH>
__device__ void nvls_vec(const SH& sh, uint32_t nvec) {
  for (uint32_t v = threadIdx.x; v < nvec; v += kThreads)
    mm_st(sh.dst[0] + (size_t)v * 16, mm_ld_reduce<DT>(sh.src[0] + (size_t)v * 16));
}
// Loopback emulation of the switch (adapcc_nvls_setup on one device): the
// multicast address is virtual rank 0's copy; every rank's copy sits at the
// same offset from its own unicast base (uc[q]); the sum runs over the n
// copies in ascending rank order (fp32 adds, bf16 accumulated in fp32 and
// rounded once, int32 wrapping) and is stored to every copy.
template <int DT, class SH>
__device__ void nvls_vec_emul(const SH& sh, uint32_t nvec, char* const* uc, const char* mc, int n) {
  using O = Ops<DT>;
  const size_t so = (size_t)(sh.src[0] - mc), dof = (size_t)(sh.dst[0] - mc);
  for (uint32_t v = threadIdx.x; v < nvec; v += kThreads) {
    const size_t o = (size_t)v * 16;
    typename O::Acc a = O::widen(ld16(uc[0] + so + o));
    for (int q = 1; q < n; ++q) O::add(a, ld16(uc[q] + so + o));
    const uint4 r = O::narrow(a);
    for (int q = 0; q < n; ++q) st16(uc[q] + dof + o, r);
  }
}
__device__ __forceinline__ void fence_proxy_alias() { asm volatile("fence.proxy.alias;" ::: "memory"); }

// element path (misaligned slots / ragged tail): e in [e_begin, e_end)
template <int DT>
__device__ __forceinline__ void fold_scalar(const Shared& sh, int nsrc, int ndst, uint64_t e_begin,
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
__device__ void fold_chunk(const Shared& sh, int nsrc, int ndst, uint64_t n, int op,
                           char* const* nvls_uc = nullptr, const char* nvls_mc = nullptr, int nranks = 0) {
  using O = Ops<DT>;
  using E = typename O::E;
  if (op == kOpNone) return;  // (STAGED late join: nothing to move for this chunk)
  if (op == kOpNvls) {        // (planned on whole 16-byte vectors only)
    if (nvls_uc) nvls_vec_emul<DT>(sh, (uint32_t)(n * O::kEsize / 16), nvls_uc, nvls_mc, nranks);
    else nvls_vec<DT>(sh, (uint32_t)(n * O::kEsize / 16));
    return;
  }
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
  const uint32_t nvec = (uint32_t)(n / VE);
  // bf16 accumulators are 8 floats per vector: fewer vectors per source
  // keep the kernel within 128 registers (2 CTAs/SM) without spills
  if (sh.any_acc) fold_acc_vec<DT, 4, 8>(sh, nsrc, ndst, nvec);
  else if (nsrc == 1) copy_vec<DT, ADAPCC_COPY_UNROLL>(sh, ndst, nvec);
  else if (nsrc <= 4) fold_vec<DT, (DT == kBF16 ? 1 : 2), 4>(sh, nsrc, ndst, nvec);
  else fold_vec<DT, 1, 8>(sh, nsrc, ndst, nvec);
  if ((uint64_t)nvec * VE < n) fold_scalar<DT>(sh, nsrc, ndst, (uint64_t)nvec * VE, n);
}

template <int DT, int NR>
__global__ void __launch_bounds__(kThreads, ADAPCC_MINB) engine_kernel(const __grid_constant__ LaunchParamsT<NR> P) {
  __shared__ Shared sh;
  // P.send / P.recv / P.hdr / NVLS scratch (unicast, multicast), indexed by BufKind
  __shared__ char* sbase[kNumBufKinds][NR];
  const bool sys = P.ipc;
  const uint64_t t_entry = P.trace ? globaltimer() : 0;
  Item pre{};  // thread 0: this CTA's first item, loaded together with the epoch
  // first item, its task and refs in one round trip (plan-time blob)
  const bool use_blob = blockIdx.x < P.nfirst;
  if (use_blob && threadIdx.x < P.first_words)
    sh.blob[0][threadIdx.x] = P.first[(size_t)blockIdx.x * P.first_words + threadIdx.x];
  const bool stat = P.sched_static != 0;
  int buf = 0;  // blob buffer of the current item (static schedule)
  // buffer bases into shared memory (indexed by BufKind): read once per CTA,
  // before the stream-order wait
  for (int i = threadIdx.x; i < kNumBufKinds * P.nranks; i += kThreads) {
    const int k = i / P.nranks, q = i - k * P.nranks;
    sbase[k][q] = k == 0 ? P.send[q] : k == 1 ? P.recv[q] : k == 2 ? P.hdr[q]
                : k == 3 ? P.nvls_uc + (uint64_t)q * P.nvls_stride : P.nvls_mc;
  }
  if (threadIdx.x == 0 && !use_blob && blockIdx.x < P.nitems) pre = P.items[blockIdx.x];
  constexpr int esize = Ops<DT>::kEsize;

  // thread 0: stage item `it`'s header in shared memory, so that no task field
  // stays live in registers across the fold (fb: from blob buffer b)
  auto stage = [&](uint32_t it, bool fb, int b, bool is_first) {
    sh.item = it;
    if (P.trace) sh.tr0 = globaltimer();
    sh.bad_align = 0;
    sh.any_acc = 0;
    sh.nvls_alias = 0;
    if (it >= P.nitems) return;
    const Item item = fb ? *reinterpret_cast<const Item*>(&sh.blob[b][0]) : is_first ? pre : P.items[it];
    const Task& t = fb ? *reinterpret_cast<const Task*>(&sh.blob[b][1]) : P.tasks[item.task];
    Cur& c = sh.cur;
    c.blob = fb ? (int8_t)b : (int8_t)-1;
    c.tnsrc = t.nsrc;
    c.nreg = t.nsrc;
    c.ndst = t.ndst;
    c.nwait = t.nwait;
    c.npost = t.npost;
    c.op = t.op;
    c.dropped = (int)t.owner == P.drop_rank;
    c.late = 0;
    c.force_acc = false;
    c.lkind = t.lkind;
    c.decide = 0;
    c.dec_dst = 0;
    c.dec_out = 1;
    c.tnwait = t.nwait;
    c.wait0 = 0;
    c.tnlate = t.nlate;
    c.tlo = t.lo;
    c.tnch = t.nchunks;
    if (P.late_mode && !c.dropped && t.lkind == kLatePush) {
      // the late rank's own chunk goes to the root iff it is ready now
      // (phase 1) / iff it did not go in phase 1 (phase 2)
      bool pushed;
      if (P.late_mode == 1) {
        pushed = ld_acquire(reinterpret_cast<const uint64_t*>(sbase[kBufArena][t.owner] + ArenaHeader::kReady),
                            P.ipc) >= P.late_ticket;
        P.late_bits[it] = pushed ? 1 : 0;
      } else {
        pushed = P.late_bits[it] == 0;
      }
      if (!pushed) c.op = kOpNone;
      c.dec_dst = 1;
      c.dec_out = pushed ? 1 : 0;
    } else if (P.late_mode && !c.dropped && t.lkind == kLateRoot) {
      c.decide = 1;  // candidates are decided after the waits (their decision words)
      if (P.late_mode == 2) {  // only the late slots' flags; recv += fold of what is left
        c.nreg = 0;
        c.wait0 = (uint16_t)(t.nwait - t.nlwait);
        c.nwait = t.nlwait;
        c.op = kOpFold;
        c.force_acc = true;
      }
    } else if (P.late_mode && !c.dropped && t.lkind == kLatePull) {
      c.decide = P.late_mode == 2;  // accumulate iff the parent broadcast anything
    } else if (P.late_mode && !c.dropped) {
      if (t.nlate == 0) {
        c.dropped = P.late_mode == 2;  // phase 2 only runs the roots' folds
      } else {
        const uint64_t m = late_select(P, t, it, sh.epoch);
        c.late = m;
        if (P.late_mode == 2) {  // recv += sum of the late ranks not yet included
          c.nreg = 0;
          c.nwait = 0;
          c.op = kOpFold;
          c.force_acc = true;
          c.dropped = m == 0;
        } else if (m && t.op == kOpZero) {
          c.op = kOpFold;
        }
      }
    }
    c.nsrc = (uint16_t)(c.nreg + __popcll(c.late));
    c.ref0 = t.ref0;
    c.flag0 = t.flag0;
    c.chunk = item.chunk;
    c.len = item.len;
    c.e0 = t.lo + (uint64_t)item.chunk * t.chunk_elems + item.off;
  };
  // threads < nsrc + ndst: resolve the staged item's stream pointers.  Arena
  // streams get `hoff` (the parity half); returns whether this thread's
  // stream is an arena stream.
  auto resolve = [&](uint64_t hoff) -> bool {
    const int nsrc = sh.cur.nsrc, ndst = sh.cur.ndst;
    if (threadIdx.x >= nsrc + ndst) return false;
    const int i = threadIdx.x;
    // index of this stream's ref, relative to the task's first ref
    const uint32_t j = i < sh.cur.nreg ? i
                     : i < nsrc ? sh.cur.tnsrc + ndst + nth_bit(sh.cur.late, i - sh.cur.nreg)
                                : sh.cur.tnsrc + (i - nsrc);
    const BufRef r = sh.cur.blob >= 0 ? *reinterpret_cast<const BufRef*>(&sh.blob[sh.cur.blob][kBlobRef0 + j])
                                      : P.refs[sh.cur.ref0 + j];
    const bool arena = r.kind == kBufArena;
    char* p = sbase[r.kind][r.rank] + (arena ? hoff : 0) + r.bias + (int64_t)(sh.cur.e0 * esize);
    if (reinterpret_cast<uintptr_t>(p) & 15) atomicOr(&sh.bad_align, 1);  // (hoff is 256-byte aligned)
    if (r.kind >= kBufNvlsUc) atomicOr(&sh.nvls_alias, 1);
    if (i < nsrc) {
      sh.src[i] = p;
    } else {
      sh.dst[i - nsrc] = p;
      // (force_acc: recv += result; a STAGED broadcast slot still takes the plain result)
      const bool acc = r.accum || (sh.cur.force_acc && r.kind == kBufRecv);
      sh.acc[i - nsrc] = acc;
      if (acc) atomicOr(&sh.any_acc, 1);
    }
    return arena;
  };
  // STAGED late join: decision word of chunk sh.cur.chunk of the slot `r`
  // (an arena stream of the current task) -- 8 bytes per chunk before the slot
  auto dec_word = [&](const BufRef& r, uint64_t hoff) {
    return reinterpret_cast<uint64_t*>(sbase[kBufArena][r.rank] + hoff + r.bias + (int64_t)(sh.cur.tlo * esize) -
                                       (int64_t)late_dec_bytes(sh.cur.tnch)) + sh.cur.chunk;
  };
  auto ref_of = [&](uint32_t j) {
    return sh.cur.blob >= 0 ? *reinterpret_cast<const BufRef*>(&sh.blob[sh.cur.blob][kBlobRef0 + j])
                            : P.refs[sh.cur.ref0 + j];
  };
  // thread 0, after the item's waits: which late candidates the root folds
  // (phase 1: the pushed slots and, for a late root, its own input if ready;
  // phase 2: the slots pushed now and a late root's own input if not yet
  // folded), or whether a phase-2 broadcast pull has anything to add
  auto decide = [&](uint64_t hoff) {
    Cur& c = sh.cur;
    if (c.lkind == kLateRoot) {
      const uint64_t prev = P.late_mode == 2 ? P.late_bits[sh.item] : 0;
      uint64_t m = 0;
      for (uint32_t j = 0; j < c.tnlate; ++j) {
        const BufRef r = ref_of(c.tnsrc + c.ndst + j);
        bool in;
        if (r.kind == kBufArena) in = *reinterpret_cast<volatile uint64_t*>(dec_word(r, hoff)) != 0;
        else if (P.late_mode == 1)
          in = ld_acquire(reinterpret_cast<const uint64_t*>(sbase[kBufArena][r.rank] + ArenaHeader::kReady),
                          P.ipc) >= P.late_ticket;
        else in = ((prev >> j) & 1) == 0;
        if (in) m |= 1ull << j;
      }
      if (P.late_mode == 1) {
        P.late_bits[sh.item] = m;
        if (m && c.op == kOpZero) c.op = kOpFold;
      } else {
        if (!m) c.op = kOpNone;
        c.dec_dst = 1;
        c.dec_out = m ? 1 : 0;
      }
      c.late = m;
      c.nsrc = (uint16_t)(c.nreg + __popcll(m));
    } else {  // kLatePull, phase 2
      const bool any = *reinterpret_cast<volatile uint64_t*>(dec_word(ref_of(0), hoff)) != 0;
      if (!any) c.op = kOpNone;
      else c.force_acc = true;
      c.dec_dst = 1;
      c.dec_out = any ? 1 : 0;
    }
  };
  // The first item of a blob CTA is staged and resolved here, before the
  // stream-order wait: under PDL this overlaps the previous kernel instead of
  // sitting between the epoch read and the first load (~0.8 us, in-kernel
  // trace).  Arena pointers get the parity half once the epoch is known.
  // Late join decides per item from ready words, so it stages after the wait.
  const bool prestage = use_blob && P.late_mode == 0;
  bool my_arena = false;
  if (threadIdx.x == 0) {
    sh.abort = 0;
    sh.nclaim = P.nitems;  // (phase 2 of a late join: its list length, set after the wait)
  }
  if (prestage) {
    __syncthreads();  // blob words and buffer bases
    if (threadIdx.x == 0) {
      sh.claim = blockIdx.x;
      stage(blockIdx.x, true, 0, true);
    }
    __syncthreads();
    if (sh.item < P.nitems && !sh.cur.dropped) my_arena = resolve(0);
  }
  // the plan tables above are immutable; the epoch, counters, arenas and user
  // buffers below belong to the stream order (PDL: the previous launch)
  pdl_trigger();
  pdl_wait();
  // Lazy epoch: a loopback plan without arena streams or flags whose CTAs
  // need no claim counter only uses the epoch to count itself done at the
  // end, so its load stays in flight during the fold instead of costing a
  // round trip and a barrier up front.
  const bool lazy = !P.ipc && P.arena_free && prestage && (stat || P.nitems <= gridDim.x);
  uint64_t e_lazy = 0;
  if (lazy) {
    if (threadIdx.x == 0) e_lazy = *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) + 1;
  } else {
    if (threadIdx.x == 0) {
      // late join (never lazy): phase 2 claims positions in phase 1's list
      if (P.late_mode == 2 && P.late_list && !stat) sh.nclaim = late_listed(P);
      // this launch's epoch = the one the previous launch published + 1
      const uint64_t e = *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) + 1;
      sh.epoch = e;
      if (blockIdx.x == 0) {  // re-arm the other parity's counters for the next launch
        P.state->work[(e + 1) & 1] = 0;
        P.state->done[(e + 1) & 1] = 0;
      }
    }
    __syncthreads();
  }
  const uint64_t t_ready = P.trace ? globaltimer() : 0;
  const uint64_t epoch = lazy ? 0 : sh.epoch;  // (lazy: unused before the end)
  const unsigned par = (unsigned)(epoch & 1);
  const uint64_t half_off = kArenaHeader + par * P.half_bytes;
  // multi-process: every peer must have finished the call that last used this
  // parity half of the arenas (epoch - 2) before we write into any arena
  if (P.ipc && epoch > 2) {
    const int r = threadIdx.x;
    if (r < P.nranks && r != P.my_rank && ((P.members >> r) & 1)) {
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[r]), epoch - 2, P)) sh.abort = 1;
    }
    __syncthreads();
  }
  if (P.ipc && P.check_sig && !check_call_sig(P, epoch)) sh.abort = 1;  // before any byte moves
  if (P.ipc && P.zc) {  // zero-copy: peers read/write our user buffers directly
    if (blockIdx.x == 0 && threadIdx.x == 0)
      st_release(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank] + ArenaHeader::kEntered), epoch, true);  // entered
    if (threadIdx.x < P.nranks && threadIdx.x != P.my_rank && ((P.members >> threadIdx.x) & 1))
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[threadIdx.x] + ArenaHeader::kEntered), epoch, P)) sh.abort = 1;
    __syncthreads();
  }
  // Item claiming: CTA b starts with item b (no atomic), later items come from
  // the counter offset by the grid.  A CTA whose item is among the last
  // gridDim.x stops after it: every CTA makes exactly one such claim, so those
  // items are all taken and no CTA pays a final failed atomic (small calls run
  // with no claim atomics at all).
  bool first = true, last = false, staged = prestage;
  // Phase 2 of a late join claims positions in phase 1's list of incomplete
  // items (no waits in phase 2, so any order is deadlock-free)
  const bool listed = P.late_mode == 2 && P.late_list != nullptr && !stat;
  while (!sh.abort && !last) {
    if (!staged) {
      if (threadIdx.x == 0) {
        const uint32_t k = first ? blockIdx.x : stat ? sh.item + gridDim.x
                                                     : gridDim.x + atomicAdd(&P.state->work[par], 1u);
        sh.claim = k;
        uint32_t it = k;
        if (listed) it = k < sh.nclaim ? P.late_list[k] : P.nitems;
        // (a listed phase-2 item is not the CTA's first item: no blob, no preloaded item)
        const bool fb = stat || (first && use_blob && !listed);
        stage(it, fb, buf, first && !listed);
      }
      __syncthreads();
    }
    if (sh.item >= P.nitems) break;
    first = false;
    last = (uint64_t)sh.claim + gridDim.x >= (listed ? sh.nclaim : P.nitems);
    // static schedule: fetch the next item's blob into the other buffer while
    // this item folds (its last readers finished before the barrier above)
    if (stat && !last && threadIdx.x < P.first_words)
      cp_async16(&sh.blob[buf ^ 1][threadIdx.x],
                 P.first + (size_t)(sh.item + gridDim.x) * P.first_words + threadIdx.x);
    const bool dropped = sh.cur.dropped, deferred = sh.cur.decide != 0;
    if (!dropped) {
      // input flags, one waiter thread per flag
      if (threadIdx.x < sh.cur.nwait) {
        const FlagRef f = P.flags[sh.cur.flag0 + sh.cur.wait0 + threadIdx.x];
        const uint64_t* fl =
            reinterpret_cast<const uint64_t*>(sbase[kBufArena][f.rank] + half_off + f.off) + sh.cur.chunk;
        if (!wait_flag(fl, epoch, P)) sh.abort = 1;
      }
      if (!staged) {
        if (!deferred) resolve(half_off);
      } else if (my_arena) {  // pre-staged before the epoch was known
        const int i = threadIdx.x, nsrc = sh.cur.nsrc;
        if (i < nsrc) sh.src[i] += half_off;
        else sh.dst[i - nsrc] += half_off;
      }
    }
    staged = false;
    __syncthreads();
    if (P.trace && threadIdx.x == 0) sh.tr1 = globaltimer();
    if (sh.abort) {
      if (stat) cp_async_wait_all();
      break;
    }
    if (!dropped && deferred) {  // STAGED late join: decision words are readable now
      if (threadIdx.x == 0) decide(half_off);
      __syncthreads();
      resolve(half_off);
      __syncthreads();
    }
    const int nsrc = sh.cur.nsrc, ndst = sh.cur.ndst, npost = sh.cur.npost;
    const bool alias = sh.nvls_alias != 0;
    if (!dropped) {
      // NVLS scratch is written through one address alias (unicast or
      // multicast) and read through the other: proxy fences on both sides
      if (alias) fence_proxy_alias();
      fold_chunk<DT>(sh, nsrc, ndst, sh.cur.len, sh.cur.op, P.nvls_stride ? sbase[kBufNvlsUc] : nullptr,
                     sbase[kBufNvlsMc][0], P.nranks);
      if (alias) fence_proxy_alias();
      if (stat) cp_async_wait_all();  // the next blob has landed before the barrier publishes it
      __syncthreads();
      // npost was read before the barrier: after it, only thread 0 touches
      // sh.cur (it rewrites it for the next item)
      if (threadIdx.x == 0 && npost) {
        const uint64_t e = sh.epoch;
        const char* const* hdr = P.hdr;
        if (sh.cur.dec_dst)  // STAGED late join: the decision travels with the chunk's flag
          for (int k = 0; k < ndst; ++k) {
            const BufRef r = ref_of(sh.cur.tnsrc + k);
            if (r.kind == kBufArena) *reinterpret_cast<volatile uint64_t*>(dec_word(r, half_off)) = sh.cur.dec_out;
          }
        fence(sys);  // the chunk's bytes (incl. remote NVLink stores) before its flag
        for (int i = 0; i < sh.cur.npost; ++i) {
          const FlagRef f = P.flags[sh.cur.flag0 + sh.cur.tnwait + i];
          st_release(reinterpret_cast<uint64_t*>(const_cast<char*>(hdr[f.rank]) + half_off + f.off) +
                         sh.cur.chunk, e, sys);
        }
      }
      if (P.trace && threadIdx.x == 0)
        trace_put(P, sh.item, 0, sh.tr0, sh.tr1, globaltimer(),
                  (uint64_t)sh.cur.len * esize * (uint64_t)(sh.cur.nsrc + sh.cur.ndst));
    } else if (stat) {
      cp_async_wait_all();
      __syncthreads();
    }
    buf ^= stat ? 1 : 0;
  }
  __syncthreads();
  if (P.trace && threadIdx.x == 0) trace_put(P, kTraceCta, 0, t_entry, t_ready, globaltimer(), 0);
  if (threadIdx.x == 0) {
    // across processes the done word published to peers must follow every
    // CTA's data; in loopback only the next launch reads anything, after
    // this one completes, so counting needs no fence
    if (sys) fence(sys);
    const uint64_t ep = lazy ? e_lazy : epoch;
    if (lazy && blockIdx.x == 0) {  // re-arm the other parity's counters for the next launch
      P.state->work[(ep + 1) & 1] = 0;
      P.state->done[(ep + 1) & 1] = 0;
    }
    const unsigned done = atomicAdd(&P.state->done[ep & 1], 1u);
    if (done == gridDim.x - 1) {
      // last CTA: publish the epoch for the next launch on this stream and,
      // across processes, "this rank finished epoch" to the peers
      // late join: phase 1 validates its list for phase 2; phase 2 consumed it
      // (every CTA is past its claims), so a repeated phase 2 adds nothing
      if (P.late_mode && P.late_count) P.late_count[1] = P.late_mode == 1 ? ep : ~0ull;
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

}  // namespace

int engine_threads() { return kThreads; }

cudaError_t engine_occupancy(int dtype, int* blocks_per_sm) {
  switch (dtype) {
    case kF32: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kF32, kMaxRanksDev>, kThreads, 0);
    case kBF16: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kBF16, kMaxRanksDev>, kThreads, 0);
    default: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_kernel<kI32, kMaxRanksDev>, kThreads, 0);
  }
}

namespace {
__global__ void signal_kernel(uint64_t* word, uint64_t value, int sys, uint64_t* board) {
  fence(sys);
  st_release(word, value, sys);
  if (board) st_release(board, value, true);  // host-visible readiness board (coordinator)
}
__global__ void spin_kernel(uint64_t ns) {
  const uint64_t t0 = globaltimer();
  while (globaltimer() - t0 < ns) {
  }
}
}  // namespace

cudaError_t engine_signal(uint64_t* word, uint64_t value, bool sys, uint64_t* board, cudaStream_t stream) {
  cudaGetLastError();
  signal_kernel<<<1, 1, 0, stream>>>(word, value, sys ? 1 : 0, board);
  return cudaGetLastError();
}

cudaError_t engine_spin(uint64_t ns, cudaStream_t stream) {
  cudaGetLastError();
  spin_kernel<<<1, 1, 0, stream>>>(ns);
  return cudaGetLastError();
}

namespace {
template <int NR>
cudaError_t launch_nr(const LaunchParamsT<NR>& p, int grid, cudaStream_t stream, bool pdl) {
  switch (p.dtype) {
    case kF32: return launch_kernel(engine_kernel<kF32, NR>, grid, kThreads, 0, stream, pdl, p);
    case kBF16: return launch_kernel(engine_kernel<kBF16, NR>, grid, kThreads, 0, stream, pdl, p);
    default: return launch_kernel(engine_kernel<kI32, NR>, grid, kThreads, 0, stream, pdl, p);
  }
}
}  // namespace

cudaError_t engine_launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl) {
  cudaGetLastError();  // clear any stale error so the check below is about this launch
  if (p.nranks <= kNarrowRanks) return launch_nr(narrow(p), grid, stream, pdl);
  return launch_nr(p, grid, stream, pdl);
}

}  // namespace adapcc
