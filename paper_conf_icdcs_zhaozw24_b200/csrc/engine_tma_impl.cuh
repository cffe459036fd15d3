// AdapCC transfer engine, TMA variant: warp-specialised persistent kernel in
// which one producer warp moves every source tile with TMA bulk copies
// (cp.async.bulk global -> shared, completion on an mbarrier) through a
// 3-stage shared-memory ring, and 8 consumer warps fold the K tiles of a
// stage from shared memory and store the result to the D destinations.
//
// Same work items, flags, epochs and deadlock-freedom argument as engine.cu
// (DESIGN.md §6); what changes is the data path:
//   - bytes in flight no longer cost registers: 2 CTAs x 3 stages x 32 KiB =
//     192 KiB per SM, issued by ONE thread per CTA (the TMA engine does the
//     addressing), also for peer (NVLink) sources;
//   - the producer claims and waits for the next item while the consumers are
//     still folding the current one (an item queue in shared memory), so the
//     per-item claim / flag latency is hidden.
// Paper mapping: the producer is the "receive" side of the chunk pipeline
// (wait for the chunk, then aggregate), consumers are the
// aggregation kernel + send.
// Compiled twice (engine_tma_direct.cu, engine_tma_staged.cu) with different
// pipeline shapes: ADAPCC_TMA_NS names the instantiation's namespace.
#include "engine_common.cuh"

#ifndef ADAPCC_TMA_NS
#error "include through engine_tma_direct.cu / engine_tma_staged.cu"
#endif

namespace adapcc {
namespace ADAPCC_TMA_NS {
namespace {

using namespace dev;

constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kTmaThreads = kConsumers + 32;  // + 1 producer warp
#ifndef ADAPCC_TMA_STAGES
#define ADAPCC_TMA_STAGES 3      // shared-memory ring depth
#endif
#ifndef ADAPCC_TMA_STAGE_KB
#define ADAPCC_TMA_STAGE_KB 32   // bytes per stage (all K source tiles of one step)
#endif
#ifndef ADAPCC_TMA_MINB
#define ADAPCC_TMA_MINB 2        // resident CTAs per SM
#endif
constexpr int kStages = ADAPCC_TMA_STAGES;
constexpr uint32_t kStageBytes = ADAPCC_TMA_STAGE_KB * 1024;
// Tiles larger than one consumer round (K = 1 with accumulation: > 32 KiB;
// K = 2, 3: > 16 KiB) exist only with stages above 32 KiB.
constexpr bool kLargeTiles = kStageBytes > 32 * 1024;
constexpr int kMaxKS = (kStageBytes / 4096) < 8 ? (int)(kStageBytes / 4096) : 8;  // sources per stage
constexpr int kQ = 2;           // item queue depth
#ifndef ADAPCC_FOLD_TMA
#define ADAPCC_FOLD_TMA 1        // K >= 2 folds stored by TMA bulk stores from shared memory
#endif
constexpr bool kFoldTma = ADAPCC_FOLD_TMA != 0;
constexpr int kMaxPost = 4;
// ACCUMULATE (phase 2, recv += result) with every tile in shared memory: the
// producer also loads each accumulating destination's tile, so a stage holds
// nsrc + nacc tiles of at least 512 B (acc_tma in the item descriptor)
constexpr int kMaxAccTiles = 24;
// tuning overrides (ADAPCC_TMA_STAGE_KB / _STAGES) must leave at least one
// 4 KiB source tile and one 512-byte ACCUMULATE tile per stage
static_assert(kStageBytes % 4096 == 0 && kStageBytes >= kMaxAccTiles * 512, "TMA stage too small");
static_assert(kMaxKS >= 1 && kStages >= 2, "TMA pipeline shape");

struct ItemDesc {
  const char* src[kMaxFold];
  char* dst[kMaxDst];
  uint64_t* post[kMaxPost];
  uint64_t len;         // elements
  uint32_t vec_bytes;   // bytes moved by tiles (multiple of 16)
  uint32_t tile;        // bytes per source per stage
  uint32_t ntiles;
  uint16_t nsrc, ndst, op, npost, passes, ks;
  uint8_t acc[kMaxDst];
  uint8_t stop, dropped, scalar_only, any_acc;
  uint8_t acc_tma;            // accumulating destinations are loaded by TMA and stored from the stage
  uint8_t acc_red;            // accumulating destinations take bulk reduce-adds of the folded tile
  uint8_t need_decide;        // STAGED late join: sources / op are fixed after the waits (decision words)
  uint8_t ndec, dec_val;      // STAGED late join: decision words to write before the posts, and their value
  uint16_t wait0;             // first of the task's waits this item waits for
  uint64_t* dec[2];
  uint8_t acc_slot[kMaxDst];  // acc_tma: stage tile of destination k's recv (0 = plain destination)
  uint32_t item;        // trace: item index, claim and inputs-ready times
  uint64_t tr0, tr1;
};

struct Smem {
  uint64_t full[kStages];
  uint64_t empty[kStages];
  uint64_t qfull[kQ];
  uint64_t qempty[kQ];
  uint64_t epoch;
  int abort;
  int pad;
  ItemDesc q[kQ];
  uint4 blob[kFirstMaxWords];  // this CTA's first item: Item | Task | refs (plan-time blob)
};

constexpr size_t kSmemHeader = (sizeof(Smem) + 127) / 128 * 128;
constexpr size_t kSmemBytes = kSmemHeader + (size_t)kStages * kStageBytes;

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t su32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ bool mbar_try(uint64_t* b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(su32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  while (!mbar_try(b, parity)) {
  }
}
// TMA bulk copy global -> shared, completes `bytes` on the mbarrier
__device__ __forceinline__ void tma_load(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          su32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(su32(bar))
      : "memory");
}
// TMA bulk copy shared -> global (bulk-group completion)
__device__ __forceinline__ void tma_store(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(su32(ssrc)),
               "r"(bytes)
               : "memory");
}
// TMA bulk reduction shared -> global: dst[i] = dst[i] + src[i], performed
// by the memory system (L2) as one read-modify-write per element -- recv +=
// result without bringing recv into the SM (SASS UBLKRED ... .RN).  fp32 adds
// round to nearest even, bf16 (.noftz) rounds the exact sum once to bf16
// (reading Q6), int32 wraps (.u32 add = the same bits as .s32).
template <int DT>
__device__ __forceinline__ void tma_red_add(void* gdst, const void* ssrc, uint32_t bytes) {
  if constexpr (DT == kF32)
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(gdst),
                 "r"(su32(ssrc)), "r"(bytes) : "memory");
  else if constexpr (DT == kBF16)
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.noftz.bf16 [%0], [%1], %2;" ::"l"(gdst),
                 "r"(su32(ssrc)), "r"(bytes) : "memory");
  else
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.u32 [%0], [%1], %2;" ::"l"(gdst),
                 "r"(su32(ssrc)), "r"(bytes) : "memory");
}
// one destination tile leaves the stage: plain bulk store, or bulk reduce-add
// into an accumulating destination (acc_red)
template <int DT>
__device__ __forceinline__ void tma_put(void* gdst, const void* ssrc, uint32_t bytes, bool acc) {
  if (acc) tma_red_add<DT>(gdst, ssrc, bytes);
  else tma_store(gdst, ssrc, bytes);
}
__device__ __forceinline__ void tma_store_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void tma_store_wait_read() {  // all but N groups have read their smem
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void tma_store_wait_all() {  // all bulk stores complete (writes performed)
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_cnt(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ void consumer_sync() {
  asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory");
}
__device__ __forceinline__ uint4 lds16(const char* p) { return *reinterpret_cast<const uint4*>(p); }
__device__ __forceinline__ void sts16(char* p, uint4 v) { *reinterpret_cast<uint4*>(p) = v; }
__device__ __forceinline__ void fence_proxy_async_smem() {  // generic-proxy smem writes -> async proxy (TMA)
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ------------------------------------------------------------ consumers
template <int DT>
__device__ __forceinline__ void store_result(const ItemDesc& d, size_t off, uint4 r) {
  using O = Ops<DT>;
  for (int k = 0; k < d.ndst; ++k) {
    char* p = d.dst[k] + off;
    if (d.acc[k]) {  // recv += result (phase 2)
      typename O::Acc q = O::widen(ld16(p));
      O::add(q, r);
      st16(p, O::narrow(q));
    } else {
      st16(p, r);
    }
  }
}

// element path for misaligned streams and the sub-16-byte tail
template <int DT>
__device__ void scalar_range(const ItemDesc& d, uint64_t e_begin, uint64_t e_end, int tid) {
  using O = Ops<DT>;
  using E = typename O::E;
  for (uint64_t e = e_begin + tid; e < e_end; e += kConsumers) {
    E x0 = *reinterpret_cast<const volatile E*>(d.src[0] + e * sizeof(E));
    E r;
    if (d.nsrc == 1) {
      r = x0;
    } else {
      auto a = O::w1(x0);
      for (int k = 1; k < d.nsrc; ++k)
        a = O::a1(a, *reinterpret_cast<const volatile E*>(d.src[k] + e * sizeof(E)));
      r = O::n1(a);
    }
    for (int k = 0; k < d.ndst; ++k) {
      E* p = reinterpret_cast<E*>(d.dst[k] + e * sizeof(E));
      if (d.acc[k]) *p = O::n1(O::a1(O::w1(*reinterpret_cast<volatile E*>(p)), r));
      else *p = r;
    }
  }
}

// Large-tile rounds (tile > one round of the caller's VPT), kept out of line
// so that the common one-round path keeps its register budget.
template <int DT>
__device__ __noinline__ void copy_rounds(const char* sb, const ItemDesc& d, int tid, uint32_t t, uint32_t nv) {
  for (uint32_t v = tid; v < nv; v += kConsumers)
    store_result<DT>(d, (size_t)t * d.tile + (size_t)v * 16, lds16(sb + (size_t)v * 16));
}
template <int DT>
__device__ __noinline__ void fold_rounds(const char* sb, const ItemDesc& d, int tid, uint32_t t, uint32_t nv) {
  using O = Ops<DT>;
  for (uint32_t v = tid; v < nv; v += kConsumers) {
    const char* pv = sb + (size_t)v * 16;
    typename O::Acc a = O::widen(lds16(pv));
    for (int k = 1; k < (int)d.nsrc; ++k) O::add(a, lds16(pv + (size_t)k * d.tile));
    store_result<DT>(d, (size_t)t * d.tile + (size_t)v * 16, O::narrow(a));  // one rounding
  }
}

// Copy the tiles of a one-source item (bytes unchanged) into destinations
// that need the generic proxy (accumulation): VPT vectors per thread per
// round; a tile larger than one round (VPT x 16 B x consumers) is walked in
// rounds while the stage is held.
template <int DT, int VPT>
__device__ __forceinline__ void consume_copy(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                             uint32_t& stage, uint32_t& sphase) {
  const bool warp_lane0 = (tid & 31) == 0;
  constexpr uint32_t kRound = VPT * kConsumers;
  for (uint32_t t = 0; t < d.ntiles; ++t) {
    const uint32_t nv = min(d.tile, d.vec_bytes - t * d.tile) / 16;
    mbar_wait(&sm.full[stage], sphase);
    const char* sb = stages + (size_t)stage * kStageBytes;
    if (!kLargeTiles || nv <= kRound) {  // one round: registers hold the tile, release the stage before storing
      uint4 raw[VPT];
#pragma unroll
      for (int j = 0; j < VPT; ++j) {
        const uint32_t v = tid + j * kConsumers;
        if (v < nv) raw[j] = lds16(sb + (size_t)v * 16);
      }
      __syncwarp();
      if (warp_lane0) mbar_arrive(&sm.empty[stage]);
#pragma unroll
      for (int j = 0; j < VPT; ++j) {
        const uint32_t v = tid + j * kConsumers;
        if (v < nv) store_result<DT>(d, (size_t)t * d.tile + (size_t)v * 16, raw[j]);
      }
    } else {
      copy_rounds<DT>(sb, d, tid, t, nv);
      __syncwarp();
      if (warp_lane0) mbar_arrive(&sm.empty[stage]);
    }
    if (++stage == kStages) { stage = 0; sphase ^= 1; }
  }
}

// Pure copy (one source, no accumulation) entirely on the TMA engines: one
// thread waits for each loaded stage and issues the D bulk stores straight
// from shared memory; a stage is released once its stores have read it.
// Other consumer threads only advance their ring position.
template <int DT>
__device__ __forceinline__ void copy_tma(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                         uint32_t& stage, uint32_t& sphase) {
  if (tid == 0) {
    int prev = -1;
    for (uint32_t t = 0; t < d.ntiles; ++t) {
      const uint32_t tb = min(d.tile, d.vec_bytes - t * d.tile);
      mbar_wait(&sm.full[stage], sphase);
      const char* sb = stages + (size_t)stage * kStageBytes;
      for (int k = 0; k < d.ndst; ++k) tma_put<DT>(d.dst[k] + (size_t)t * d.tile, sb, tb, d.acc[k]);
      tma_store_commit();
      if (prev >= 0) {
        tma_store_wait_read<1>();
        mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
      }
      prev = (int)stage;
      if (++stage == kStages) { stage = 0; sphase ^= 1; }
    }
    if (prev >= 0) {
      tma_store_wait_read<0>();
      mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
    }
  } else {
    const uint32_t total = stage + d.ntiles;
    sphase ^= (total / kStages) & 1;
    stage = total % kStages;
  }
}

// ACCUMULATE items (acc_tma): a stage holds the K source tiles and, after
// them, the current tile of every accumulating destination.  The consumers
// fold the sources (one rounding), write the result over source 0's tile when
// a plain destination needs it, and add it into each recv tile in place (one
// more rounding, as store_result does); one thread then bulk-stores every
// destination's tile.  No consumer global load or store is left.
template <int DT>
__device__ __forceinline__ void consume_acc_tma(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                                uint32_t& stage, uint32_t& sphase) {
  using O = Ops<DT>;
  const uint32_t tile = d.tile;
  const int ks = d.nsrc, ndst = d.ndst;
  bool plain = false;
  for (int k = 0; k < ndst; ++k) plain |= !d.acc[k];
  int prev = -1;  // tid 0: the stage whose bulk stores may still be reading it
  for (uint32_t t = 0; t < d.ntiles; ++t) {
    const uint32_t tb = min(tile, d.vec_bytes - t * tile);
    const uint32_t nv = tb / 16;
    mbar_wait(&sm.full[stage], sphase);
    char* sb = stages + (size_t)stage * kStageBytes;
    for (uint32_t v = tid; v < nv; v += kConsumers) {
      char* pv = sb + (size_t)v * 16;
      uint4 r;
      if (ks == 1) {
        r = lds16(pv);
      } else {
        typename O::Acc a = O::widen(lds16(pv));
        for (int k = 1; k < ks; ++k) O::add(a, lds16(pv + (size_t)k * tile));
        r = O::narrow(a);
        if (plain) sts16(pv, r);
      }
      for (int k = 0; k < ndst; ++k) {
        if (!d.acc[k]) continue;
        char* q = pv + (size_t)d.acc_slot[k] * tile;
        typename O::Acc b = O::widen(lds16(q));
        O::add(b, r);
        sts16(q, O::narrow(b));
      }
    }
    fence_proxy_async_smem();
    consumer_sync();  // every tile of this stage is final in shared memory
    if (tid == 0) {
      for (int k = 0; k < ndst; ++k)
        tma_store(d.dst[k] + (size_t)t * tile, sb + (size_t)(d.acc[k] ? d.acc_slot[k] : 0) * tile, tb);
      tma_store_commit();
      if (prev >= 0) {
        tma_store_wait_read<1>();
        mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
      }
      prev = (int)stage;
    }
    if (++stage == kStages) { stage = 0; sphase ^= 1; }
  }
  if (tid == 0 && prev >= 0) {
    tma_store_wait_read<0>();
    mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
  }
}

// Fold the tiles of a K >= 2 item whose destinations are all plain stores
// (no accumulation) and whose sources fit one stage: the consumers fold each
// vector in shared memory, in place over source 0's tile, and one thread
// stores the folded tile to every destination with TMA bulk stores (as
// copy_tma does for K = 1).  Consumer threads then issue no global stores at
// all; a stage is released once its bulk stores have read it.
template <int DT>
__device__ __forceinline__ void consume_fold_tma(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                                 uint32_t& stage, uint32_t& sphase) {
  using O = Ops<DT>;
  const uint32_t tile = d.tile, vec_bytes = d.vec_bytes, ntiles = d.ntiles;
  const int ks = d.nsrc, ndst = d.ndst;
  int prev = -1;  // tid 0: the stage whose bulk stores may still be reading it
  for (uint32_t t = 0; t < ntiles; ++t) {
    const uint32_t tb = min(tile, vec_bytes - t * tile);
    const uint32_t nv = tb / 16;
    mbar_wait(&sm.full[stage], sphase);
    char* sb = stages + (size_t)stage * kStageBytes;
#pragma unroll 2
    for (uint32_t v = tid; v < nv; v += kConsumers) {
      char* pv = sb + (size_t)v * 16;
      typename O::Acc a = O::widen(lds16(pv));
      for (int k = 1; k < ks; ++k) O::add(a, lds16(pv + (size_t)k * tile));
      sts16(pv, O::narrow(a));  // one rounding; each thread overwrites only vectors it read
    }
    fence_proxy_async_smem();
    consumer_sync();  // the whole folded tile is in shared memory
    if (tid == 0) {
      for (int k = 0; k < ndst; ++k) tma_put<DT>(d.dst[k] + (size_t)t * tile, sb, tb, d.acc[k]);
      tma_store_commit();
      if (prev >= 0) {
        tma_store_wait_read<1>();
        mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
      }
      prev = (int)stage;
    }
    if (++stage == kStages) { stage = 0; sphase ^= 1; }
  }
  if (tid == 0 && prev >= 0) {
    tma_store_wait_read<0>();
    mbar_arrive_cnt(&sm.empty[prev], kConsumerWarps);
  }
}

// Fold the tiles of a K >= 2 item: every stage holds ks source tiles; a tile
// of K > 8 sources spans several stages (passes) accumulated in registers
// (then the tile is at most stage / 8 bytes, one round).  A single-pass tile
// larger than one round (VPT x 16 B x consumers: K = 2, 3 with 64 KiB stages)
// is folded round by round while the stage is held.
template <int DT, int VPT>
__device__ __forceinline__ void consume_fold(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                             uint32_t& stage, uint32_t& sphase) {
  using O = Ops<DT>;
  const bool warp_lane0 = (tid & 31) == 0;
  constexpr uint32_t kRound = VPT * kConsumers;
  for (uint32_t t = 0; t < d.ntiles; ++t) {
    const uint32_t nv = min(d.tile, d.vec_bytes - t * d.tile) / 16;
    if (kLargeTiles && nv > kRound) {  // single pass (d.passes == 1), several rounds
      mbar_wait(&sm.full[stage], sphase);
      fold_rounds<DT>(stages + (size_t)stage * kStageBytes, d, tid, t, nv);
      __syncwarp();
      if (warp_lane0) mbar_arrive(&sm.empty[stage]);
      if (++stage == kStages) { stage = 0; sphase ^= 1; }
      continue;
    }
    typename O::Acc a[VPT];
    for (int p = 0; p < d.passes; ++p) {
      const int ks = min((int)d.ks, (int)d.nsrc - p * (int)d.ks);
      mbar_wait(&sm.full[stage], sphase);
      const char* sb = stages + (size_t)stage * kStageBytes;
#pragma unroll
      for (int j = 0; j < VPT; ++j) {
        const uint32_t v = tid + j * kConsumers;
        if (v < nv) {
          const char* pv = sb + (size_t)v * 16;
          int k = 0;
          if (p == 0) {
            a[j] = O::widen(lds16(pv));
            k = 1;
          }
          for (; k < ks; ++k) O::add(a[j], lds16(pv + (size_t)k * d.tile));
        }
      }
      __syncwarp();
      if (warp_lane0) mbar_arrive(&sm.empty[stage]);
      if (++stage == kStages) { stage = 0; sphase ^= 1; }
    }
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const uint32_t v = tid + j * kConsumers;
      if (v < nv) store_result<DT>(d, (size_t)t * d.tile + (size_t)v * 16, O::narrow(a[j]));  // one rounding
    }
  }
}

// Single-pass fold whose tile is larger than one register round: every tile
// is folded round by round (fold_rounds) while its stage is held.
template <int DT>
__device__ __forceinline__ void consume_fold_held(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                                  uint32_t& stage, uint32_t& sphase) {
  for (uint32_t t = 0; t < d.ntiles; ++t) {
    const uint32_t nv = min(d.tile, d.vec_bytes - t * d.tile) / 16;
    mbar_wait(&sm.full[stage], sphase);
    fold_rounds<DT>(stages + (size_t)stage * kStageBytes, d, tid, t, nv);
    __syncwarp();
    if ((tid & 31) == 0) mbar_arrive(&sm.empty[stage]);
    if (++stage == kStages) { stage = 0; sphase ^= 1; }
  }
}

// One-source item with generic-proxy destinations (accumulation without
// acc_red / acc_tma): every tile is copied round by round while its stage is
// held (rare path, kept small so it does not set the kernel's register budget)
template <int DT>
__device__ __forceinline__ void consume_copy_held(Smem& sm, char* stages, const ItemDesc& d, int tid,
                                                  uint32_t& stage, uint32_t& sphase) {
  for (uint32_t t = 0; t < d.ntiles; ++t) {
    const uint32_t nv = min(d.tile, d.vec_bytes - t * d.tile) / 16;
    mbar_wait(&sm.full[stage], sphase);
    copy_rounds<DT>(stages + (size_t)stage * kStageBytes, d, tid, t, nv);
    __syncwarp();
    if ((tid & 31) == 0) mbar_arrive(&sm.empty[stage]);
    if (++stage == kStages) { stage = 0; sphase ^= 1; }
  }
}

// ------------------------------------------------------------- producer
// STAGED late join: decision word of chunk `chunk` of the slot `r` of task t
template <int DT, class LP>
__device__ __forceinline__ uint64_t* dec_word(char* const (*base)[LP::kRanks], const BufRef& r, const Task& t,
                                              uint64_t half_off, uint32_t chunk) {
  return reinterpret_cast<uint64_t*>(base[kBufArena][r.rank] + half_off + r.bias +
                                     (int64_t)(t.lo * Ops<DT>::kEsize) - (int64_t)late_dec_bytes(t.nchunks)) + chunk;
}

// R: the task's refs (R[0] = refs[t.ref0]), in global memory or in the
// CTA's first-item blob.  decided: STAGED late join, second pass after the
// item's waits with `decision` = the late mask (kLateRoot) or "the parent
// broadcast anything" (kLatePull).
template <int DT, class LP>
__device__ __forceinline__ void fill_desc(const LP& P, char* const (*base)[LP::kRanks],
                                          ItemDesc& d, const Item& item, const Task& t, const BufRef* R,
                                          uint64_t half_off, int lane, uint32_t it, int* nwait_eff,
                                          uint64_t epoch, bool decided = false, uint64_t decision = 0) {
  constexpr int esize = Ops<DT>::kEsize;
  const uint64_t e0 = t.lo + (uint64_t)item.chunk * t.chunk_elems + item.off;
  // late join (phase 1) / complement (phase 2): which candidate ranks are folded
  uint64_t late = 0;
  bool dropped = (int)t.owner == P.drop_rank, force_acc = false;
  int nreg = t.nsrc, op = t.op;
  int need_decide = 0, has_dec = 0, dec_val = 1, wait0 = 0;
  *nwait_eff = t.nwait;
  if (P.late_mode && !dropped && t.lkind == kLatePush) {
    // the late rank's own chunk goes to the root iff it is ready now (phase 1)
    // / iff it did not go in phase 1 (phase 2)
    int pushed = 0;
    if (lane == 0) {
      if (P.late_mode == 1) {
        pushed = ld_acquire(reinterpret_cast<const uint64_t*>(base[kBufArena][t.owner] + ArenaHeader::kReady),
                            P.ipc) >= P.late_ticket;
        P.late_bits[it] = pushed ? 1 : 0;
      } else {
        pushed = P.late_bits[it] == 0;
      }
    }
    pushed = __shfl_sync(0xffffffffu, pushed, 0);
    if (!pushed) op = kOpNone;
    has_dec = 1;
    dec_val = pushed;
  } else if (P.late_mode && !dropped && t.lkind == kLateRoot) {
    if (P.late_mode == 2) {  // only the late slots' flags; recv += fold of what is left
      nreg = 0;
      wait0 = t.nwait - t.nlwait;
      *nwait_eff = t.nlwait;
      op = kOpFold;
      force_acc = true;
    }
    if (!decided) {
      need_decide = 1;
    } else {
      late = decision;
      if (P.late_mode == 2) {
        if (!late) op = kOpNone;
        has_dec = 1;
        dec_val = late != 0;
      } else if (late && t.op == kOpZero) {
        op = kOpFold;
      }
    }
  } else if (P.late_mode && !dropped && t.lkind == kLatePull) {
    if (P.late_mode == 2) {
      if (!decided) {
        need_decide = 1;
      } else {  // add the parent's slot iff it broadcast anything, and forward the decision
        if (decision) force_acc = true;
        else op = kOpNone;
        has_dec = 1;
        dec_val = decision != 0;
      }
    }
  } else if (P.late_mode && !dropped) {
    if (t.nlate == 0) {
      dropped = P.late_mode == 2;  // phase 2 only runs the roots' folds
    } else {
      late = late_select_warp(P, t, it, lane, epoch);
      if (P.late_mode == 2) {
        nreg = 0;
        *nwait_eff = 0;
        op = kOpFold;
        force_acc = true;
        dropped = late == 0;
      } else if (late && t.op == kOpZero) {
        op = kOpFold;
      }
    }
  }
  const int nsrc = nreg + __popcll(late);
  int misaligned = 0;
  for (int i = lane; i < nsrc + t.ndst; i += 32) {
    const BufRef r = i < nreg ? R[i]
                   : i < nsrc ? R[t.nsrc + t.ndst + nth_bit(late, i - nreg)]
                              : R[t.nsrc + (i - nsrc)];
    char* p = base[r.kind][r.rank] + (r.kind == kBufArena ? half_off : 0) + r.bias + (int64_t)(e0 * esize);
    misaligned |= (reinterpret_cast<uintptr_t>(p) & 15) != 0;
    if (i < nsrc) {
      d.src[i] = p;
    } else {
      d.dst[i - nsrc] = p;
      // (force_acc: recv += result; a STAGED broadcast slot still takes the plain result)
      d.acc[i - nsrc] = r.accum || (force_acc && r.kind == kBufRecv);
    }
  }
  for (int i = lane; i < t.npost; i += 32) {
    const FlagRef f = P.flags[t.flag0 + t.nwait + i];
    d.post[i] = reinterpret_cast<uint64_t*>(base[kBufArena][f.rank] + half_off + f.off) + item.chunk;
  }
  misaligned = __any_sync(0xffffffffu, misaligned);
  __syncwarp();
  if (lane == 0) {
    d.need_decide = (uint8_t)need_decide;
    d.wait0 = (uint16_t)wait0;
    d.dec_val = (uint8_t)dec_val;
    d.ndec = 0;
    if (has_dec)  // decision words of the arena destinations (the slots this chunk lands in)
      for (int k = 0; k < t.ndst && d.ndec < 2; ++k) {
        const BufRef r = R[t.nsrc + k];
        if (r.kind == kBufArena) d.dec[d.ndec++] = dec_word<DT, LP>(base, r, t, half_off, item.chunk);
      }
    d.nsrc = (uint16_t)nsrc;
    d.ndst = t.ndst;
    d.op = (uint16_t)op;
    d.npost = t.npost;
    d.len = item.len;
    d.dropped = dropped;
    int any_acc = 0;
    for (int k = 0; k < t.ndst; ++k) any_acc |= d.acc[k];
    d.any_acc = any_acc;
    const uint64_t bytes = (uint64_t)item.len * esize;
    d.scalar_only = misaligned || op != kOpFold || bytes < 16;
    d.vec_bytes = d.scalar_only ? 0 : (uint32_t)(bytes & ~uint64_t(15));
    const int ks = nsrc < kMaxKS ? (nsrc > 0 ? nsrc : 1) : kMaxKS;
    d.ks = (uint16_t)ks;
    d.passes = (uint16_t)((nsrc + kMaxKS - 1) / kMaxKS);
    uint32_t tile = kStageBytes / (uint32_t)ks / 4096u * 4096u;
    d.tile = tile;
    d.ntiles = d.vec_bytes ? (d.vec_bytes + tile - 1) / tile : 0;
    // Phase 2 (ACCUMULATE): recv += result used to be a load, add and store
    // per destination per vector, one memory latency after another; with the
    // recv tiles brought in by TMA next to the sources, the read-modify-write
    // happens in shared memory and leaves by bulk stores.
    int nacc = 0;
    for (int k = 0; k < t.ndst; ++k) nacc += d.acc[k] ? 1 : 0;
    // accumulating destinations by bulk reduce-add (default): the stage holds
    // only the sources; the folded tile goes to every destination by TMA
    d.acc_red = kFoldTma && P.acc_red && nacc > 0 && !d.scalar_only && nsrc >= 1 && nsrc <= kMaxKS;
    d.acc_tma = kFoldTma && !d.acc_red && nacc > 0 && !d.scalar_only && nsrc >= 1 && nsrc <= kMaxKS &&
                nsrc + nacc <= kMaxAccTiles;
    if (d.acc_tma) {
      int j = 0;
      for (int k = 0; k < t.ndst; ++k) d.acc_slot[k] = d.acc[k] ? (uint8_t)(nsrc + j++) : (uint8_t)0;
      const uint32_t at = kStageBytes / (uint32_t)(nsrc + nacc) / 512u * 512u;
      d.ks = (uint16_t)nsrc;
      d.passes = 1;
      d.tile = at;
      d.ntiles = (d.vec_bytes + at - 1) / at;
    }
  }
}

template <int DT, int NR>
#ifdef ADAPCC_TMA_MAXNREG
// explicit register budget (tuning only, see engine_tma_staged.cu)
__global__ void __maxnreg__(ADAPCC_TMA_MAXNREG)
#else
__global__ void __launch_bounds__(kTmaThreads, ADAPCC_TMA_MINB)
#endif
engine_tma_kernel(const __grid_constant__ LaunchParamsT<NR> P) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  Smem& sm = *reinterpret_cast<Smem*>(smem_raw);
  __shared__ char* sbase[3][NR];  // P.send / P.recv / P.hdr (indexed by BufKind), copied from the params
  char* stages = reinterpret_cast<char*>(smem_raw) + kSmemHeader;
  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;
  const bool sys = P.ipc;
  const uint64_t t_entry = P.trace ? globaltimer() : 0;
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], kConsumerWarps);
    }
    for (int s = 0; s < kQ; ++s) {
      mbar_init(&sm.qfull[s], 1);
      mbar_init(&sm.qempty[s], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    sm.abort = 0;
  }
  // the producer's first item, its task and refs: one round trip of
  // immutable plan data, issued before the stream-order wait below
  const bool use_blob = blockIdx.x < P.nfirst;
  if (warp == kConsumerWarps) {
    if (use_blob)
      for (uint32_t i = lane; i < P.first_words; i += 32)
        sm.blob[i] = P.first[(size_t)blockIdx.x * P.first_words + i];
    // buffer bases into shared memory (indexed by BufKind)
    for (int i = lane; i < 3 * P.nranks; i += 32) {
      const int k = i / P.nranks, q = i - k * P.nranks;
      sbase[k][q] = k == 0 ? P.send[q] : k == 1 ? P.recv[q] : P.hdr[q];
    }
    __syncwarp();
    // A plan without arena streams or flags (DIRECT: loopback and zero-copy)
    // describes its first item before the stream-order wait: its pointers do
    // not depend on the epoch's parity half, so under PDL this overlaps the
    // previous kernel.  Late join decides per item from ready words: after.
    if (use_blob && P.arena_free && P.late_mode == 0) {
      int nwait = 0;
      fill_desc<DT>(P, sbase, sm.q[0], *reinterpret_cast<const Item*>(&sm.blob[0]),
                    *reinterpret_cast<const Task*>(&sm.blob[1]),
                    reinterpret_cast<const BufRef*>(&sm.blob[kBlobRef0]), 0, lane, blockIdx.x, &nwait, 0);
      __syncwarp();
    }
  }
  // shared-memory set-up above; the epoch, counters, arenas and user buffers
  // below belong to the stream order (PDL: the previous launch)
  pdl_trigger();
  pdl_wait();
  if (tid == 0) {
    const uint64_t e = *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) + 1;
    sm.epoch = e;
    if (blockIdx.x == 0) {
      P.state->work[(e + 1) & 1] = 0;
      P.state->done[(e + 1) & 1] = 0;
    }
  }
  __syncthreads();
  const uint64_t t_ready = P.trace ? globaltimer() : 0;
  const uint64_t epoch = sm.epoch;
  const unsigned par = (unsigned)(epoch & 1);
  const uint64_t half_off = kArenaHeader + par * P.half_bytes;
  if (P.ipc && epoch > 2) {  // peers done with the last user of this half
    if (tid < P.nranks && tid != P.my_rank && ((P.members >> tid) & 1))
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[tid]), epoch - 2, P)) sm.abort = 1;
    __syncthreads();
  }
  if (P.ipc && P.check_sig && !check_call_sig(P, epoch)) sm.abort = 1;  // before any byte moves
  if (P.ipc && P.zc) {  // zero-copy: peers read/write our user buffers directly
    if (blockIdx.x == 0 && tid == 0)
      st_release(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank] + ArenaHeader::kEntered), epoch, true);  // entered
    if (tid < P.nranks && tid != P.my_rank && ((P.members >> tid) & 1))
      if (!wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[tid] + ArenaHeader::kEntered), epoch, P)) sm.abort = 1;
    __syncthreads();
  }

  if (warp == kConsumerWarps) {
    // ================================================================ producer
    uint32_t stage = 0, sphase = 0, qi = 0, qphase = 0;
    // claiming as in the LDG kernel: item blockIdx.x first, then the counter
    // offset by the grid; stop after an item among the last gridDim.x
    bool first = true, last = false;
    // Phase 2 of a late join (LATE_COMPLEMENT) has work only in the items
    // phase 1 listed as incomplete: claims index that list (no waits in phase
    // 2, so any order is deadlock-free) and everything else is never touched.
    const bool listed = P.late_mode == 2 && P.late_list != nullptr;
    const uint32_t nclaim = listed ? late_listed(P) : P.nitems;
    for (;;) {
      uint32_t it = 0;
      int stop_i = 0;
      if (lane == 0 && !last) {
        it = first ? blockIdx.x : gridDim.x + atomicAdd(&P.state->work[par], 1u);
        last = (uint64_t)it + gridDim.x >= nclaim;
        if (listed) it = it < nclaim ? P.late_list[it] : P.nitems;
      } else if (lane == 0) {
        it = P.nitems;
      }
      const uint64_t tr0 = P.trace ? globaltimer() : 0;
      // queue slot free: every lane waits (acquire), since every lane rewrites
      // the slot's descriptor that the consumers of item i - kQ were reading
      mbar_wait(&sm.qempty[qi], qphase ^ 1);
      if (lane == 0) {
        stop_i = it >= P.nitems || *reinterpret_cast<volatile int*>(&sm.abort) != 0;
        first = false;
      }
      it = __shfl_sync(0xffffffffu, it, 0);
      bool stop = __shfl_sync(0xffffffffu, stop_i, 0) != 0;
      ItemDesc& d = sm.q[qi];
      const bool fb = use_blob && !listed && it == blockIdx.x;  // this CTA's first item (blob in shared memory)
      const Item item = stop ? Item{} : fb ? *reinterpret_cast<const Item*>(&sm.blob[0]) : P.items[it];
      const Task& t = fb ? *reinterpret_cast<const Task*>(&sm.blob[1]) : P.tasks[item.task];
      if (!stop) {
        int nwait = 0;
        if (!(fb && P.arena_free && P.late_mode == 0)) {  // (else described before the wait, above)
          const BufRef* R = fb ? reinterpret_cast<const BufRef*>(&sm.blob[kBlobRef0]) : P.refs + t.ref0;
          fill_desc<DT>(P, sbase, d, item, t, R, half_off, lane, it, &nwait, epoch);
          __syncwarp();
        }
        if (!d.dropped) {
          int ok = 1;
          for (int i = lane; i < nwait; i += 32) {
            const FlagRef f = P.flags[t.flag0 + d.wait0 + i];
            const uint64_t* fl = reinterpret_cast<const uint64_t*>(sbase[kBufArena][f.rank] + half_off + f.off) + item.chunk;
            ok &= wait_flag(fl, epoch, P);
          }
          if (!__all_sync(0xffffffffu, ok)) {
            stop = true;
            if (lane == 0) sm.abort = 1;
          }
          if (!stop && d.need_decide) {
            // STAGED late join: the decision words are readable now (their flags acquired)
            const BufRef* R = fb ? reinterpret_cast<const BufRef*>(&sm.blob[kBlobRef0]) : P.refs + t.ref0;
            uint64_t decision = 0;
            if (lane == 0) {
              if (t.lkind == kLateRoot) {
                const uint64_t prev = P.late_mode == 2 ? P.late_bits[it] : 0;
                for (uint32_t j = 0; j < t.nlate; ++j) {
                  const BufRef r = R[t.nsrc + t.ndst + j];
                  bool in;
                  if (r.kind == kBufArena)
                    in = *reinterpret_cast<volatile uint64_t*>(dec_word<DT, LaunchParamsT<NR>>(sbase, r, t, half_off,
                                                                                            item.chunk)) != 0;
                  else if (P.late_mode == 1)
                    in = ld_acquire(reinterpret_cast<const uint64_t*>(sbase[kBufArena][r.rank] + ArenaHeader::kReady),
                                    P.ipc) >= P.late_ticket;
                  else
                    in = ((prev >> j) & 1) == 0;
                  if (in) decision |= 1ull << j;
                }
                if (P.late_mode == 1) P.late_bits[it] = decision;
              } else {  // kLatePull, phase 2: did the parent broadcast anything?
                decision = *reinterpret_cast<volatile uint64_t*>(
                               dec_word<DT, LaunchParamsT<NR>>(sbase, R[0], t, half_off, item.chunk)) != 0;
              }
            }
            decision = __shfl_sync(0xffffffffu, decision, 0);
            int nw2 = 0;
            fill_desc<DT>(P, sbase, d, item, t, R, half_off, lane, it, &nw2, epoch, true, decision);
            __syncwarp();
          }
        }
      }
      if (lane == 0) {
        d.stop = stop;
        if (P.trace) {
          d.item = it;
          d.tr0 = tr0;
          d.tr1 = globaltimer();
        }
        fence_proxy_async();      // acquired peer/arena data -> async-proxy (TMA) reads
        mbar_arrive(&sm.qfull[qi]);
      }
      __syncwarp();
      if (stop) break;
      if (!d.dropped && !d.scalar_only) {
        for (uint32_t tt = 0; tt < d.ntiles; ++tt) {
          const uint32_t tb = min(d.tile, d.vec_bytes - tt * d.tile);
          for (int p = 0; p < d.passes; ++p) {
            const int ks = min((int)d.ks, (int)d.nsrc - p * (int)d.ks);
            // every issuing lane acquires the stage's release (its TMA load
            // overwrites what the consumers read); lane 0 arms the tx count
#ifndef ADAPCC_LANE0_EMPTY_WAIT
            mbar_wait(&sm.empty[stage], sphase ^ 1);
#else
            if (lane == 0) mbar_wait(&sm.empty[stage], sphase ^ 1);
            __syncwarp();
#endif
            if (lane == 0) {
              int nacc = 0;
              if (d.acc_tma)
                for (int k = 0; k < d.ndst; ++k) nacc += d.acc[k] ? 1 : 0;
              mbar_expect_tx(&sm.full[stage], (uint32_t)(ks + nacc) * tb);
            }
            __syncwarp();
            // One bulk load per lane: a stage's K source tiles (and, with
            // acc_tma, the accumulating destinations' recv tiles) are issued
            // warp-parallel instead of one after another from lane 0.
            char* sb = stages + (size_t)stage * kStageBytes;
            if (lane < ks) {
              tma_load(sb + (size_t)lane * d.tile, d.src[p * d.ks + lane] + (size_t)tt * d.tile, tb,
                       &sm.full[stage]);
            } else if (d.acc_tma) {
              for (int k = 0; k < d.ndst; ++k)
                if (d.acc[k] && d.acc_slot[k] == lane)
                  tma_load(sb + (size_t)lane * d.tile, d.dst[k] + (size_t)tt * d.tile, tb, &sm.full[stage]);
            }
            if (++stage == kStages) { stage = 0; sphase ^= 1; }
          }
        }
      }
      if (++qi == kQ) { qi = 0; qphase ^= 1; }
    }
  } else {
    // =============================================================== consumers
    uint32_t stage = 0, sphase = 0, qi = 0, qphase = 0;
    for (;;) {
      mbar_wait(&sm.qfull[qi], qphase);
      const ItemDesc& d = sm.q[qi];
      if (d.stop) break;
      if (!d.dropped) {
        if (d.op == kOpZero) {
          using E = typename Ops<DT>::E;
          for (int k = 0; k < d.ndst; ++k)
            for (uint64_t e = tid; e < d.len; e += kConsumers) reinterpret_cast<E*>(d.dst[k])[e] = E(0);
        } else if (d.op != kOpNone) {
          if (!d.scalar_only) {
            const uint32_t vpt = d.tile / (16u * kConsumers);  // tile / one round of 1 vector per thread
            if (d.acc_tma) consume_acc_tma<DT>(sm, stages, d, tid, stage, sphase);
            else if (d.nsrc == 1 && (!d.any_acc || d.acc_red)) copy_tma<DT>(sm, stages, d, tid, stage, sphase);
            else if (d.acc_red) consume_fold_tma<DT>(sm, stages, d, tid, stage, sphase);
            // TMA-stored fold where per-thread stores are the cost: tiles above 16 KiB (K = 2, 3 in
            // 64 KiB stages, else fold_rounds; G1 k = 2: 0.86 -> 1.02 of the copy peak) or >= 3
            // destinations (star roots); with 1-2 destinations of small tiles the register path,
            // which frees the stage before storing, is as fast or faster (G1 k = 8: 1.08 vs 1.04)
            else if (kFoldTma && !d.any_acc && d.passes == 1 && (d.tile > 16384 || d.ndst >= 3))
              consume_fold_tma<DT>(sm, stages, d, tid, stage, sphase);
            else if (d.nsrc == 1) {
              // (32 KiB stages: the 8-vector register round of consume_copy set the whole
              // kernel's register budget and made it spill at 2 CTAs/SM -- 96 registers)
              if constexpr (kLargeTiles) consume_copy<DT, 8>(sm, stages, d, tid, stage, sphase);
              else consume_copy_held<DT>(sm, stages, d, tid, stage, sphase);
            }
            else if (vpt >= 4) {
              if constexpr (DT == kBF16) {  // 4 x 8 fp32 accumulators per thread spill at 2 CTAs/SM
                if (!d.any_acc) consume_fold_tma<DT>(sm, stages, d, tid, stage, sphase);
                else consume_fold_held<DT>(sm, stages, d, tid, stage, sphase);
              } else {
                consume_fold<DT, 4>(sm, stages, d, tid, stage, sphase);
              }
            }
            else if (vpt >= 2) consume_fold<DT, 2>(sm, stages, d, tid, stage, sphase);
            else consume_fold<DT, 1>(sm, stages, d, tid, stage, sphase);
          }
          constexpr int esize = Ops<DT>::kEsize;
          scalar_range<DT>(d, d.vec_bytes / esize, d.len, tid);
        }
        consumer_sync();  // every consumer's stores for this item are issued
        if (tid == 0 && d.npost) {
          tma_store_wait_all();  // bulk (async-proxy) stores performed ...
          fence_proxy_async();   // ... and ordered before generic-proxy accesses
          for (int k = 0; k < d.ndec; ++k)  // STAGED late join: the decision travels with the flag
            *reinterpret_cast<volatile uint64_t*>(d.dec[k]) = d.dec_val;
          fence(sys);      // the chunk's bytes (incl. remote NVLink stores) before its flag
          for (int i = 0; i < d.npost; ++i) st_release(d.post[i], epoch, sys);
        }
      }
      if (P.trace && tid == 0 && !d.dropped)
        trace_put(P, d.item, 0, d.tr0, d.tr1, globaltimer(), d.len * Ops<DT>::kEsize * (uint64_t)(d.nsrc + d.ndst));
      consumer_sync();    // all consumers are done reading the descriptor
      if (tid == 0) mbar_arrive(&sm.qempty[qi]);
      if (++qi == kQ) { qi = 0; qphase ^= 1; }
    }
  }
  __syncthreads();
  if (P.trace && tid == 0) trace_put(P, kTraceCta, 0, t_entry, t_ready, globaltimer(), 0);
  if (tid == 0) {
    // across processes this CTA's bulk stores are complete before it counts as
    // done (peers read the published word); in loopback only the next launch
    // reads the epoch, after this grid has completed, so the count goes first
    // and the store drain overlaps it
    if (sys) {
      tma_store_wait_all();
      fence_proxy_async();
      fence(sys);
    }
    const unsigned done = atomicAdd(&P.state->done[par], 1u);
    if (done == gridDim.x - 1) {
      // late join: phase 1 validates its list for phase 2; phase 2 consumed it
      // (every CTA is past its claims), so a repeated phase 2 adds nothing
      if (P.late_mode && P.late_count) P.late_count[1] = P.late_mode == 1 ? epoch : ~0ull;
      *reinterpret_cast<volatile unsigned long long*>(&P.state->epoch) = epoch;
      if (P.ipc) {
        __threadfence_system();
        st_release(reinterpret_cast<uint64_t*>(P.hdr[P.my_rank]), epoch, true);
        if (P.zc)  // our buffers stay in use until every peer has finished this call
          for (int q = 0; q < P.nranks; ++q)
            if (q != P.my_rank && ((P.members >> q) & 1))
              wait_flag(reinterpret_cast<const uint64_t*>(P.hdr[q]), epoch, P);
      }
    }
    if (!sys) tma_store_wait_all();  // bulk stores complete before the CTA exits
  }
}

template <int DT, int NR>
cudaError_t prepare() {
  static bool done = false;
  if (done) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(engine_tma_kernel<DT, NR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)kSmemBytes);
  done = e == cudaSuccess;
  return e;
}

template <int NR>
cudaError_t launch_nr(const LaunchParamsT<NR>& p, int grid, cudaStream_t stream, bool pdl) {
  switch (p.dtype) {
    case kF32:
      if (cudaError_t e = prepare<kF32, NR>()) return e;
      return launch_kernel(engine_tma_kernel<kF32, NR>, grid, kTmaThreads, kSmemBytes, stream, pdl, p);
    case kBF16:
      if (cudaError_t e = prepare<kBF16, NR>()) return e;
      return launch_kernel(engine_tma_kernel<kBF16, NR>, grid, kTmaThreads, kSmemBytes, stream, pdl, p);
    default:
      if (cudaError_t e = prepare<kI32, NR>()) return e;
      return launch_kernel(engine_tma_kernel<kI32, NR>, grid, kTmaThreads, kSmemBytes, stream, pdl, p);
  }
}

}  // namespace

int threads() { return kTmaThreads; }

cudaError_t occupancy(int dtype, int* blocks_per_sm) {
  switch (dtype) {
    case kF32:
      if (cudaError_t e = prepare<kF32, kMaxRanksDev>()) return e;
      return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_tma_kernel<kF32, kMaxRanksDev>,
                                                           kTmaThreads, kSmemBytes);
    case kBF16:
      if (cudaError_t e = prepare<kBF16, kMaxRanksDev>()) return e;
      return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_tma_kernel<kBF16, kMaxRanksDev>,
                                                           kTmaThreads, kSmemBytes);
    default:
      if (cudaError_t e = prepare<kI32, kMaxRanksDev>()) return e;
      return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, engine_tma_kernel<kI32, kMaxRanksDev>,
                                                           kTmaThreads, kSmemBytes);
  }
}

cudaError_t launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl) {
  cudaGetLastError();
  if (p.nranks <= kNarrowRanks) return launch_nr(narrow(p), grid, stream, pdl);
  return launch_nr(p, grid, stream, pdl);
}

}  // namespace ADAPCC_TMA_NS
}  // namespace adapcc
