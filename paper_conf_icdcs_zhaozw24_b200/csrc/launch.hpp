// Kernel launch parameters of the transfer engine (host <-> device contract).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"

namespace adapcc {

constexpr int kMaxRanksDev = 64;

// Per-communicator device state.  Counters are double-buffered by epoch
// parity: launch e uses [e & 1] and block 0 re-arms [(e + 1) & 1] for the
// next launch, so no host reset is needed between launches (CUDA graphs).
struct DevState {
  unsigned work[2];          // work-item cursor
  unsigned done[2];          // finished CTAs
  unsigned abort;            // watchdog fired
  unsigned pad;
  unsigned long long epoch;  // last completed launch
};

// In-kernel trace record (adapcc_config("trace", capacity)): one per work
// item a CTA executes plus one per CTA and launch (item == kTraceCta), times
// from %globaltimer (ns).  Item: t0 claimed, t1 inputs ready (flags acquired),
// t2 done (stores issued, flags posted).  CTA: t0 entry, t1 after the stream-
// order wait and the epoch read, t2 exit.
struct TraceRec {
  uint32_t launch;  // launch sequence number of the communicator
  uint32_t cta;
  uint32_t item;
  uint32_t task;
  uint64_t t0, t1, t2;
  uint64_t bytes;   // traffic of the item (sources + destinations)
};
static_assert(sizeof(TraceRec) == 48, "TraceRec layout");
constexpr uint32_t kTraceCta = 0xFFFFFFFFu;

// Scalar part of the launch parameters; the per-rank pointer arrays follow in
// LaunchParamsT<NR>.  Kernel parameters are copied into every launch, and a
// launch with 1.8 KB of them costs ~1.5 us more host time than one with a few
// bytes (scripts/debug/host_floor.cu): calls over <= 8 ranks launch the
// kernels instantiated for 8-entry arrays.
struct LaunchCore {
  const Task* tasks;
  const BufRef* refs;
  const FlagRef* flags;
  const Item* items;
  uint32_t nitems;
  uint32_t ntasks;      // flat kernel: it strides through tasks[0 .. ntasks) (no items)
  // LDG kernel: CTA b < nfirst reads its first item (items[b]), that item's
  // task and refs as ONE blob of first_words 16-byte words at first + b *
  // first_words, loaded in a single round trip together with the epoch
  const uint4* first;
  uint32_t nfirst, first_words;
  // static schedule (nfirst == nitems): CTA b runs items b, b + grid, ... in
  // order, reading each item's blob (prefetched during the previous fold)
  // instead of claiming from the counter; still deadlock-free, because the
  // smallest unfinished item's CTA has finished all its earlier items and its
  // inputs come from smaller items
  uint32_t sched_static;
  // 1: no task has arena streams, flag waits or posts (DIRECT plans): item
  // pointers do not depend on the epoch (the TMA kernel describes its first
  // item before the stream-order wait)
  uint32_t arena_free;
  int dtype;
  int nranks;
  int my_rank;          // multi-process: this rank; loopback: -1
  int ipc;              // 1: multi-process (.sys scope, start check, done publish)
  int zc;               // 1: zero-copy DIRECT plan across processes (entry/exit barriers)
  int late_mode;        // 0: off; 1: late join (phase 1); 2: complement (phase 2)
  int acc_red;          // TMA kernel: accumulating destinations by bulk reduce-add (else smem read-modify-write)
  uint64_t late_ticket; // ready word value that admits a late rank (phase 1)
  uint64_t* late_bits;  // per work item: late candidates included in phase 1
  // Phase 1 lists the items that missed a late rank (late_list[i], i < count)
  // and phase 2 runs exactly those.  late_count[0] = (gen << 32) | count, where
  // gen is the low 32 bits of the epoch of the phase-1 launch that appended:
  // the first append of a launch with a new gen restarts the count, so a list
  // never holds a stale entry (no reset step, CUDA-graph replays included).
  // late_count[1] = epoch of the last completed phase 1 of this plan (written
  // by its last CTA; ~0 after a phase 2 consumed the list): phase 2 runs the
  // list only if its gen matches, so a phase 1 that listed nothing, or a
  // repeated phase 2, adds nothing.  Both words are per plan: phase 1 / phase 2
  // pairs of different plans may interleave on a stream.
  uint32_t* late_list;
  unsigned long long* late_count;
  int drop_rank;        // test hook (loopback): tasks owned by this rank are skipped
  uint64_t members;     // live ranks: excluded ranks are skipped by the IPC barriers
  uint64_t half_bytes;  // bytes of one parity half of an arena
  uint64_t timeout_ns;
  uint64_t sig;         // call signature (debug check): hash of the call every rank must agree on
  int check_sig;        // 1: multi-process debug mode, compare `sig` with every peer's before any data moves
  TraceRec* trace;        // nullptr: tracing off
  unsigned* trace_n;      // records written (may exceed trace_cap: the excess is dropped)
  uint32_t trace_cap;
  uint32_t launch_seq;
  DevState* state;
  int* err;             // host-mapped error word
  char* nvls_uc;        // NVLS scratch of this rank: unicast / multicast address (nullptr: no NVLS)
  char* nvls_mc;
  uint64_t nvls_stride; // 0: a real multicast team; > 0: loopback emulation -- virtual rank q's scratch is
                        // nvls_uc + q * nvls_stride and the kernel sums / stores the n copies itself
};

template <int NR>
struct LaunchParamsT : LaunchCore {
  static constexpr int kRanks = NR;
  char* send[NR];
  char* recv[NR];
  char* hdr[NR];  // arena base of each rank (peer-mapped): [header | half 0 | half 1]
};
constexpr int kNarrowRanks = 8;
using LaunchParams = LaunchParamsT<kMaxRanksDev>;  // what the host fills
using LaunchParamsNarrow = LaunchParamsT<kNarrowRanks>;

// the same call in the narrow parameter block (nranks <= kNarrowRanks)
inline LaunchParamsNarrow narrow(const LaunchParams& p) {
  LaunchParamsNarrow n;
  static_cast<LaunchCore&>(n) = static_cast<const LaunchCore&>(p);
  for (int q = 0; q < kNarrowRanks; ++q) {
    n.send[q] = p.send[q];
    n.recv[q] = p.recv[q];
    n.hdr[q] = p.hdr[q];
  }
  return n;
}

// Words of the 4 KiB arena header (byte offsets).  Each rank writes only its
// own header; peers read it over NVLink.
struct ArenaHeader {
  static constexpr int kDone = 0;      // last epoch this rank finished (parity-half reuse, exit barrier)
  static constexpr int kEntered = 8;   // zero-copy: epoch this rank's kernel entered
  static constexpr int kReady = 16;    // late join: ticket this rank signalled ready for
  static constexpr int kSig = 64;      // debug check: call signature of epoch e in slot e & 3 ...
  static constexpr int kSigEpoch = 96; // ... published by epoch e in slot e & 3 (release)
};

// engine.cu: 128-bit LDG/STG fold (256 threads, 2 CTAs/SM)
int engine_threads();
cudaError_t engine_occupancy(int dtype, int* blocks_per_sm);
cudaError_t engine_launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl);
// probe.cu: one probe message -- `bytes` from src to each of dst[0..ndst) by
// TMA bulk copies (link profiling, NEXT-2)
cudaError_t probe_launch(const char* src, char* const* dst, int ndst, uint64_t bytes, int grid,
                         cudaStream_t stream);
// store `value` into a ready word after all prior work on `stream` (late join)
// (and into board, a host-mapped readiness word, if not null)
cudaError_t engine_signal(uint64_t* word, uint64_t value, bool sys, uint64_t* board, cudaStream_t stream);
// one thread spinning on %globaltimer for `ns` (controlled straggler, benchmarks)
cudaError_t engine_spin(uint64_t ns, cudaStream_t stream);
// engine_tma_impl.cuh: TMA bulk-copy pipeline (1 producer + 8 consumer warps),
// one instantiation per plan kind
namespace tma_direct {
int threads();
cudaError_t occupancy(int dtype, int* blocks_per_sm);
cudaError_t launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl);
}  // namespace tma_direct
// engine_flat.cu: plans without flags or arena streams -- the whole grid
// strides through one task after another
namespace flat {
cudaError_t launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl);
}  // namespace flat
namespace tma_staged {
int threads();
cudaError_t occupancy(int dtype, int* blocks_per_sm);
cudaError_t launch(const LaunchParams& p, int grid, cudaStream_t stream, bool pdl);
}  // namespace tma_staged

}  // namespace adapcc
