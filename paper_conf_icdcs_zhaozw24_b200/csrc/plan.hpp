// Plan compiler: (strategy, ready mask, count, dtype, flags, mode) -> FOLD
// tasks + per-chunk flags + ordered work items (engine.cuh).
//
// This is the B200 replacement of the paper's Executor, which "parses
// communication strategies ... together with the information of relay workers
// to generate respective CUDA codes": instead of generating
// code per behaviour tuple we compile the tuples into a task table that one
// persistent, parameterised kernel executes.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "engine.cuh"
#include "strategy.hpp"

namespace adapcc {

enum Mode : int { kDirect = 0, kStaged = 1 };

struct PlanStats {
  uint64_t tasks = 0, items = 0, levels = 0, segments = 0;
  uint64_t bytes_read = 0, bytes_written = 0, remote_bytes = 0, arena_bytes = 0;
};

// One launch worth of work.
struct SegmentPlan {
  std::vector<Task> tasks;
  std::vector<BufRef> refs;
  std::vector<FlagRef> flags;
  std::vector<uint64_t> arena_used;  // per rank, bytes inside one parity half
  uint32_t max_level = 0;
  bool fits = true;                  // flags and data fit their regions
  bool nvls = false;                 // has NVLS tasks (LDG kernel only)
  std::string unsupported;           // non-empty: the call cannot run (reason)
};

struct PlanRequest {
  const Strategy* st = nullptr;
  uint64_t count = 0;       // allreduce: count; allgather: sendcount; alltoall: per peer
  int esize = 4;
  uint64_t ready_mask = 0;
  bool accumulate = false;
  bool late_join = false;   // root tasks carry the non-ready ranks as optional sources (NEXT-1)
  Mode mode = kDirect;
  uint64_t half_bytes = 0;  // arena bytes available per rank per parity half
  // AlltoAllv (NEXT-4): counts[s * n + d] elements go from rank s to rank d;
  // blocks are packed in destination order in the sendbuf and source order in
  // the recvbuf.  nullptr for every other collective.
  const uint64_t* counts = nullptr;
  // Live ranks (NEXT-3: faulty ranks excluded): an excluded rank
  // owns no task and no buffer of it is read or written.
  uint64_t members = ~uint64_t(0);
  // CTAs the call will run on (0: pipeline in units of the strategy's chunks
  // only); small calls subdivide chunks so that every CTA gets work (R8).
  int grid = 0;
  // NVLS scratch bytes per rank (adapcc_nvls_setup; 0 = none): nvls lines
  // need it, the whole mask, and a multi-process communicator
  uint64_t nvls_bytes = 0;
};

// Bytes at the start of each parity half reserved for per-chunk flag words.
uint64_t flag_region_bytes(uint64_t half);

// Builds the segment plans of one call (one per launch; more than one only
// when the staging slots exceed half_bytes).  Returns false + *err when the
// call cannot be planned (e.g. arena too small even for 1 unit per segment).
bool build_plan(const PlanRequest& rq, std::vector<SegmentPlan>* segs, std::string* err);

// Work items of `rank` (-1: all ranks) in deadlock-free order; `grid` CTAs
// will execute them (used to size the pieces of flag-free tasks).
// piece_bytes: traffic per piece (all streams); 0 = automatic (see plan.cpp).
// tma: items for the TMA pipeline kernel (larger mid-size pieces).
// taper: the last ~2 x grid splittable items (flag-free tasks) are cut into
// `taper` sub-pieces each, so the dynamic claim loop ends on short items
// (1 = off, 0 = automatic).
// acc_red: items for the TMA kernel's bulk reduce-add ACCUMULATE path (phase 2):
// automatic pieces of <= 256 KiB and an unconditional tail taper.
std::vector<Item> order_items(const SegmentPlan& p, int rank, int esize, int grid,
                              uint64_t piece_bytes = 0, int taper = 1, bool tma = false, bool acc_red = false);

// Byte accounting for adapcc_plan_stats.
void accumulate_stats(const SegmentPlan& p, int rank, int esize, PlanStats* s);

// Sub-collective ranges (before segmentation) in the collective's element
// coordinates: allreduce/alltoall use partition() over all subs; allgather
// partitions each source's shard over that source's bcast lines.
std::vector<std::pair<uint64_t, uint64_t>> sub_ranges(const Strategy& st, uint64_t count,
                                                      int esize);

}  // namespace adapcc
