// Device-visible plan tables of the AdapCC transfer engine.
//
// A call is compiled on the host (plan.cpp) into FOLD tasks: "wait for these
// per-chunk flags, fold K source streams left to right, write the result to D
// destination streams (some accumulating), post these per-chunk flags".  Every
// step of the paper's executor maps onto one task kind:
//   - aggregation kernel at a node with hasKernel: K >= 2
//   - chunk send / relay forward: K = 1
//   - root hand-off + broadcast "reversely": K = 1, D >= 1
// A work item is one (task, chunk); items are ordered by (chunk + level,
// level, task) so that every wait targets an item earlier in the order, which
// makes the dynamic fetch deadlock-free.
#pragma once

#include <cstdint>

namespace adapcc {

constexpr int kMaxFold = 64;   // max sources of one fold (<= ranks)
constexpr int kMaxDst = 65;    // max destinations of one task (<= ranks + 1)
constexpr int kArenaHeader = 4096;  // per-rank arena header (done epoch)
// LDG kernel: per-CTA "first item" blob = Item, Task, then the task's refs
// (sources, destinations, late candidates), in 16-byte words; plans whose
// first items need more words go without blobs.
constexpr int kFirstMaxWords = 72;

enum BufKind : uint8_t { kBufSend = 0, kBufRecv = 1, kBufArena = 2,
                         kBufNvlsUc = 3,   // this rank's NVLS scratch, unicast address (adapcc_nvls_setup)
                         kBufNvlsMc = 4 }; // the NVLS scratch, multicast address (every rank's copy at once)
constexpr int kNumBufKinds = 5;
enum DType : int { kF32 = 0, kBF16 = 1, kI32 = 2 };
enum TaskOp : uint16_t { kOpFold = 0, kOpZero = 1, kOpNone = 2 /* (runtime only) no data */,
                         kOpNvls = 3 /* dst(mc) = switch sum of src(mc) over every rank: multimem.ld_reduce + st */ };
// Late join on STAGED plans (NEXT-1): the late rank pushes its chunk
// to the tree root itself, conditionally, and every decision travels in a
// per-chunk word placed before the slot it describes.
enum LateKind : uint8_t {
  kLateNone = 0,  // DIRECT late join (nlate > 0 at roots) or no late join
  kLatePush = 1,  // owner = a late rank: push its chunk into its landing slot at the root iff
                  // ready (phase 1) / iff not pushed in phase 1 (phase 2); decision word = pushed
  kLateRoot = 2,  // root: late candidates = landing slots (decision words) or its own input
                  // (ready word); the last nlwait waits are the late slots' flags
  kLatePull = 3,  // broadcast pull: phase 2 accumulates iff the parent's decision word says so
};

// address(e) = base(kind, rank) + bias + e * esize, e = element index in the
// task's coordinate system.
struct BufRef {
  int64_t bias;
  uint8_t kind;
  uint8_t rank;
  uint8_t accum;   // destination: recv += value (ACCUMULATE)
  uint8_t pad[5];
};
static_assert(sizeof(BufRef) == 16, "BufRef layout");

// per-chunk flag word: arena(rank) + off + 8 * chunk (inside the parity half)
struct FlagRef {
  uint64_t off;
  uint32_t rank;
  uint32_t pad;
};
static_assert(sizeof(FlagRef) == 16, "FlagRef layout");

struct Task {
  uint64_t lo, hi;          // element range covered by the task
  uint32_t chunk_elems;     // C_m / esize
  uint32_t nchunks;
  uint16_t nsrc, ndst, nwait, npost;
  uint32_t ref0;            // refs[ref0 .. ref0+nsrc) sources, then ndst destinations
  uint32_t flag0;           // flags[flag0 .. +nwait) waits, then npost posts
  uint32_t level;
  uint16_t op;
  uint16_t owner;           // executing rank
  uint16_t nlate;           // late-join candidates: refs[ref0+nsrc+ndst .. +nlate) (root tasks)
  uint8_t lkind;            // LateKind
  uint8_t nlwait;           // kLateRoot: the last nlwait of the nwait waits belong to late candidates
};

// A work item covers elements [off, off+len) of chunk `chunk` of `task`.  A
// task that posts flags is executed one whole chunk per item (the flag means
// "the whole chunk is written"); a task without posts may be split into
// several pieces per chunk so that CTAs get even work (grid balance).
struct Item {
  uint32_t task;
  uint32_t chunk;
  uint32_t off;   // elements from the chunk start
  uint32_t len;   // elements
};
static_assert(sizeof(Item) == 16, "Item layout");

// Flat kernel (engine_flat.cu) descriptor blob, built at plan time: one
// FlatTask per task, then every task's refs (sources, then destinations) with
// the task's range start folded into BufRef::bias and the task's index in
// BufRef::pad[0..1].
struct FlatTask {
  uint64_t len;      // elements of the task
  uint64_t vstart;   // set on the device: first index of the task's vectors in the launch's vector space
  uint32_t ref0;     // its first ref in the blob's ref array
  uint16_t nsrc, ndst;
  uint16_t op, owner;
  uint8_t any_acc;   // some destination accumulates (recv += result)
  uint8_t bad;       // set on the device: some stream is not 16-byte aligned
  uint8_t pad[2];
};
static_assert(sizeof(FlatTask) == 32, "FlatTask layout");
constexpr uint32_t kFlatMaxRefs = 1536;  // per segment (shared memory: blob + pointers + flags < 48 KiB)
constexpr uint32_t kFlatMaxTasks = 128;
#ifdef __CUDACC__
__host__ __device__
#endif
inline uint32_t flat_nrefs(uint32_t words, uint32_t ntasks) { return words - 2 * ntasks; }
#ifdef __CUDACC__
__host__ __device__
#endif
inline size_t flat_smem_bytes(uint32_t words, uint32_t ntasks) {
  const uint32_t nrefs = flat_nrefs(words, ntasks);
  return ((size_t)words * 16 + (size_t)nrefs * 9 + 15) / 16 * 16;
}

// STAGED late join: per-chunk decision words (8 bytes each) sit just before
// the slot they describe, in an array of late_dec_bytes(nchunks) bytes
#ifdef __CUDACC__
__host__ __device__
#endif
inline uint64_t late_dec_bytes(uint32_t nchunks) { return ((uint64_t)nchunks * 8 + 255) / 256 * 256; }

// first-item blob layout (16-byte words): [0] Item, [1, kBlobRef0) Task, then refs
constexpr int kBlobRef0 = 1 + (int)((sizeof(Task) + 15) / 16);

}  // namespace adapcc
