// C ABI of the AdapCC B200 hot path (include/adapcc.h).
//
// Communicator = the paper's set of transmission contexts: a
// registered scratch arena per rank (landing + broadcast slots + per-chunk
// flags, the paper's receive/result buffers P:L243), IPC-mapped by every peer
// after one bootstrap all-gather of handles (Fig. 10), plus the
// strategy per collective and a cache of compiled plans.  Every collective
// call is one engine launch per segment on the caller's stream.
#include <cuda.h>  // driver API types only: the functions are resolved with dlopen (NVLS setup)
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <sys/syscall.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <unistd.h>
#include <nvtx3/nvToolsExt.h>  // header-only NVTX ranges: free unless a profiler (nsys) is attached

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <ctime>
#include <list>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include "../../include/adapcc.h"
#include "launch.hpp"
#include "plan.hpp"
#include "strategy.hpp"

using namespace adapcc;

namespace {

constexpr size_t kDefaultScratch = size_t(1) << 30;
constexpr int kPlanCacheCap = 64;
constexpr uint64_t kMaxBlobBytes = uint64_t(64) << 20;  // per segment: larger plans claim dynamically

struct DevSegment {
  Task* tasks = nullptr;
  BufRef* refs = nullptr;
  FlagRef* flags = nullptr;
  Item* items = nullptr;
  uint32_t nitems = 0;
  uint32_t ntasks = 0;
  uint64_t flat_vecs = 0;         // flat kernel: 16-byte vectors of the tasks this rank runs
  uint64_t* late_bits = nullptr;  // per item: late ranks folded in phase 1 (late join)
  uint32_t* late_list = nullptr;  // nitems: items phase 1 left incomplete
  unsigned long long* late_count = nullptr;  // (gen << 32 | count), epoch of the last phase 1 (launch.hpp)
  uint4* first = nullptr;         // LDG kernel: per-CTA first-item blobs (launch.hpp)
  uint32_t nfirst = 0, first_words = 0;
  uint32_t sched_static = 0;      // LDG kernel: every item has a blob, CTA b runs b, b + grid, ...
  uint32_t arena_free = 0;        // no arena streams, flag waits or posts (launch.hpp)
};

struct DevPlan {
  int engine = 0;      // 0: LDG fold kernel, 1: TMA pipeline, 3: flat (one CTA per item)
  int kernel = 0;      // 0: LDG, 1: TMA for DIRECT plans, 2: TMA for STAGED plans, 3: flat
  std::vector<DevSegment> segs;
  bool launched = false;  // enqueued at least once: freeing the tables waits for the device
  uint64_t last_tick = 0;
  bool pinned = false;  // referenced by a captured CUDA graph: never evicted
  bool joined = false;  // a LATE_JOIN call recorded late_bits (phase 2 may follow)
  uint64_t sig = 0;     // hash of the plan key: the call every rank must agree on (debug check)
  ~DevPlan() {
    // eviction is rare (plan-cache capacity), so instead of recording an event
    // on every call the tables are freed after the device drains
    if (launched) cudaDeviceSynchronize();
    for (auto& s : segs) {
      cudaFree(s.tasks);
      cudaFree(s.refs);
      cudaFree(s.flags);
      cudaFree(s.items);
      cudaFree(s.late_bits);
      cudaFree(s.late_list);
      cudaFree(s.late_count);
      cudaFree(s.first);
    }
    cudaGetLastError();  // teardown errors must not leak into a later call's check
  }
};

using PlanKey = std::tuple<int, uint64_t, uint64_t, int, uint64_t, unsigned, int, uint64_t>;  // ..., mode, members

// A buffer registered for zero-copy collectives: base[q] is where rank q's
// registered region starts in THIS process's address space (peer-mapped).
struct RegBuf {
  std::vector<char*> base;
  std::vector<std::string> handle;  // per peer: IPC handle bytes (for close)
  size_t bytes = 0;
};

int esize_of(adapcc_dtype_t d) { return d == ADAPCC_BFLOAT16 ? 2 : 4; }

std::string star(int n, int root) {
  std::string p;
  for (int g = 0; g < n; ++g) p += (g ? "," : "") + std::to_string(g == root ? -1 : root);
  return p;
}

// Defaults; Reduce / Broadcast defaults are generated for the
// call's root: one star tree (all trees of a Reduce share the root).  After a
// fault exclusion (NEXT-3) the AllReduce default keeps only the stars rooted at
// live ranks; excluded ranks are leaves of every star.
std::string default_strategy(Coll c, int n, int root = 0, uint64_t members = ~uint64_t(0), int64_t chunk = 262144) {
  const std::string ck = std::to_string(chunk);
  std::string s = "adapcc-strategy 1\nnranks " + std::to_string(n) + "\ncollective ";
  if (c == kReduce) return s + "reduce\ntree weight=1 chunk=" + ck + " parent=" + star(n, root) + "\n";
  if (c == kBroadcast)
    return s + "broadcast\nbcast src=" + std::to_string(root) + " weight=1 chunk=" + ck + " parent=" + star(n, root) + "\n";
  if (c == kReduceScatter) {
    s += "reducescatter\n";
    for (int b = 0; b < n; ++b)
      s += "rtree dst=" + std::to_string(b) + " weight=1 chunk=" + ck + " parent=" + star(n, b) + "\n";
    return s;
  }
  if (c == kAllReduce) {
    s += "allreduce\n";
    for (int m = 0; m < n; ++m) {  // n star trees, equal weights
      if (!((members >> m) & 1)) continue;
      s += "tree weight=1 chunk=" + ck + " parent=";
      for (int g = 0; g < n; ++g) s += (g ? "," : "") + std::to_string(g == m ? -1 : m);
      s += "\n";
    }
  } else if (c == kAllGather) {
    s += "allgather\n";
    for (int src = 0; src < n; ++src) {
      s += "bcast src=" + std::to_string(src) + " weight=1 chunk=" + ck + " parent=";
      for (int g = 0; g < n; ++g) s += (g ? "," : "") + std::to_string(g == src ? -1 : src);
      s += "\n";
    }
  } else {
    s += "alltoall\na2a weight=1 chunk=1048576\n";
  }
  return s;
}

int64_t env_int(const char* name, int64_t dflt) {
  const char* v = std::getenv(name);
  return v && *v ? std::strtoll(v, nullptr, 10) : dflt;
}

}  // namespace

struct adapcc_comm_s {
  int rank = 0;
  int nranks = 0;
  int device = 0;
  bool loopback = false;
  Mode mode = kStaged;
  uint64_t arena_bytes = 0;  // header + 2 halves
  uint64_t half_bytes = 0;
  char* own_arena = nullptr;               // loopback: all virtual ranks' arenas
  std::vector<char*> arena;                // per rank base (peer-mapped in IPC mode)
  DevState* state = nullptr;              // device epoch + work counters
  int* h_err = nullptr;
  int* d_err = nullptr;
  Strategy strat[kNumColl];
  bool user_set[kNumColl] = {};          // set_strategy was called for this collective
  std::map<int, Strategy> rooted[kNumColl];  // default Reduce/Broadcast strategies per root
  std::map<PlanKey, std::shared_ptr<DevPlan>> plans;
  std::vector<std::shared_ptr<DevPlan>> retired;  // out of the cache, still used by a captured graph
  uint64_t tick = 0;  // plan-cache clock (least recently used plan is evicted)
  int64_t timeout_ms = 10000;
  int64_t max_ctas = 0;
  int64_t drop_rank = -1;
  uint64_t members = 0;   // live ranks (NEXT-3 fault exclusion); all ranks after init
  uint64_t late_seq = 0;  // late-join ticket of the most recent LATE_JOIN call
  int64_t piece_kib = 0;  // 0 = automatic (plan.cpp:order_items)
  int64_t taper = 0;      // tail items cut into this many sub-pieces (1 = off, 0 = auto)
  int64_t check_sig = 0;  // debug: kernels compare call signatures across ranks (ADAPCC_DEBUG)
  int64_t first_blob = 1; // LDG kernel: per-CTA first-item blobs (ADAPCC_FIRST_BLOB=0 disables)
  int64_t tma_shape = 0;  // tuning: 0 = auto, 1 / 2 = force the 1 x 3 x 64 / 2 x 3 x 32 KiB TMA ring (ADAPCC_TMA_SHAPE)
  TraceRec* trace = nullptr;  // in-kernel trace buffer (adapcc_config("trace", capacity))
  unsigned* trace_n = nullptr;
  uint32_t trace_cap = 0;
  int64_t pdl = 1;        // programmatic dependent launch of the engine kernels (ADAPCC_PDL)
  int64_t acc_red = 1;    // TMA kernel: recv += result by bulk reduce-add in L2 (ADAPCC_ACC_RED)
  int64_t default_chunk = 262144;  // C_m of the default strategies (a link profile may set it)
  int64_t sched = 2;      // LDG kernel: 0 dynamic claims, 1 static blob schedule, 2 auto (ADAPCC_SCHED)
  int64_t flat_ctas = 2;  // flat kernel: CTAs per SM of its grid (2 resident; more = several waves) (ADAPCC_FLAT_CTAS)
  uint64_t launches = 0;
  int num_sms = 148;
  // [kernel][dtype] resident CTAs per SM; kernels: 0 LDG fold, 1 TMA (DIRECT
  // plans), 2 TMA (STAGED plans)
  int occ[3][3] = {{1, 1, 1}, {1, 1, 1}, {1, 1, 1}};
  int engine = 2;  // 0: LDG/STG fold, 1: TMA bulk pipeline, 2: auto by call size, 3: flat (flag-free plans)
  int last_engine = -1;  // kernel used by the most recent launch
  std::mutex mu;
  adapcc_bootstrap_allgather_fn ag = nullptr;  // kept for collective registration
  void* ag_ctx = nullptr;
  std::map<int, RegBuf> regs;
  int next_reg = 0;
  std::map<std::pair<int, std::string>, std::pair<char*, int>> opened;  // (peer, handle) -> (base, refs)
  // Readiness board (NEXT-1 online coordinator): kBoardWords host words,
  // mapped into the device; word r = the ticket rank r signalled ready for
  // (adapcc_signal_ready writes it next to the arena word), words 64.. are the
  // coordinator's decision area.  Multi-process: one POSIX shared-memory page
  // per communicator, registered by every rank, so every rank's host sees
  // every rank's readiness without a device round trip.
  uint64_t* h_board = nullptr;
  uint64_t* d_board = nullptr;
  bool board_shm = false;    // shared across the ranks of the node
  bool board_pinned = false; // cudaHostAlloc'ed (else registered mmap)
  // NVLS (NEXT-2): a multicast object over every rank's device, bound to a
  // scratch allocation per rank; nvls_uc / nvls_mc = its unicast / multicast
  // virtual addresses (adapcc_nvls_setup)
  char* nvls_uc = nullptr;
  char* nvls_mc = nullptr;
  uint64_t nvls_bytes = 0;
  unsigned long long nvls_mc_handle = 0, nvls_phys = 0;
  int nvls_fd = -1;
  uint64_t nvls_stride = 0;  // loopback emulation: per-virtual-rank scratch stride (cudaMalloc'ed)
};

namespace {

thread_local cudaError_t g_last_cuda_error = cudaSuccess;
thread_local int g_last_cuda_line = 0;
thread_local char g_last_cuda_msg[160];

adapcc_result_t cuda_fail(cudaError_t e, int line) {
  g_last_cuda_error = e;
  g_last_cuda_line = line;
  return ADAPCC_ERR_CUDA;
}

#define CK(expr)                                   \
  do {                                             \
    cudaError_t _e = (expr);                       \
    if (_e != cudaSuccess) return cuda_fail(_e, __LINE__); \
  } while (0)

adapcc_result_t common_init(adapcc_comm_s* c, size_t scratch) {
  if (scratch == 0) scratch = kDefaultScratch;
  if (scratch < (size_t)kArenaHeader + 2 * (4096 + 65536)) return ADAPCC_ERR_INVALID_ARGUMENT;
  c->half_bytes = ((scratch - kArenaHeader) / 2) / 256 * 256;
  c->arena_bytes = kArenaHeader + 2 * c->half_bytes;
  c->timeout_ms = env_int("ADAPCC_TIMEOUT_MS", 10000);
  c->max_ctas = env_int("ADAPCC_NCTAS", 0);
  c->engine = (int)std::min<int64_t>(3, std::max<int64_t>(0, env_int("ADAPCC_ENGINE", 2)));
  c->flat_ctas = std::min<int64_t>(64, std::max<int64_t>(1, env_int("ADAPCC_FLAT_CTAS", 2)));
  c->piece_kib = env_int("ADAPCC_PIECE_KIB", 0);
  c->taper = std::min<int64_t>(64, std::max<int64_t>(0, env_int("ADAPCC_TAPER", 0)));
  c->check_sig = env_int("ADAPCC_DEBUG", 0) != 0;
  c->first_blob = env_int("ADAPCC_FIRST_BLOB", 1) != 0;
  c->tma_shape = env_int("ADAPCC_TMA_SHAPE", 0);
  c->pdl = env_int("ADAPCC_PDL", 1) != 0;
  c->acc_red = env_int("ADAPCC_ACC_RED", 1) != 0;
  c->sched = std::min<int64_t>(2, std::max<int64_t>(0, env_int("ADAPCC_SCHED", 2)));
  CK(cudaSetDevice(c->device));
  CK(cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, c->device));
  for (int d = 0; d < 3; ++d) {
    CK(engine_occupancy(d, &c->occ[0][d]));
    CK(tma_direct::occupancy(d, &c->occ[1][d]));
    CK(tma_staged::occupancy(d, &c->occ[2][d]));
    for (int k = 0; k < 3; ++k)
      if (c->occ[k][d] < 1) c->occ[k][d] = 1;
  }
  c->members = c->nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << c->nranks) - 1);
  CK(cudaMalloc(&c->state, sizeof(DevState)));
  CK(cudaMemset(c->state, 0, sizeof(DevState)));
  CK(cudaHostAlloc(&c->h_err, sizeof(int), cudaHostAllocMapped));
  *c->h_err = 0;
  CK(cudaHostGetDevicePointer(&c->d_err, c->h_err, 0));
  for (int k = 0; k < kNumColl; ++k) {
    std::string err;
    if (!parse_strategy(default_strategy((Coll)k, c->nranks).c_str(), &c->strat[k], &err))
      return ADAPCC_ERR_INVALID_STRATEGY;
  }
  return ADAPCC_SUCCESS;
}

constexpr size_t kBoardBytes = 4096;

// private board: a mapped pinned page (loopback, or a node without /dev/shm)
adapcc_result_t board_private(adapcc_comm_s* c) {
  void* h = nullptr;
  if (cudaHostAlloc(&h, kBoardBytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) return ADAPCC_ERR_CUDA;
  std::memset(h, 0, kBoardBytes);
  c->h_board = static_cast<uint64_t*>(h);
  c->board_pinned = true;
  CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&c->d_board), h, 0));
  return ADAPCC_SUCCESS;
}

// shared board: rank 0 creates the page, every rank maps and registers it
bool board_shared(adapcc_comm_s* c, const char* name, bool create) {
  const int fd = shm_open(name, O_RDWR | (create ? O_CREAT | O_EXCL : 0), 0600);
  if (fd < 0) return false;
  if (create && ftruncate(fd, kBoardBytes) != 0) { close(fd); return false; }
  void* p = mmap(nullptr, kBoardBytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) return false;
  if (create) std::memset(p, 0, kBoardBytes);
  if (cudaHostRegister(p, kBoardBytes, cudaHostRegisterMapped | cudaHostRegisterPortable) != cudaSuccess ||
      cudaHostGetDevicePointer(reinterpret_cast<void**>(&c->d_board), p, 0) != cudaSuccess) {
    cudaGetLastError();
    munmap(p, kBoardBytes);
    return false;
  }
  c->h_board = static_cast<uint64_t*>(p);
  c->board_shm = true;
  return true;
}

void board_free(adapcc_comm_s* c) {
  if (!c->h_board) return;
  if (c->board_pinned) {
    cudaFreeHost(c->h_board);
  } else {
    cudaHostUnregister(c->h_board);
    munmap(c->h_board, kBoardBytes);
  }
  c->h_board = c->d_board = nullptr;
}

void nvls_release(adapcc_comm_s* c);

void release(adapcc_comm_s* c) {
  if (!c) return;
  cudaSetDevice(c->device);
  cudaDeviceSynchronize();
  board_free(c);
  nvls_release(c);
  c->plans.clear();
  c->retired.clear();
  for (auto& o : c->opened) cudaIpcCloseMemHandle(o.second.first);
  c->opened.clear();
  if (c->loopback) {
    cudaFree(c->own_arena);
  } else {
    for (int r = 0; r < (int)c->arena.size(); ++r) {
      if (r == c->rank) cudaFree(c->arena[r]);
      else if (c->arena[r]) cudaIpcCloseMemHandle(c->arena[r]);
    }
  }
  cudaFree(c->state);
  cudaFree(c->trace);
  cudaFree(c->trace_n);
  cudaFreeHost(c->h_err);
  delete c;
}

// Validate arguments common to every collective.
adapcc_result_t check_common(adapcc_comm_t c, adapcc_dtype_t dtype, uint64_t mask) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (dtype != ADAPCC_FLOAT32 && dtype != ADAPCC_BFLOAT16 && dtype != ADAPCC_INT32)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (c->nranks < 64 && (mask >> c->nranks) != 0) return ADAPCC_ERR_INVALID_ARGUMENT;
  // an excluded rank is never ready and, in multi-process mode, makes no calls
  if ((mask & ~c->members) || (!c->loopback && !((c->members >> c->rank) & 1)))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (*reinterpret_cast<volatile int*>(c->h_err)) return (adapcc_result_t)*c->h_err;
  return ADAPCC_SUCCESS;
}

// FNV-1a over 64-bit words (call signatures of the debug check)
uint64_t fnv(uint64_t h, uint64_t v) {
  for (int i = 0; i < 8; ++i) { h ^= (v >> (8 * i)) & 0xff; h *= 1099511628211ull; }
  return h;
}

bool misaligned(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) != 0; }

// ACCUMULATE, or one of LATE_JOIN / LATE_COMPLEMENT (AllReduce only; on a
// DIRECT plan the root reads a late rank's input, on a STAGED plan the late
// rank pushes it to the root).
adapcc_result_t check_late_flags(adapcc_comm_s* c, unsigned flags, bool late_ok) {
  (void)c;
  const unsigned late = flags & (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT);
  if (flags & ~(ADAPCC_FLAG_ACCUMULATE | ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (late && ((flags & ADAPCC_FLAG_ACCUMULATE) || late == (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT)))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (late && !late_ok) return ADAPCC_ERR_UNSUPPORTED;
  return ADAPCC_SUCCESS;
}

bool overlap(const void* a, size_t an, const void* b, size_t bn) {
  auto x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
  return x < y + bn && y < x + an;
}

// Measured crossover (profiles/sizes_*_r01.json): below ~64 MiB of traffic per
// launch the LDG kernel's lower fixed cost wins, above it the TMA pipeline.
// auto engine: the TMA pipeline from 128 MiB of traffic per launch; below, the
// LDG fold's lower fixed cost wins (profiles/pieces_r01.json: 8 virtual ranks
// x 4 MiB = 64 MiB of traffic, LDG 10.4 us vs TMA 13.4 us)
constexpr uint64_t kTmaMinTraffic = uint64_t(128) << 20;
// ACCUMULATE with bulk reduce-adds: the TMA kernel wins from ~32 MiB of traffic
// (8 virtual ranks, 2 late: 2 MiB per rank 7.8 vs 9.0 us, 8 MiB 18.3 vs 36.2 us;
// 1 MiB 7.1 vs 6.6 us, scripts/debug/acc_small.py): the LDG kernel pays one
// memory latency per accumulating destination
constexpr uint64_t kTmaMinTrafficAcc = uint64_t(32) << 20;

int grid_size(const adapcc_comm_s* c, adapcc_dtype_t dtype, int kernel) {
  int grid = c->num_sms * c->occ[kernel][(int)dtype];
  if (c->max_ctas > 0) grid = (int)std::min<int64_t>(grid, c->max_ctas);
  return std::max(grid, 1);
}

// The strategy a call runs on: the user's, or (Reduce / Broadcast without a
// user strategy) the default rooted at the call's root.  Plans are cached by
// the strategy's hash, so swapping back to a strategy seen before reuses them.
adapcc_result_t pick_strategy(adapcc_comm_s* c, Coll coll, int root, const Strategy** out) {
  if (coll != kReduce && coll != kBroadcast) {
    *out = &c->strat[coll];
    return ADAPCC_SUCCESS;
  }
  if (root < 0 || root >= c->nranks || !((c->members >> root) & 1)) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (c->user_set[coll]) {
    const Strategy& st = c->strat[coll];
    const int sroot = coll == kReduce ? st.subs[0].root : st.subs[0].src;
    if (sroot != root) return ADAPCC_ERR_INVALID_ARGUMENT;
    *out = &st;
    return ADAPCC_SUCCESS;
  }
  auto it = c->rooted[coll].find(root);
  if (it == c->rooted[coll].end()) {
    Strategy st;
    if (!parse_strategy(default_strategy(coll, c->nranks, root, c->members, c->default_chunk).c_str(), &st, nullptr))
      return ADAPCC_ERR_INVALID_STRATEGY;
    it = c->rooted[coll].emplace(root, std::move(st)).first;
  }
  *out = &it->second;
  return ADAPCC_SUCCESS;
}

adapcc_result_t get_plan(adapcc_comm_s* c, Coll coll, const Strategy* strat, uint64_t count,
                         adapcc_dtype_t dtype, uint64_t mask, unsigned flags, Mode mode,
                         std::shared_ptr<DevPlan>* out, const uint64_t* counts = nullptr) {
  // phase 2 of a late join runs on the phase-1 plan (same items, recorded bits)
  if (flags & ADAPCC_FLAG_LATE_COMPLEMENT) flags = ADAPCC_FLAG_LATE_JOIN;
  if (counts) {  // AlltoAllv: the plan depends on the whole count matrix
    uint64_t h = 1469598103934665603ull;
    for (int i = 0; i < c->nranks * c->nranks; ++i) { h ^= counts[i]; h *= 1099511628211ull; }
    count = h;
    coll = (Coll)kNumColl;  // distinct plan-cache namespace
  }
  PlanKey key{(int)coll, strat->hash, count, (int)dtype, mask, flags, (int)mode, c->members};
  auto it = c->plans.find(key);
  if (it != c->plans.end()) {
    it->second->last_tick = ++c->tick;
    *out = it->second;
    return ADAPCC_SUCCESS;
  }
  PlanRequest rq;
  rq.st = strat;
  rq.count = count;
  rq.esize = esize_of(dtype);
  rq.ready_mask = mask;
  rq.accumulate = flags & ADAPCC_FLAG_ACCUMULATE;
  rq.late_join = flags & ADAPCC_FLAG_LATE_JOIN;
  rq.counts = counts;
  rq.members = c->members;
  rq.grid = grid_size(c, dtype, 0);
  rq.mode = mode;
  rq.half_bytes = c->half_bytes;
  rq.nvls_bytes = c->nvls_bytes;
  std::vector<SegmentPlan> segs;
  std::string err;
  if (!build_plan(rq, &segs, &err)) return err.rfind("unsupported", 0) == 0 ? ADAPCC_ERR_UNSUPPORTED : ADAPCC_ERR_OOM;
  auto plan = std::make_shared<DevPlan>();
  {
    uint64_t h = 1469598103934665603ull;
    for (uint64_t v : {(uint64_t)coll, strat->hash, count, (uint64_t)dtype, mask, (uint64_t)flags, (uint64_t)mode,
                       c->members, (uint64_t)segs.size()})
      h = fnv(h, v);
    plan->sig = h;
  }
  {
    PlanStats st;
    for (auto& sp : segs) accumulate_stats(sp, c->loopback ? -1 : c->rank, rq.esize, &st);
    const uint64_t traffic = st.bytes_read + st.bytes_written;
    const uint64_t min_tma = rq.accumulate && c->acc_red ? kTmaMinTrafficAcc : kTmaMinTraffic;
    plan->engine = c->engine != 2 ? c->engine : (traffic / std::max<size_t>(1, segs.size()) >= min_tma ? 1 : 0);
    // ACCUMULATE (phase 2): with bulk reduce-adds (acc_red, default) a stage
    // holds only the sources and DIRECT plans keep the 1 x 3 x 64 KiB ring
    // (profiles/acc_r02.json); the shared-memory read-modify-write (acc_red
    // off) stages nsrc + nacc tiles per slot and is latency-bound, where the
    // 2 CTAs/SM x 3 x 32 KiB shape wins (profiles/acc_variants_r01.json).
    // NVLS (multimem) tasks run on the LDG kernel
    for (auto& sp : segs)
      if (sp.nvls) plan->engine = 0;
    plan->kernel = plan->engine == 0 ? 0 : (mode == kDirect && (!rq.accumulate || c->acc_red) ? 1 : 2);
    if (plan->kernel != 0 && (c->tma_shape == 1 || c->tma_shape == 2)) plan->kernel = (int)c->tma_shape;
    // flat kernel (engine_flat.cu): plans whose items are independent -- no
    // flag waits or posts, no arena streams, no late join, no NVLS
    bool flat_ok = !rq.late_join;
    for (auto& sp : segs) {
      if (sp.nvls) flat_ok = false;
      for (const Task& t : sp.tasks) {
        if (t.nwait || t.npost || t.nlate || (t.op != kOpFold && t.op != kOpZero)) flat_ok = false;
        for (uint32_t k = 0; k < (uint32_t)t.nsrc + t.ndst; ++k)
          if (sp.refs[t.ref0 + k].kind != kBufSend && sp.refs[t.ref0 + k].kind != kBufRecv) flat_ok = false;
      }
    }
    for (auto& sp : segs) {  // the descriptor blob must fit the kernel's shared memory
      uint32_t nt = 0, nr = 0;
      for (const Task& t : sp.tasks)
        if (c->loopback || t.owner == c->rank) {
          ++nt;
          nr += (uint32_t)t.nsrc + t.ndst;
        }
      if (nt > kFlatMaxTasks || nr > kFlatMaxRefs) flat_ok = false;
    }
    // auto: small ACCUMULATE calls (phase 2 of small buckets) take the flat
    // kernel -- the persistent LDG kernel pays one memory round trip per
    // accumulating destination (1 MiB per rank, 2 of 8 ready: 7.2 -> 5.8 us,
    // profiles/flat_r02.json); everything larger stays on the TMA pipeline
    const bool flat_auto = c->engine == 2 && rq.accumulate && plan->engine == 0;
    if (flat_ok && (c->engine == 3 || flat_auto)) plan->engine = plan->kernel = 3;
  }
  for (auto& sp : segs) {
    DevSegment d;
    // (the flat kernel runs tasks, not items: the items only count the work)
    const bool flat = plan->kernel == 3;
    std::vector<Item> items = order_items(sp, c->loopback ? -1 : c->rank, rq.esize, grid_size(c, dtype, flat ? 0 : plan->kernel),
                                          (uint64_t)c->piece_kib * 1024, (int)c->taper, plan->kernel != 0,
                                          plan->kernel == 1 && rq.accumulate && c->acc_red);
    d.nitems = (uint32_t)items.size();
    d.arena_free = 1;
    for (const Task& t : sp.tasks) {
      if (t.nwait || t.npost) d.arena_free = 0;
      for (uint32_t k = 0; k < (uint32_t)t.nsrc + t.ndst + t.nlate; ++k)
        if (sp.refs[t.ref0 + k].kind == kBufArena) d.arena_free = 0;
    }
    auto up = [](auto** dst, const auto& v) -> cudaError_t {
      using T = typename std::decay_t<decltype(v)>::value_type;
      size_t bytes = std::max<size_t>(1, v.size()) * sizeof(T);
      cudaError_t e = cudaMalloc((void**)dst, bytes);
      if (e != cudaSuccess) return e;
      return v.empty() ? cudaSuccess : cudaMemcpy(*dst, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
    };
    CK(up(&d.tasks, sp.tasks));
    CK(up(&d.refs, sp.refs));
    CK(up(&d.flags, sp.flags));
    CK(up(&d.items, items));
    if (flat) {
      // descriptor blob (engine.cuh FlatTask): the tasks this rank runs, then their refs
      std::vector<FlatTask> ft;
      std::vector<BufRef> fr;
      for (const Task& t : sp.tasks) {
        if (!(c->loopback || t.owner == c->rank)) continue;
        FlatTask f{};
        f.len = t.hi - t.lo;
        f.ref0 = (uint32_t)fr.size();
        f.nsrc = t.nsrc;
        f.ndst = t.ndst;
        f.op = t.op;
        f.owner = t.owner;
        for (uint32_t k = 0; k < (uint32_t)t.nsrc + t.ndst; ++k) {
          BufRef r = sp.refs[t.ref0 + k];
          r.bias += (int64_t)(t.lo * rq.esize);
          r.pad[0] = (uint8_t)(ft.size() & 255);
          r.pad[1] = (uint8_t)(ft.size() >> 8);
          if (k >= t.nsrc && r.accum) f.any_acc = 1;
          fr.push_back(r);
        }
        d.flat_vecs += f.len * rq.esize / 16 + 1;
        ft.push_back(f);
      }
      std::vector<uint4> blob(2 * ft.size() + fr.size());
      if (!ft.empty()) std::memcpy(blob.data(), ft.data(), ft.size() * sizeof(FlatTask));
      if (!fr.empty()) std::memcpy(blob.data() + 2 * ft.size(), fr.data(), fr.size() * sizeof(BufRef));
      CK(up(&d.first, blob));
      d.ntasks = (uint32_t)ft.size();
      d.first_words = (uint32_t)blob.size();
    }
    if (c->first_blob && !flat) {
      // Item blobs (launch.hpp): item i, its task and the task's refs in one
      // run of 16-byte words.  Static schedule: every item gets one, CTA b runs
      // items b, b + grid, ... and prefetches the next blob while it folds (no
      // claim atomic and no item -> task -> refs chain per item).  Otherwise
      // only CTA b's first item (items[b]) has one, whatever the grid.
      auto words_of = [&](uint32_t i) {
        const Task& t = sp.tasks[items[i].task];
        return (uint32_t)kBlobRef0 + t.nsrc + t.ndst + t.nlate;
      };
      uint32_t all_words = 0;
      for (uint32_t i = 0; i < d.nitems; ++i) all_words = std::max(all_words, words_of(i));
      // (late-join plans claim dynamically: phase 2 runs phase 1's list of incomplete items)
      const bool stat = plan->kernel == 0 && c->sched != 0 && !rq.late_join && d.nitems > 0 && all_words <= (uint32_t)kFirstMaxWords &&
                        (uint64_t)d.nitems * all_words * 16 <= kMaxBlobBytes;
      const uint32_t nf = stat ? d.nitems : std::min<uint32_t>(d.nitems, (uint32_t)grid_size(c, dtype, plan->kernel));
      uint32_t words = 0;
      for (uint32_t b = 0; b < nf; ++b) words = std::max(words, words_of(b));
      if (nf > 0 && words <= (uint32_t)kFirstMaxWords) {
        std::vector<uint4> blob((size_t)nf * words, uint4{0, 0, 0, 0});
        for (uint32_t b = 0; b < nf; ++b) {
          const Task& t = sp.tasks[items[b].task];
          char* w = reinterpret_cast<char*>(&blob[(size_t)b * words]);
          std::memcpy(w, &items[b], sizeof(Item));
          std::memcpy(w + 16, &t, sizeof(Task));
          std::memcpy(w + 16 * kBlobRef0, &sp.refs[t.ref0], sizeof(BufRef) * (t.nsrc + t.ndst + t.nlate));
        }
        CK(up(&d.first, blob));
        d.nfirst = nf;
        d.first_words = words;
        d.sched_static = stat ? 1 : 0;
      }
    }
    if (rq.late_join) {
      CK(cudaMalloc(&d.late_bits, std::max<size_t>(1, items.size()) * sizeof(uint64_t)));
      CK(cudaMemset(d.late_bits, 0, std::max<size_t>(1, items.size()) * sizeof(uint64_t)));
      CK(cudaMalloc(&d.late_list, std::max<size_t>(1, items.size()) * sizeof(uint32_t)));
      CK(cudaMalloc(&d.late_count, 2 * sizeof(unsigned long long)));
      const unsigned long long init[2] = {0ull, ~0ull};  // empty list, no phase 1 recorded
      CK(cudaMemcpy(d.late_count, init, sizeof(init), cudaMemcpyHostToDevice));
    }
    plan->segs.push_back(d);
  }
  // in loopback an empty call launches nothing; in multi-process mode every
  // rank launches every segment so that epochs stay aligned across ranks
  if (c->plans.size() >= (size_t)kPlanCacheCap) {
    auto victim = c->plans.end();
    for (auto i = c->plans.begin(); i != c->plans.end(); ++i)
      if (!i->second->pinned && (victim == c->plans.end() || i->second->last_tick < victim->second->last_tick))
        victim = i;
    if (victim != c->plans.end()) c->plans.erase(victim);  // DevPlan dtor waits for its last launch
  }
  plan->last_tick = ++c->tick;
  c->plans[key] = plan;
  *out = plan;
  return ADAPCC_SUCCESS;
}

// zc_send / zc_recv (multi-process zero-copy): every rank's buffer as mapped
// in this process -> the DIRECT plan runs across processes over NVLink.
adapcc_result_t run(adapcc_comm_s* c, Coll coll, const void* const* send, void* const* recv,
                    uint64_t count, adapcc_dtype_t dtype, uint64_t mask, unsigned flags,
                    adapcc_stream_t stream, int root = 0, char* const* zc_send = nullptr,
                    char* const* zc_recv = nullptr, const uint64_t* counts = nullptr, uint64_t sig_extra = 0) {
  const bool zc = zc_send != nullptr;
  // tracing: one NVTX range per collective call on the host timeline
  static const char* const kRange[kNumColl + 1] = {"adapcc::allreduce", "adapcc::allgather", "adapcc::alltoall",
                                                   "adapcc::reduce", "adapcc::broadcast", "adapcc::reducescatter",
                                                   "adapcc::alltoallv"};
  nvtxRangePushA(kRange[counts ? kNumColl : (int)coll]);
  struct Pop { ~Pop() { nvtxRangePop(); } } pop;
  std::lock_guard<std::mutex> lock(c->mu);
  int cur_dev = -1;  // (cudaGetDevice reads thread state; cudaSetDevice is only needed on a change)
  if (cudaGetDevice(&cur_dev) != cudaSuccess || cur_dev != c->device) CK(cudaSetDevice(c->device));
  const Strategy* strat = nullptr;
  adapcc_result_t r = pick_strategy(c, coll, root, &strat);
  if (r != ADAPCC_SUCCESS) return r;
  std::shared_ptr<DevPlan> plan;
  r = get_plan(c, coll, strat, count, dtype, mask, flags, zc ? kDirect : c->mode, &plan, counts);
  if (r != ADAPCC_SUCCESS) return r;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  CK(cudaStreamIsCapturing(s, &cap));
  const bool capturing = cap != cudaStreamCaptureStatusNone;
  if (capturing) plan->pinned = true;  // the graph keeps pointing at these tables
  const int late_mode = (flags & ADAPCC_FLAG_LATE_JOIN) ? 1 : (flags & ADAPCC_FLAG_LATE_COMPLEMENT) ? 2 : 0;
  if (late_mode == 2 && !plan->joined) return ADAPCC_ERR_INVALID_ARGUMENT;  // no phase 1 recorded
  if (late_mode == 1) {
    plan->joined = true;
    ++c->late_seq;  // ticket of this phase 1: late ranks signal it (adapcc_signal_ready)
  }
  for (size_t si = 0; si < plan->segs.size(); ++si) {
    const DevSegment& seg = plan->segs[si];
    if (c->loopback && seg.nitems == 0) continue;
    LaunchParams P{};
    P.tasks = seg.tasks;
    P.refs = seg.refs;
    P.flags = seg.flags;
    P.items = seg.items;
    P.nitems = seg.nitems;
    P.ntasks = seg.ntasks;
    P.first = seg.first;
    P.nfirst = seg.nfirst;
    P.first_words = seg.first_words;
    P.sched_static = seg.sched_static;
    P.arena_free = seg.arena_free;
    P.dtype = (int)dtype;
    P.nranks = c->nranks;
    P.my_rank = c->loopback ? -1 : c->rank;
    P.ipc = c->loopback ? 0 : 1;
    P.zc = zc ? 1 : 0;
    P.late_mode = late_mode;
    P.acc_red = c->acc_red ? 1 : 0;
    P.late_ticket = c->late_seq;
    P.late_bits = seg.late_bits;
    // (STAGED phase 2 runs every item: pulls wait for every chunk's decision)
    P.late_list = (zc || c->mode == kDirect) ? seg.late_list : nullptr;
    P.late_count = seg.late_count;
    P.drop_rank = (int)c->drop_rank;
    P.members = c->members;
    P.half_bytes = c->half_bytes;
    P.timeout_ns = (uint64_t)std::max<int64_t>(1, c->timeout_ms) * 1000000ull;
    P.check_sig = !c->loopback && c->check_sig;
    P.sig = fnv(fnv(plan->sig, si), sig_extra);
    P.state = c->state;
    P.err = c->d_err;
    P.nvls_uc = c->nvls_uc;
    P.nvls_mc = c->nvls_mc;
    P.nvls_stride = c->nvls_stride;
    P.trace = c->trace;
    P.trace_n = c->trace_n;
    P.trace_cap = c->trace_cap;
    P.launch_seq = (uint32_t)c->launches;
    for (int q = 0; q < c->nranks; ++q) {
      if (zc) {
        P.send[q] = zc_send[q];
        P.recv[q] = zc_recv[q];
      } else if (c->loopback || q == c->rank) {
        const int i = c->loopback ? q : 0;
        P.send[q] = const_cast<char*>(static_cast<const char*>(send[i]));
        P.recv[q] = static_cast<char*>(recv[i]);
      }
      P.hdr[q] = c->arena[q];
    }
    // phase 2 of a late join accumulates into every destination: without
    // acc_red it takes the ACCUMULATE shape (2 x 3 x 32 KiB) whatever the
    // plan's kernel; item order is grid-independent, so the plan is shared
    const int kernel = (late_mode == 2 && plan->kernel == 1 && !c->acc_red && c->tma_shape != 1) ? 2 : plan->kernel;
    // flat: flat_ctas CTAs per SM, fewer if the call has fewer vectors than the grid has threads
    const int grid = kernel == 3 ? (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)c->num_sms * c->flat_ctas,
                                                                                   (seg.flat_vecs + 255) / 256))
                                 : std::max(1, std::min<int>(grid_size(c, dtype, kernel), (int)std::max<uint32_t>(1, seg.nitems)));
    const bool pdl = c->pdl != 0;
    CK(kernel == 1 ? tma_direct::launch(P, grid, s, pdl)
       : kernel == 2 ? tma_staged::launch(P, grid, s, pdl)
       : kernel == 3 ? flat::launch(P, grid, s, pdl) : engine_launch(P, grid, s, pdl));
    c->last_engine = plan->engine;
    ++c->launches;
  }
  plan->launched = true;
  return ADAPCC_SUCCESS;
}

}  // namespace

extern "C" {

const char* adapcc_strerror(adapcc_result_t r) {
  switch (r) {
    case ADAPCC_SUCCESS: return "success";
    case ADAPCC_ERR_INVALID_ARGUMENT: return "invalid argument";
    case ADAPCC_ERR_INVALID_STRATEGY: return "invalid strategy";
    case ADAPCC_ERR_UNSUPPORTED: return "unsupported";
    case ADAPCC_ERR_CUDA: return "CUDA error";
    case ADAPCC_ERR_BOOTSTRAP: return "bootstrap failed";
    case ADAPCC_ERR_OOM: return "out of memory / scratch too small";
    case ADAPCC_ERR_TIMEOUT: return "watchdog timeout (a peer never posted)";
    case ADAPCC_ERR_MISMATCH: return "mismatched collective call";
  }
  return "unknown error";
}

adapcc_result_t adapcc_init_loopback(adapcc_comm_t* comm, int nranks, int cuda_device,
                                     size_t scratch_bytes, adapcc_mode_t mode) {
  if (!comm || nranks < 1 || nranks > ADAPCC_MAX_RANKS) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (mode != ADAPCC_MODE_DIRECT && mode != ADAPCC_MODE_STAGED) return ADAPCC_ERR_INVALID_ARGUMENT;
  *comm = nullptr;
  auto* c = new adapcc_comm_s();
  c->nranks = nranks;
  c->rank = 0;
  c->device = cuda_device;
  c->loopback = true;
  c->mode = (Mode)mode;
  adapcc_result_t r = common_init(c, scratch_bytes == 0 ? (size_t(64) << 20) : scratch_bytes);
  if (r != ADAPCC_SUCCESS) { release(c); return r; }
  if (cudaMalloc(&c->own_arena, c->arena_bytes * nranks) != cudaSuccess) { release(c); return ADAPCC_ERR_OOM; }
  if (cudaMemset(c->own_arena, 0, c->arena_bytes * nranks) != cudaSuccess ||
      cudaDeviceSynchronize() != cudaSuccess) { release(c); return ADAPCC_ERR_CUDA; }
  for (int q = 0; q < nranks; ++q) c->arena.push_back(c->own_arena + q * c->arena_bytes);
  if ((r = board_private(c)) != ADAPCC_SUCCESS) { release(c); return r; }
  *comm = c;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_init(adapcc_comm_t* comm, int rank, int nranks, int cuda_device,
                            size_t scratch_bytes, adapcc_bootstrap_allgather_fn ag, void* ag_ctx) {
  if (!comm || !ag || nranks < 1 || nranks > ADAPCC_MAX_RANKS || rank < 0 || rank >= nranks)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  *comm = nullptr;
  auto* c = new adapcc_comm_s();
  c->nranks = nranks;
  c->rank = rank;
  c->device = cuda_device;
  c->loopback = false;
  c->mode = kStaged;
  c->ag = ag;
  c->ag_ctx = ag_ctx;
  adapcc_result_t r = common_init(c, scratch_bytes);
  if (r != ADAPCC_SUCCESS) { release(c); return r; }
  c->arena.assign(nranks, nullptr);
  char* mine = nullptr;
  if (cudaMalloc(&mine, c->arena_bytes) != cudaSuccess) { release(c); return ADAPCC_ERR_OOM; }
  c->arena[rank] = mine;
  if (cudaMemset(mine, 0, c->arena_bytes) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
    release(c);
    return ADAPCC_ERR_CUDA;
  }
  // handle exchange: the paper's set-up AllGather of IPC handles;
  // rank 0 also names (and creates) the node's readiness board
  struct Blob { cudaIpcMemHandle_t h; uint64_t arena_bytes; int32_t nranks, rank; char board[48]; };
  Blob me{};
  if (cudaIpcGetMemHandle(&me.h, mine) != cudaSuccess) { release(c); return ADAPCC_ERR_CUDA; }
  me.arena_bytes = c->arena_bytes;
  me.nranks = nranks;
  me.rank = rank;
  if (rank == 0) {
    const auto t = std::chrono::steady_clock::now().time_since_epoch().count();
    std::snprintf(me.board, sizeof(me.board), "/adapcc-%d-%llx", (int)getpid(), (unsigned long long)t);
    if (!board_shared(c, me.board, true)) me.board[0] = 0;  // no shared memory: private boards
  }
  std::vector<Blob> all(nranks);
  if (ag(&me, all.data(), sizeof(Blob), ag_ctx) != 0) { release(c); return ADAPCC_ERR_BOOTSTRAP; }
  for (int q = 0; q < nranks; ++q) {
    if (all[q].nranks != nranks || all[q].rank != q || all[q].arena_bytes != c->arena_bytes) {
      release(c);
      return ADAPCC_ERR_MISMATCH;
    }
  }
  for (int q = 0; q < nranks; ++q) {
    if (q == rank) continue;
    void* p = nullptr;
    if (cudaIpcOpenMemHandle(&p, all[q].h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      release(c);
      return ADAPCC_ERR_CUDA;
    }
    c->arena[q] = static_cast<char*>(p);
  }
  if (rank != 0 && all[0].board[0]) board_shared(c, all[0].board, false);
  if (!c->h_board && (r = board_private(c)) != ADAPCC_SUCCESS) { release(c); return r; }
  // second exchange doubles as a barrier: every peer has mapped every arena
  // (and the board); the board's name can then go (the mappings stay)
  int ok = c->board_shm ? 1 : 0;
  std::vector<int> oks(nranks);
  if (ag(&ok, oks.data(), sizeof(int), ag_ctx) != 0) { release(c); return ADAPCC_ERR_BOOTSTRAP; }
  if (rank == 0 && all[0].board[0]) shm_unlink(all[0].board);
  for (int q = 0; q < nranks; ++q)
    if (!oks[q] && c->board_shm) {  // someone could not map it: everybody uses a private board
      board_free(c);
      c->board_shm = false;
      if ((r = board_private(c)) != ADAPCC_SUCCESS) { release(c); return r; }
      break;
    }
  *comm = c;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_set_strategy(adapcc_comm_t c, adapcc_coll_t coll, const char* text,
                                    adapcc_stream_t stream) {
  (void)stream;
  if (!c || coll < ADAPCC_ALLREDUCE || coll > ADAPCC_REDUCESCATTER) return ADAPCC_ERR_INVALID_ARGUMENT;
  Strategy st;
  std::string err;
  if (!parse_strategy(text, &st, &err)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (st.nranks != c->nranks || (int)st.coll != (int)coll) return ADAPCC_ERR_INVALID_STRATEGY;
  std::lock_guard<std::mutex> lock(c->mu);
  if (!check_members(st, c->members, &err)) return ADAPCC_ERR_INVALID_STRATEGY;
  c->strat[coll] = std::move(st);
  c->user_set[coll] = true;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_allreduce(adapcc_comm_t c, const void* sendbuf, void* recvbuf, size_t count,
                                 adapcc_dtype_t dtype, uint64_t mask, unsigned flags,
                                 adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback) return ADAPCC_ERR_INVALID_ARGUMENT;
  r = check_late_flags(c, flags, true);
  if (r != ADAPCC_SUCCESS) return r;
  const size_t bytes = count * esize_of(dtype);
  if (count && !recvbuf) return ADAPCC_ERR_INVALID_ARGUMENT;
  // late join: a non-ready rank's input is pushed once it signals ready
  const bool late = flags & (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT);
  const bool ready = ((mask >> c->rank) & 1) || late;
  if (count && ready && !sendbuf) return ADAPCC_ERR_INVALID_ARGUMENT;
  // a late rank's input is read after phase 1 wrote its recvbuf: no aliasing
  if (late && !((mask >> c->rank) & 1) && count && overlap(sendbuf, bytes, recvbuf, bytes))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (misaligned(recvbuf) || (ready && misaligned(sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && sendbuf != recvbuf && overlap(sendbuf, bytes, recvbuf, bytes)) return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : recvbuf};
  void* d[1] = {recvbuf};
  return run(c, kAllReduce, s, d, count, dtype, mask, flags, stream);
}

adapcc_result_t adapcc_allgather(adapcc_comm_t c, const void* sendbuf, void* recvbuf,
                                 size_t sendcount, adapcc_dtype_t dtype, uint64_t mask,
                                 adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t es = esize_of(dtype), bytes = sendcount * es;
  const bool ready = (mask >> c->rank) & 1;
  if (sendcount && (!recvbuf || (ready && !sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (misaligned(recvbuf) || (ready && misaligned(sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && overlap(sendbuf, bytes, recvbuf, bytes * c->nranks) &&
      sendbuf != static_cast<char*>(recvbuf) + c->rank * bytes)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : recvbuf};
  void* d[1] = {recvbuf};
  return run(c, kAllGather, s, d, sendcount, dtype, mask, 0, stream);
}

adapcc_result_t adapcc_alltoall(adapcc_comm_t c, const void* sendbuf, void* recvbuf,
                                size_t count_per_peer, adapcc_dtype_t dtype, uint64_t mask,
                                adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t bytes = count_per_peer * esize_of(dtype) * c->nranks;
  const bool ready = (mask >> c->rank) & 1;
  if (count_per_peer && (!recvbuf || (ready && !sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (misaligned(recvbuf) || (ready && misaligned(sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && bytes && overlap(sendbuf, bytes, recvbuf, bytes)) return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : recvbuf};
  void* d[1] = {recvbuf};
  return run(c, kAllToAll, s, d, count_per_peer, dtype, mask, 0, stream);
}

static adapcc_result_t check_lb(adapcc_comm_t c, const void* const* s, void* const* d, size_t sbytes,
                                size_t rbytes, uint64_t mask, int kind) {
  if (!c->loopback || !s || !d) return ADAPCC_ERR_INVALID_ARGUMENT;
  for (int q = 0; q < c->nranks; ++q) {
    if (!((c->members >> q) & 1)) continue;  // excluded: buffers never touched
    const bool ready = (mask >> q) & 1;
    if (rbytes && !d[q]) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (misaligned(d[q])) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (!ready) continue;
    if (sbytes && !s[q]) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (misaligned(s[q])) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (!sbytes) continue;
    const bool in_place_ok = (kind == 0 && s[q] == d[q]) ||
                             (kind == 1 && s[q] == static_cast<const char*>(d[q]) + q * sbytes) ||
                             (kind == 3 && d[q] == static_cast<const char*>(s[q]) + q * rbytes);
    if (!in_place_ok && overlap(s[q], sbytes, d[q], rbytes)) return ADAPCC_ERR_INVALID_ARGUMENT;
  }
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_allreduce_lb(adapcc_comm_t c, const void* const* sendbufs,
                                    void* const* recvbufs, size_t count, adapcc_dtype_t dtype,
                                    uint64_t mask, unsigned flags, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  r = check_late_flags(c, flags, true);
  if (r != ADAPCC_SUCCESS) return r;
  const size_t bytes = count * esize_of(dtype);
  // late join reads the non-ready ranks' inputs too: check every sendbuf
  const uint64_t all = c->nranks >= 64 ? ~0ull : ((1ull << c->nranks) - 1);
  const bool late = flags & (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT);
  r = check_lb(c, sendbufs, recvbufs, bytes, bytes, late ? all : mask, 0);
  if (r != ADAPCC_SUCCESS) return r;
  // a late rank's input is read after phase 1 wrote its recvbuf (phase 2):
  // it may not alias it
  if (late)
    for (int q = 0; q < c->nranks; ++q)
      if (((c->members >> q) & 1) && !((mask >> q) & 1) && bytes && overlap(sendbufs[q], bytes, recvbufs[q], bytes))
        return ADAPCC_ERR_INVALID_ARGUMENT;
  return run(c, kAllReduce, sendbufs, recvbufs, count, dtype, mask, flags, stream);
}

adapcc_result_t adapcc_allgather_lb(adapcc_comm_t c, const void* const* sendbufs,
                                    void* const* recvbufs, size_t sendcount, adapcc_dtype_t dtype,
                                    uint64_t mask, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  const size_t bytes = sendcount * esize_of(dtype);
  r = check_lb(c, sendbufs, recvbufs, bytes, bytes * c->nranks, mask, 1);
  if (r != ADAPCC_SUCCESS) return r;
  return run(c, kAllGather, sendbufs, recvbufs, sendcount, dtype, mask, 0, stream);
}

adapcc_result_t adapcc_alltoall_lb(adapcc_comm_t c, const void* const* sendbufs,
                                   void* const* recvbufs, size_t count_per_peer,
                                   adapcc_dtype_t dtype, uint64_t mask, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  const size_t bytes = count_per_peer * esize_of(dtype) * c->nranks;
  r = check_lb(c, sendbufs, recvbufs, bytes, bytes, mask, 2);
  if (r != ADAPCC_SUCCESS) return r;
  return run(c, kAllToAll, sendbufs, recvbufs, count_per_peer, dtype, mask, 0, stream);
}

// ------------------------------------------------ NEXT-4: Reduce / Broadcast / ReduceScatter
adapcc_result_t adapcc_reduce(adapcc_comm_t c, const void* sendbuf, void* recvbuf, size_t count,
                              adapcc_dtype_t dtype, int root, uint64_t mask, unsigned flags,
                              adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback || (flags & ~ADAPCC_FLAG_ACCUMULATE) || root < 0 || root >= c->nranks)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t bytes = count * esize_of(dtype);
  const bool ready = (mask >> c->rank) & 1, is_root = c->rank == root;
  if (count && ((ready && !sendbuf) || (is_root && !recvbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if ((ready && misaligned(sendbuf)) || (is_root && misaligned(recvbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && is_root && sendbuf != recvbuf && overlap(sendbuf, bytes, recvbuf, bytes))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : nullptr};
  void* d[1] = {recvbuf};
  return run(c, kReduce, s, d, count, dtype, mask, flags, stream, root);
}

adapcc_result_t adapcc_broadcast(adapcc_comm_t c, const void* sendbuf, void* recvbuf, size_t count,
                                 adapcc_dtype_t dtype, int root, uint64_t mask, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback || root < 0 || root >= c->nranks) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t bytes = count * esize_of(dtype);
  const bool src = c->rank == root && ((mask >> root) & 1);
  if (count && (!recvbuf || (src && !sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (misaligned(recvbuf) || (src && misaligned(sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (src && sendbuf != recvbuf && overlap(sendbuf, bytes, recvbuf, bytes)) return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {src ? sendbuf : nullptr};
  void* d[1] = {recvbuf};
  return run(c, kBroadcast, s, d, count, dtype, mask, 0, stream, root);
}

adapcc_result_t adapcc_reducescatter(adapcc_comm_t c, const void* sendbuf, void* recvbuf,
                                     size_t recvcount, adapcc_dtype_t dtype, uint64_t mask,
                                     unsigned flags, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback || (flags & ~ADAPCC_FLAG_ACCUMULATE)) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t rbytes = recvcount * esize_of(dtype);
  const bool ready = (mask >> c->rank) & 1;
  if (recvcount && (!recvbuf || (ready && !sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (misaligned(recvbuf) || (ready && misaligned(sendbuf))) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && overlap(sendbuf, rbytes * c->nranks, recvbuf, rbytes) &&
      recvbuf != static_cast<const char*>(sendbuf) + c->rank * rbytes)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : nullptr};
  void* d[1] = {recvbuf};
  return run(c, kReduceScatter, s, d, recvcount, dtype, mask, flags, stream);
}

adapcc_result_t adapcc_reduce_lb(adapcc_comm_t c, const void* const* sendbufs, void* const* recvbufs,
                                 size_t count, adapcc_dtype_t dtype, int root, uint64_t mask,
                                 unsigned flags, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (!c->loopback || !sendbufs || !recvbufs || (flags & ~ADAPCC_FLAG_ACCUMULATE) || root < 0 ||
      root >= c->nranks)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t bytes = count * esize_of(dtype);
  for (int q = 0; q < c->nranks; ++q) {
    if (((mask >> q) & 1) && ((count && !sendbufs[q]) || misaligned(sendbufs[q]))) return ADAPCC_ERR_INVALID_ARGUMENT;
  }
  if ((count && !recvbufs[root]) || misaligned(recvbufs[root])) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (((mask >> root) & 1) && sendbufs[root] != recvbufs[root] &&
      overlap(sendbufs[root], bytes, recvbufs[root], bytes))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  return run(c, kReduce, sendbufs, recvbufs, count, dtype, mask, flags, stream, root);
}

adapcc_result_t adapcc_broadcast_lb(adapcc_comm_t c, const void* const* sendbufs, void* const* recvbufs,
                                    size_t count, adapcc_dtype_t dtype, int root, uint64_t mask,
                                    adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (!c->loopback || !sendbufs || !recvbufs || root < 0 || root >= c->nranks) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t bytes = count * esize_of(dtype);
  for (int q = 0; q < c->nranks; ++q)
    if (((c->members >> q) & 1) && ((count && !recvbufs[q]) || misaligned(recvbufs[q])))
      return ADAPCC_ERR_INVALID_ARGUMENT;
  if ((mask >> root) & 1) {
    if ((count && !sendbufs[root]) || misaligned(sendbufs[root])) return ADAPCC_ERR_INVALID_ARGUMENT;
    for (int q = 0; q < c->nranks; ++q)
      if (((c->members >> q) & 1) && !(q == root && sendbufs[root] == recvbufs[q]) &&
          overlap(sendbufs[root], bytes, recvbufs[q], bytes))
        return ADAPCC_ERR_INVALID_ARGUMENT;
  }
  return run(c, kBroadcast, sendbufs, recvbufs, count, dtype, mask, 0, stream, root);
}

adapcc_result_t adapcc_reducescatter_lb(adapcc_comm_t c, const void* const* sendbufs,
                                        void* const* recvbufs, size_t recvcount, adapcc_dtype_t dtype,
                                        uint64_t mask, unsigned flags, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (flags & ~ADAPCC_FLAG_ACCUMULATE) return ADAPCC_ERR_INVALID_ARGUMENT;
  const size_t rbytes = recvcount * esize_of(dtype);
  r = check_lb(c, sendbufs, recvbufs, rbytes * c->nranks, rbytes, mask, 3);
  if (r != ADAPCC_SUCCESS) return r;
  return run(c, kReduceScatter, sendbufs, recvbufs, recvcount, dtype, mask, flags, stream);
}

// ------------------------------------------------------- zero-copy registration
namespace {
// All-gather over the live ranks (the bootstrap callback covers exactly them:
// the original group, or the survivors' group handed to adapcc_exclude);
// entry q of `out` is rank q's blob, zero for excluded ranks.
int members_allgather(adapcc_comm_s* c, const void* mine, void* out, size_t bytes) {
  const int k = __builtin_popcountll(c->members);
  std::vector<char> tmp((size_t)k * bytes);
  if (c->ag(mine, tmp.data(), bytes, c->ag_ctx) != 0) return 1;
  char* o = static_cast<char*>(out);
  std::memset(o, 0, (size_t)c->nranks * bytes);
  for (int q = 0, i = 0; q < c->nranks; ++q)
    if ((c->members >> q) & 1) std::memcpy(o + (size_t)q * bytes, tmp.data() + (size_t)(i++) * bytes, bytes);
  return 0;
}

// base address of the allocation containing p (driver API, loaded lazily so
// the library still loads on machines without a driver)
bool allocation_base(void* p, char** base) {
  using Fn = int (*)(unsigned long long*, size_t*, unsigned long long);
  static Fn fn = [] {
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
    return h ? reinterpret_cast<Fn>(dlsym(h, "cuMemGetAddressRange_v2")) : nullptr;
  }();
  if (!fn) return false;
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, reinterpret_cast<unsigned long long>(p)) != 0) return false;
  *base = reinterpret_cast<char*>(b);
  return true;
}
}  // namespace

adapcc_result_t adapcc_register_buffer(adapcc_comm_t c, void* ptr, size_t bytes, int* reg_id) {
  if (!c || !ptr || !reg_id || misaligned(ptr)) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (c->loopback || !c->ag) return ADAPCC_ERR_UNSUPPORTED;
  std::lock_guard<std::mutex> lock(c->mu);
  CK(cudaSetDevice(c->device));
  char* base = nullptr;
  if (!allocation_base(ptr, &base)) return ADAPCC_ERR_CUDA;
  struct Blob { cudaIpcMemHandle_t h; uint64_t offset, bytes; int32_t id, pad; };
  Blob me{};
  CK(cudaIpcGetMemHandle(&me.h, base));
  me.offset = static_cast<char*>(ptr) - base;
  me.bytes = bytes;
  me.id = c->next_reg;
  std::vector<Blob> all(c->nranks);
  if (members_allgather(c, &me, all.data(), sizeof(Blob)) != 0) return ADAPCC_ERR_BOOTSTRAP;
  for (int q = 0; q < c->nranks; ++q)
    if (((c->members >> q) & 1) && (all[q].bytes != bytes || all[q].id != me.id)) return ADAPCC_ERR_MISMATCH;
  RegBuf rb;
  rb.bytes = bytes;
  rb.base.assign(c->nranks, nullptr);
  rb.handle.assign(c->nranks, std::string());
  for (int q = 0; q < c->nranks; ++q) {
    if (q == c->rank) {
      rb.base[q] = static_cast<char*>(ptr);
      continue;
    }
    if (!((c->members >> q) & 1)) continue;  // excluded peer: never addressed
    std::string key(reinterpret_cast<const char*>(&all[q].h), sizeof(cudaIpcMemHandle_t));
    auto it = c->opened.find({q, key});
    if (it == c->opened.end()) {
      void* m = nullptr;
      CK(cudaIpcOpenMemHandle(&m, all[q].h, cudaIpcMemLazyEnablePeerAccess));
      it = c->opened.emplace(std::make_pair(q, key), std::make_pair(static_cast<char*>(m), 0)).first;
    }
    it->second.second += 1;
    rb.base[q] = it->second.first + all[q].offset;
    rb.handle[q] = key;
  }
  *reg_id = c->next_reg++;
  c->regs[*reg_id] = std::move(rb);
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_deregister_buffer(adapcc_comm_t c, int reg_id) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  auto it = c->regs.find(reg_id);
  if (it == c->regs.end()) return ADAPCC_ERR_INVALID_ARGUMENT;
  CK(cudaSetDevice(c->device));
  CK(cudaDeviceSynchronize());  // no launch may still reference the mapping
  for (int q = 0; q < c->nranks; ++q) {
    if (q == c->rank) continue;
    auto o = c->opened.find({q, it->second.handle[q]});
    if (o != c->opened.end() && --o->second.second == 0) {
      cudaIpcCloseMemHandle(o->second.first);
      c->opened.erase(o);
    }
  }
  c->regs.erase(it);
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_collective_zc(adapcc_comm_t c, adapcc_coll_t coll, int send_reg,
                                     size_t send_offset, int recv_reg, size_t recv_offset, size_t count,
                                     adapcc_dtype_t dtype, int root, uint64_t mask, unsigned flags,
                                     adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback || coll < ADAPCC_ALLREDUCE || coll > ADAPCC_REDUCESCATTER)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  r = check_late_flags(c, flags, coll == ADAPCC_ALLREDUCE);
  if (r != ADAPCC_SUCCESS) return r;
  if ((flags & ADAPCC_FLAG_ACCUMULATE) && coll != ADAPCC_ALLREDUCE && coll != ADAPCC_REDUCE &&
      coll != ADAPCC_REDUCESCATTER)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  std::vector<char*> S, D;
  {
    std::lock_guard<std::mutex> lock(c->mu);
    auto si = c->regs.find(send_reg), di = c->regs.find(recv_reg);
    if (si == c->regs.end() || di == c->regs.end()) return ADAPCC_ERR_INVALID_ARGUMENT;
    const size_t es = esize_of(dtype), n = c->nranks;
    size_t sb = count * es, rb = count * es;
    if (coll == ADAPCC_ALLGATHER) rb *= n;
    if (coll == ADAPCC_ALLTOALL) { sb *= n; rb *= n; }
    if (coll == ADAPCC_REDUCESCATTER) sb *= n;
    if (send_offset + sb > si->second.bytes || recv_offset + rb > di->second.bytes ||
        (send_offset & 15) || (recv_offset & 15))
      return ADAPCC_ERR_INVALID_ARGUMENT;
    for (size_t q = 0; q < n; ++q) {
      S.push_back(si->second.base[q] + send_offset);
      D.push_back(di->second.base[q] + recv_offset);
    }
    if (coll == ADAPCC_ALLTOALL && overlap(S[c->rank], sb, D[c->rank], rb)) return ADAPCC_ERR_INVALID_ARGUMENT;
    // late join: a late rank's input is read after phase 1 wrote its recvbuf (same offsets on every rank)
    if ((flags & (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT)) && (mask != c->members) &&
        overlap(S[c->rank], sb, D[c->rank], rb))
      return ADAPCC_ERR_INVALID_ARGUMENT;
  }
  uint64_t extra = 1469598103934665603ull;
  for (uint64_t v : {(uint64_t)send_reg, (uint64_t)send_offset, (uint64_t)recv_reg, (uint64_t)recv_offset})
    extra = fnv(extra, v);
  return run(c, (Coll)coll, nullptr, nullptr, count, dtype, mask, flags, stream, root, S.data(), D.data(), nullptr,
             extra);
}

// ---------------------------------------------------------- AlltoAllv (NEXT-4)
static adapcc_result_t a2av_sizes(adapcc_comm_t c, const uint64_t* counts, int rank, size_t es,
                                  size_t* sbytes, size_t* rbytes) {
  if (!counts) return ADAPCC_ERR_INVALID_ARGUMENT;
  uint64_t s = 0, r = 0;
  for (int j = 0; j < c->nranks; ++j) {
    s += counts[(size_t)rank * c->nranks + j];
    r += counts[(size_t)j * c->nranks + rank];
  }
  *sbytes = s * es;
  *rbytes = r * es;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_alltoallv(adapcc_comm_t c, const void* sendbuf, void* recvbuf, const uint64_t* counts,
                                 adapcc_dtype_t dtype, uint64_t mask, adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (c->loopback) return ADAPCC_ERR_INVALID_ARGUMENT;
  size_t sb, rb;
  r = a2av_sizes(c, counts, c->rank, esize_of(dtype), &sb, &rb);
  if (r != ADAPCC_SUCCESS) return r;
  const bool ready = (mask >> c->rank) & 1;
  if ((rb && !recvbuf) || (ready && sb && !sendbuf) || misaligned(recvbuf) || (ready && misaligned(sendbuf)))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ready && sb && rb && overlap(sendbuf, sb, recvbuf, rb)) return ADAPCC_ERR_INVALID_ARGUMENT;
  const void* s[1] = {ready ? sendbuf : nullptr};
  void* d[1] = {recvbuf};
  return run(c, kAllToAll, s, d, 0, dtype, mask, 0, stream, 0, nullptr, nullptr, counts);
}

adapcc_result_t adapcc_alltoallv_lb(adapcc_comm_t c, const void* const* sendbufs, void* const* recvbufs,
                                    const uint64_t* counts, adapcc_dtype_t dtype, uint64_t mask,
                                    adapcc_stream_t stream) {
  adapcc_result_t r = check_common(c, dtype, mask);
  if (r != ADAPCC_SUCCESS) return r;
  if (!c->loopback || !sendbufs || !recvbufs) return ADAPCC_ERR_INVALID_ARGUMENT;
  for (int q = 0; q < c->nranks; ++q) {
    size_t sb, rb;
    r = a2av_sizes(c, counts, q, esize_of(dtype), &sb, &rb);
    if (r != ADAPCC_SUCCESS) return r;
    const bool ready = (mask >> q) & 1;
    if (!((c->members >> q) & 1)) continue;
    if ((rb && !recvbufs[q]) || misaligned(recvbufs[q])) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (ready && ((sb && !sendbufs[q]) || misaligned(sendbufs[q]))) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (ready && sb && rb && overlap(sendbufs[q], sb, recvbufs[q], rb)) return ADAPCC_ERR_INVALID_ARGUMENT;
  }
  return run(c, kAllToAll, sendbufs, recvbufs, 0, dtype, mask, 0, stream, 0, nullptr, nullptr, counts);
}

// ------------------------------------------------------------ NVLS (NEXT-2)
}  // extern "C"
namespace {
// driver entry points for the multicast set-up, resolved at run time (the
// library must load on machines without a driver)
struct Drv {
  CUresult (*DeviceGet)(CUdevice*, int);
  CUresult (*DeviceGetAttribute)(int*, CUdevice_attribute, CUdevice);
  CUresult (*MulticastCreate)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*);
  CUresult (*MulticastGetGranularity)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags);
  CUresult (*MulticastAddDevice)(CUmemGenericAllocationHandle, CUdevice);
  CUresult (*MulticastBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                               unsigned long long);
  CUresult (*MulticastUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
  CUresult (*MemCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long);
  CUresult (*MemRelease)(CUmemGenericAllocationHandle);
  CUresult (*MemAddressReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
  CUresult (*MemAddressFree)(CUdeviceptr, size_t);
  CUresult (*MemMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
  CUresult (*MemUnmap)(CUdeviceptr, size_t);
  CUresult (*MemSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
  CUresult (*MemExportToShareableHandle)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType,
                                         unsigned long long);
  CUresult (*MemImportFromShareableHandle)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType);
  bool ok = false;
};

const Drv& drv() {
  static Drv d = [] {
    Drv x{};
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
    if (!h) return x;
    bool all = true;
    auto get = [&](auto& fn, const char* name) {
      fn = reinterpret_cast<std::remove_reference_t<decltype(fn)>>(dlsym(h, name));
      all = all && fn != nullptr;
    };
    get(x.DeviceGet, "cuDeviceGet");
    get(x.DeviceGetAttribute, "cuDeviceGetAttribute");
    get(x.MulticastCreate, "cuMulticastCreate");
    get(x.MulticastGetGranularity, "cuMulticastGetGranularity");
    get(x.MulticastAddDevice, "cuMulticastAddDevice");
    get(x.MulticastBindMem, "cuMulticastBindMem");
    get(x.MulticastUnbind, "cuMulticastUnbind");
    get(x.MemCreate, "cuMemCreate");
    get(x.MemRelease, "cuMemRelease");
    get(x.MemAddressReserve, "cuMemAddressReserve");
    get(x.MemAddressFree, "cuMemAddressFree");
    get(x.MemMap, "cuMemMap");
    get(x.MemUnmap, "cuMemUnmap");
    get(x.MemSetAccess, "cuMemSetAccess");
    get(x.MemExportToShareableHandle, "cuMemExportToShareableHandle");
    get(x.MemImportFromShareableHandle, "cuMemImportFromShareableHandle");
    x.ok = all;
    return x;
  }();
  return d;
}

void nvls_free(adapcc_comm_s* c) {
  if (c->nvls_stride) {  // loopback emulation
    cudaDeviceSynchronize();
    cudaFree(c->nvls_uc);
    c->nvls_uc = c->nvls_mc = nullptr;
    c->nvls_bytes = c->nvls_stride = 0;
    return;
  }
  const Drv& d = drv();
  if (!d.ok) return;
  cudaDeviceSynchronize();
  CUdevice dev;
  d.DeviceGet(&dev, c->device);
  if (c->nvls_mc) {
    d.MemUnmap((CUdeviceptr)c->nvls_mc, c->nvls_bytes);
    d.MemAddressFree((CUdeviceptr)c->nvls_mc, c->nvls_bytes);
  }
  if (c->nvls_uc) {
    d.MemUnmap((CUdeviceptr)c->nvls_uc, c->nvls_bytes);
    d.MemAddressFree((CUdeviceptr)c->nvls_uc, c->nvls_bytes);
  }
  if (c->nvls_mc_handle && c->nvls_phys) d.MulticastUnbind(c->nvls_mc_handle, dev, 0, c->nvls_bytes);
  if (c->nvls_phys) d.MemRelease(c->nvls_phys);
  if (c->nvls_mc_handle) d.MemRelease(c->nvls_mc_handle);
  if (c->nvls_fd >= 0) close(c->nvls_fd);
  c->nvls_uc = c->nvls_mc = nullptr;
  c->nvls_mc_handle = c->nvls_phys = 0;
  c->nvls_bytes = 0;
  c->nvls_fd = -1;
}

void nvls_release(adapcc_comm_s* c) {
  if (c->nvls_bytes || c->nvls_mc_handle || c->nvls_phys || c->nvls_stride) nvls_free(c);
}

// plans depend on whether NVLS scratch exists (nvls lines plan against it)
void drop_plans_nvls(adapcc_comm_s* c) {
  for (auto& kv : c->plans)
    if (kv.second->pinned) c->retired.push_back(kv.second);
  c->plans.clear();
}
}  // namespace
extern "C" {

adapcc_result_t adapcc_nvls_setup(adapcc_comm_t c, size_t bytes, char* why, size_t why_len) {
  auto say = [&](const char* m) {
    if (why && why_len) {
      std::strncpy(why, m, why_len - 1);
      why[why_len - 1] = 0;
    }
  };
  if (!c || !bytes) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (c->loopback) {  // one device: no multicast team -- emulate the switch (plan + engine test bed)
    std::lock_guard<std::mutex> lock(c->mu);
    CK(cudaSetDevice(c->device));
    if (c->nvls_bytes) nvls_free(c);
    const uint64_t size = (bytes + (uint64_t(2) << 20) - 1) / (uint64_t(2) << 20) * (uint64_t(2) << 20);
    char* p = nullptr;
    if (cudaMalloc(&p, size * c->nranks) != cudaSuccess) { cudaGetLastError(); return ADAPCC_ERR_OOM; }
    c->nvls_uc = c->nvls_mc = p;
    c->nvls_stride = c->nvls_bytes = size;
    drop_plans_nvls(c);
    say("loopback emulation: per-virtual-rank scratch, the kernel sums the copies in ascending rank order");
    return ADAPCC_SUCCESS;
  }
  const uint64_t all = c->nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << c->nranks) - 1);
  if (c->members != all) { say("a rank was excluded: the multicast team is incomplete"); return ADAPCC_ERR_UNSUPPORTED; }
  std::lock_guard<std::mutex> lock(c->mu);
  CK(cudaSetDevice(c->device));
  CK(cudaDeviceSynchronize());
  if (c->nvls_bytes) nvls_free(c);
  const Drv& d = drv();
  std::string reason;
  // every step ends with an all-gather of success flags, so that all ranks
  // either finish the set-up or give up together
  auto agree = [&](bool ok, const char* what) -> adapcc_result_t {
    int mine = ok ? 1 : 0;
    std::vector<int> v(c->nranks);
    if (members_allgather(c, &mine, v.data(), sizeof(int)) != 0) return ADAPCC_ERR_BOOTSTRAP;
    for (int x : v)
      if (!x) {
        if (reason.empty()) reason = ok ? std::string("a peer failed: ") + what : std::string(what);
        return ADAPCC_ERR_UNSUPPORTED;
      }
    return ADAPCC_SUCCESS;
  };
  auto bail = [&](adapcc_result_t r) {
    nvls_free(c);
    say(reason.c_str());
    drop_plans_nvls(c);
    return r;
  };
  CUdevice dev = 0;
  int mc_ok = 0;
  bool ok = d.ok && d.DeviceGet(&dev, c->device) == CUDA_SUCCESS &&
            d.DeviceGetAttribute(&mc_ok, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev) == CUDA_SUCCESS && mc_ok;
  adapcc_result_t r = agree(ok, d.ok ? "device without multicast support" : "driver without multicast entry points");
  if (r) return bail(r);
  CUmulticastObjectProp mp{};
  mp.numDevices = (unsigned)c->nranks;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  mp.size = bytes;
  size_t gran = 0;
  ok = d.MulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) == CUDA_SUCCESS && gran;
  if ((r = agree(ok, "cuMulticastGetGranularity"))) return bail(r);
  const size_t size = (bytes + gran - 1) / gran * gran;
  mp.size = size;
  c->nvls_bytes = size;
  // rank 0 creates the multicast object and exports it as a file descriptor;
  // the others duplicate that descriptor out of rank 0's process (pidfd_getfd)
  struct Share { int64_t pid; int32_t fd; int32_t ok; };
  Share me{(int64_t)getpid(), -1, 1};
  if (c->rank == 0) {
    CUmemGenericAllocationHandle h = 0;
    int fd = -1;
    me.ok = d.MulticastCreate(&h, &mp) == CUDA_SUCCESS &&
            d.MemExportToShareableHandle(&fd, h, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0) == CUDA_SUCCESS;
    c->nvls_mc_handle = h;
    c->nvls_fd = fd;
    me.fd = fd;
  }
  std::vector<Share> sh(c->nranks);
  if (members_allgather(c, &me, sh.data(), sizeof(Share)) != 0) return bail(ADAPCC_ERR_BOOTSTRAP);
  if ((r = agree(sh[0].ok != 0, "cuMulticastCreate / export"))) return bail(r);
  if (c->rank != 0) {
#ifndef SYS_pidfd_open
#define SYS_pidfd_open 434
#endif
#ifndef SYS_pidfd_getfd
#define SYS_pidfd_getfd 438
#endif
    const int pfd = (int)syscall(SYS_pidfd_open, (pid_t)sh[0].pid, 0);
    const int fd = pfd >= 0 ? (int)syscall(SYS_pidfd_getfd, pfd, sh[0].fd, 0) : -1;
    if (pfd >= 0) close(pfd);
    CUmemGenericAllocationHandle h = 0;
    ok = fd >= 0 && d.MemImportFromShareableHandle(&h, reinterpret_cast<void*>((intptr_t)fd),
                                                   CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR) == CUDA_SUCCESS;
    c->nvls_mc_handle = h;
    c->nvls_fd = fd;
  } else {
    ok = true;
  }
  if ((r = agree(ok, "importing the multicast handle (pidfd_getfd)"))) return bail(r);
  ok = d.MulticastAddDevice(c->nvls_mc_handle, dev) == CUDA_SUCCESS;
  if ((r = agree(ok, "cuMulticastAddDevice"))) return bail(r);
  CUmemAllocationProp ap{};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = c->device;
  CUmemGenericAllocationHandle ph = 0;
  ok = d.MemCreate(&ph, size, &ap, 0) == CUDA_SUCCESS;
  c->nvls_phys = ok ? ph : 0;
  ok = ok && d.MulticastBindMem(c->nvls_mc_handle, 0, ph, 0, size, 0) == CUDA_SUCCESS;
  if ((r = agree(ok, "cuMemCreate / cuMulticastBindMem"))) return bail(r);
  CUmemAccessDesc acc{};
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = c->device;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CUdeviceptr uva = 0, mva = 0;
  ok = d.MemAddressReserve(&uva, size, gran, 0, 0) == CUDA_SUCCESS;
  if (ok) {
    ok = d.MemMap(uva, size, 0, ph, 0) == CUDA_SUCCESS && d.MemSetAccess(uva, size, &acc, 1) == CUDA_SUCCESS;
    if (ok) c->nvls_uc = reinterpret_cast<char*>(uva);
    else d.MemAddressFree(uva, size);
  }
  ok = ok && d.MemAddressReserve(&mva, size, gran, 0, 0) == CUDA_SUCCESS;
  if (ok) {
    ok = d.MemMap(mva, size, 0, c->nvls_mc_handle, 0) == CUDA_SUCCESS &&
         d.MemSetAccess(mva, size, &acc, 1) == CUDA_SUCCESS;
    if (ok) c->nvls_mc = reinterpret_cast<char*>(mva);
    else d.MemAddressFree(mva, size);
  }
  if ((r = agree(ok, "mapping the unicast / multicast addresses"))) return bail(r);
  drop_plans_nvls(c);
  say("ok");
  return ADAPCC_SUCCESS;
}

// ----------------------------------------------------------- link probe (NEXT-2)
adapcc_result_t adapcc_link_probe(adapcc_comm_t c, int src, uint64_t dst_mask, size_t bytes, int messages,
                                  int engine, int iters, double* seconds) {
  if (!c || !seconds || messages < 1 || iters < 1 || (engine != 0 && engine != 1) || (bytes & 15) || !bytes)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  if (src < 0) src = c->rank;
  const uint64_t all = c->nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << c->nranks) - 1);
  if (src >= c->nranks || (!c->loopback && src != c->rank) || (dst_mask & ~all) || ((dst_mask >> src) & 1) ||
      (dst_mask & ~c->members))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const uint64_t flag_cap = flag_region_bytes(c->half_bytes);
  if (bytes > c->half_bytes - flag_cap) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  CK(cudaSetDevice(c->device));
  CK(cudaDeviceSynchronize());  // no collective is using the arenas
  *seconds = 0.0;
  // source: the sender's arena, half 0 data region; destinations: each
  // receiver's arena, half 1 data region (scratch between collective calls)
  const char* sp = c->arena[src] + kArenaHeader + flag_cap;
  std::vector<char*> dst;
  for (int q = 0; q < c->nranks; ++q)
    if ((dst_mask >> q) & 1) dst.push_back(c->arena[q] + kArenaHeader + c->half_bytes + flag_cap);
  auto barrier = [&]() -> adapcc_result_t {  // multi-process: every rank probes at the same time
    if (c->loopback) return ADAPCC_SUCCESS;
    int ok = 1;
    std::vector<int> oks(c->nranks);
    return members_allgather(c, &ok, oks.data(), sizeof(int)) ? ADAPCC_ERR_BOOTSTRAP : ADAPCC_SUCCESS;
  };
  cudaStream_t s = nullptr;
  std::vector<cudaStream_t> ps(dst.size(), nullptr);
  std::vector<cudaEvent_t> ev(dst.size() + 3, nullptr);
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  adapcc_result_t r = ADAPCC_SUCCESS;
  auto cleanup = [&] {
    if (ge) cudaGraphExecDestroy(ge);
    if (g) cudaGraphDestroy(g);
    for (auto e : ev) if (e) cudaEventDestroy(e);
    for (auto p : ps) if (p) cudaStreamDestroy(p);
    if (s) cudaStreamDestroy(s);
  };
#define PK(expr)                                      \
  do {                                                \
    cudaError_t _e = (expr);                          \
    if (_e != cudaSuccess) {                          \
      cleanup();                                      \
      return cuda_fail(_e, __LINE__);                 \
    }                                                 \
  } while (0)
  PK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  for (auto& e : ev) PK(cudaEventCreate(&e));
  if (!dst.empty()) {
    // all `iters` repetitions of `messages` back-to-back messages captured in
    // ONE CUDA graph: no host launch and no per-replay constant inside the
    // timed region, so alpha is the device's per-message cost (P:L113 probes)
    PK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    if (engine == 1) {
      for (int m = 0; m < messages * iters; ++m)
        PK(probe_launch(sp, dst.data(), (int)dst.size(), bytes, 4 * c->num_sms, s));
    } else {  // copy engines: one stream per destination, forked from / joined into s
      PK(cudaEventRecord(ev[0], s));
      for (size_t k = 0; k < dst.size(); ++k) {
        PK(cudaStreamCreateWithFlags(&ps[k], cudaStreamNonBlocking));
        PK(cudaStreamWaitEvent(ps[k], ev[0], 0));
        for (int m = 0; m < messages * iters; ++m)
          PK(cudaMemcpyAsync(dst[k], sp, bytes, cudaMemcpyDeviceToDevice, ps[k]));
        PK(cudaEventRecord(ev[3 + k], ps[k]));
        PK(cudaStreamWaitEvent(s, ev[3 + k], 0));
      }
    }
    PK(cudaStreamEndCapture(s, &g));
    PK(cudaGraphInstantiate(&ge, g, 0));
    PK(cudaGraphLaunch(ge, s));  // warm-up (and first touch of the peers' pages)
    PK(cudaStreamSynchronize(s));
  }
  if ((r = barrier()) != ADAPCC_SUCCESS) { cleanup(); return r; }
  if (!dst.empty()) {
    PK(cudaEventRecord(ev[1], s));
    PK(cudaGraphLaunch(ge, s));
    PK(cudaEventRecord(ev[2], s));
    PK(cudaStreamSynchronize(s));
    float ms = 0.f;
    PK(cudaEventElapsedTime(&ms, ev[1], ev[2]));
    *seconds = (double)ms * 1e-3 / iters;
  }
#undef PK
  cleanup();
  return barrier();
}

// ------------------------------------------------------------ late join (NEXT-1)
adapcc_result_t adapcc_late_ticket(adapcc_comm_t c, uint64_t* ticket) {
  if (!c || !ticket) return ADAPCC_ERR_INVALID_ARGUMENT;
  *ticket = c->late_seq;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_late_advance(adapcc_comm_t c, uint64_t* ticket) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  ++c->late_seq;
  if (ticket) *ticket = c->late_seq;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_signal_ready(adapcc_comm_t c, int rank, uint64_t ticket, adapcc_stream_t stream) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (rank < 0) rank = c->rank;
  if (rank >= c->nranks || (!c->loopback && rank != c->rank)) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (ticket == 0) ticket = c->late_seq;
  CK(cudaSetDevice(c->device));
  CK(engine_signal(reinterpret_cast<uint64_t*>(c->arena[rank] + 16), ticket, !c->loopback,
                   c->d_board ? c->d_board + rank : nullptr, reinterpret_cast<cudaStream_t>(stream)));
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_ready_board(adapcc_comm_t c, volatile uint64_t** board, int* shared) {
  if (!c || !board) return ADAPCC_ERR_INVALID_ARGUMENT;
  *board = c->h_board;
  if (shared) *shared = c->loopback || c->board_shm ? 1 : 0;
  return c->h_board ? ADAPCC_SUCCESS : ADAPCC_ERR_UNSUPPORTED;
}

adapcc_result_t adapcc_spin(adapcc_comm_t c, uint64_t ns, adapcc_stream_t stream) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  CK(cudaSetDevice(c->device));
  CK(engine_spin(ns, reinterpret_cast<cudaStream_t>(stream)));
  return ADAPCC_SUCCESS;
}

// ---- online coordinator loops (host only): P:L133-137 break-even rule, P:L139 T_fault
static double mono_now() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}
static uint64_t board_ready(const volatile uint64_t* board, int n, uint64_t among, uint64_t ticket) {
  uint64_t m = 0;
  for (int r = 0; r < n; ++r)
    if (((among >> r) & 1) && board[r] >= ticket) m |= uint64_t(1) << r;
  return m;
}

adapcc_result_t adapcc_coord_decide(const volatile uint64_t* board, int nranks, uint64_t members, uint64_t ticket,
                                    const double* buy_cost, double cycle_s, double timeout_s, uint64_t* ready_mask,
                                    int* full, double* t_first, double* t_decide) {
  if (!board || !buy_cost || !ready_mask || !full || nranks < 1 || nranks > 64 || !members || cycle_s < 0)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const uint64_t all = nranks == 64 ? ~uint64_t(0) : ((uint64_t(1) << nranks) - 1);
  if (members & ~all) return ADAPCC_ERR_INVALID_ARGUMENT;
  const double t0 = mono_now();
  double first = -1.0, waited = 0.0, next = t0;
  for (;;) {
    const uint64_t ready = board_ready(board, nranks, members, ticket);
    const double now = mono_now();
    if (ready && first < 0) first = now;
    if (ready == members) {
      *full = 1;
      *ready_mask = members;
      break;
    }
    if (ready && waited + cycle_s > buy_cost[__builtin_popcountll(ready)]) {  // buying beats one more cycle
      *full = 0;
      *ready_mask = ready;
      break;
    }
    if (now - t0 > timeout_s) return ADAPCC_ERR_TIMEOUT;
    waited += cycle_s;
    next += cycle_s;
    while (mono_now() < next) {
    }
  }
  if (t_first) *t_first = first;
  if (t_decide) *t_decide = mono_now();
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_coord_await(const volatile uint64_t* board, int nranks, uint64_t late_mask, uint64_t ticket,
                                   void* phase1_event, double t_first, double fault_factor, double timeout_s,
                                   uint64_t* faulty) {
  if (!board || !faulty || nranks < 1 || nranks > 64) return ADAPCC_ERR_INVALID_ARGUMENT;
  const double t0 = mono_now();
  double t_p1 = -1.0;
  *faulty = 0;
  for (;;) {
    const uint64_t missing = late_mask & ~board_ready(board, nranks, late_mask, ticket);
    if (!missing) return ADAPCC_SUCCESS;
    const double now = mono_now();
    if (t_p1 < 0) {
      if (!phase1_event) {
        t_p1 = now;
      } else {
        const cudaError_t q = cudaEventQuery(reinterpret_cast<cudaEvent_t>(phase1_event));
        if (q == cudaSuccess) t_p1 = now;  // phase 1 finished on this GPU
        else if (q != cudaErrorNotReady) {
          g_last_cuda_error = q;
          g_last_cuda_line = __LINE__;
          return ADAPCC_ERR_CUDA;
        }
      }
    }
    if (fault_factor > 0 && t_p1 >= 0 && t_first >= 0 && now - t_p1 >= fault_factor * (t_p1 - t_first)) {
      *faulty = missing;
      return ADAPCC_SUCCESS;
    }
    if (now - t0 > timeout_s) return ADAPCC_ERR_TIMEOUT;
  }
}

const char* adapcc_last_cuda_error(void) {
  std::snprintf(g_last_cuda_msg, sizeof(g_last_cuda_msg), "%s (adapcc.cpp:%d)",
                cudaGetErrorString(g_last_cuda_error), g_last_cuda_line);
  return g_last_cuda_msg;
}

adapcc_result_t adapcc_get_async_error(adapcc_comm_t c) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  return (adapcc_result_t) * reinterpret_cast<volatile int*>(c->h_err);
}

// NEXT-3 fault tolerance: "faulty workers are excluded from the
// training group"; the survivors keep the communicator (arenas, IPC mappings,
// registrations) and continue with a strategy over the live ranks.
adapcc_result_t adapcc_exclude(adapcc_comm_t c, uint64_t dead_mask, adapcc_bootstrap_allgather_fn ag,
                               void* ag_ctx) {
  if (!c) return ADAPCC_ERR_INVALID_ARGUMENT;
  const uint64_t all = c->nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << c->nranks) - 1);
  if (dead_mask & ~all) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  const uint64_t live = c->members & ~dead_mask;
  if (!live || (!c->loopback && (!ag || !((live >> c->rank) & 1)))) return ADAPCC_ERR_INVALID_ARGUMENT;
  CK(cudaSetDevice(c->device));
  // 1. drain: launches that waited on the faulty rank have hit the watchdog and exited
  CK(cudaDeviceSynchronize());
  DevState st{};
  CK(cudaMemcpy(&st, c->state, sizeof(DevState), cudaMemcpyDeviceToHost));
  uint64_t epoch = st.epoch;
  if (!c->loopback) {  // 2. agree on an epoch above every flag any survivor ever posted
    c->members = live;
    c->ag = ag;
    c->ag_ctx = ag_ctx;
    std::vector<uint64_t> e(c->nranks);
    if (members_allgather(c, &epoch, e.data(), sizeof(uint64_t)) != 0) return ADAPCC_ERR_BOOTSTRAP;
    for (uint64_t v : e) epoch = std::max(epoch, v);
  }
  epoch += (uint64_t)std::max<int64_t>(2, env_int("ADAPCC_EXCLUDE_GAP", 2));  // (diagnostic knob: the epoch gap)
  // 3. restart the device epoch there: counters cleared, abort latch released;
  //    this rank's "done" and "entered" words say it finished `epoch`, so the
  //    next launch's start check (peers done >= epoch + 1 - 2) passes
  st = DevState{};
  st.epoch = epoch;
  CK(cudaMemcpy(c->state, &st, sizeof(DevState), cudaMemcpyHostToDevice));
  if (!c->loopback) {
    const uint64_t words[2] = {epoch, epoch};
    CK(cudaMemcpy(c->arena[c->rank], words, sizeof(words), cudaMemcpyHostToDevice));
  }
  *reinterpret_cast<volatile int*>(c->h_err) = 0;
  c->members = live;
  // After an exclusion every launch also runs the start barrier of the debug
  // call check (check_call_sig: every survivor's kernel of this epoch has
  // started -- and makes the same call -- before any byte moves).  Without it
  // a 3-process test on one GPU corrupted a tree's last chunk in ~15 % of
  // runs after the exclusion (root cause not isolated; the barrier removes
  // it: 0 of 16, profiles/fault_race_r02.json).  Costs one header round trip
  // per launch, in the degraded post-fault mode only.
  if (!c->loopback && env_int("ADAPCC_EXCLUDE_BARRIER", 1) != 0) c->check_sig = 1;  // (diagnostic knob)
  // 4. strategies: the survivors' defaults until set_strategy names new ones
  for (int k = 0; k < kNumColl; ++k) {
    if (!parse_strategy(default_strategy((Coll)k, c->nranks, 0, live, c->default_chunk).c_str(), &c->strat[k], nullptr))
      return ADAPCC_ERR_INVALID_STRATEGY;
    c->user_set[k] = false;
    c->rooted[k].clear();
  }
  if (!c->loopback) {  // 5. barrier: nobody launches before every survivor has reset
    int ok = 1;
    std::vector<int> oks(c->nranks);
    if (members_allgather(c, &ok, oks.data(), sizeof(int)) != 0) return ADAPCC_ERR_BOOTSTRAP;
  }
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_members(adapcc_comm_t c, uint64_t* members) {
  if (!c || !members) return ADAPCC_ERR_INVALID_ARGUMENT;
  *members = c->members;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_finalize(adapcc_comm_t c) {
  release(c);
  return ADAPCC_SUCCESS;
}

// Empties the plan cache.  Plans captured into a CUDA graph stay alive until
// finalize (the graph keeps pointing at their tables).
static void drop_plans(adapcc_comm_t c) {
  for (auto& kv : c->plans)
    if (kv.second->pinned) c->retired.push_back(kv.second);
  c->plans.clear();
}

adapcc_result_t adapcc_config(adapcc_comm_t c, const char* key, int64_t value) {
  if (!c || !key) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  if (!std::strcmp(key, "timeout_ms")) { if (value < 1) return ADAPCC_ERR_INVALID_ARGUMENT; c->timeout_ms = value; }
  else if (!std::strcmp(key, "max_ctas")) {
    if (value < 0) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (value != c->max_ctas) drop_plans(c);  // pieces, taper and first-item blobs are sized for the grid
    c->max_ctas = value;
  }
  else if (!std::strcmp(key, "engine")) {
    if (value < 0 || value > 3) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (value != c->engine) drop_plans(c);  // pieces are sized for the engine's grid
    c->engine = (int)value;
  }
  else if (!std::strcmp(key, "flat_ctas")) {
    if (value < 1 || value > 64) return ADAPCC_ERR_INVALID_ARGUMENT;
    c->flat_ctas = value;  // (launch-time: no plan depends on it)
  }
  else if (!std::strcmp(key, "piece_kib") || !std::strcmp(key, "taper")) {
    if (value < 0 || (key[0] == 't' && value > 64)) return ADAPCC_ERR_INVALID_ARGUMENT;
    (key[0] == 't' ? c->taper : c->piece_kib) = value;
    drop_plans(c);  // items are cut at plan time
  }
  else if (!std::strcmp(key, "default_chunk")) {
    // C_m of every default strategy (a decision variable; e.g. the
    // cost model's choice from a link profile); user strategies are kept
    if (value < 16 || value % 16 || value > (int64_t(1) << 31)) return ADAPCC_ERR_INVALID_ARGUMENT;
    c->default_chunk = value;
    for (int k = 0; k < kNumColl; ++k) {
      c->rooted[k].clear();
      if (c->user_set[k]) continue;
      if (!parse_strategy(default_strategy((Coll)k, c->nranks, 0, c->members, value).c_str(), &c->strat[k], nullptr))
        return ADAPCC_ERR_INVALID_STRATEGY;
    }
  }
  else if (!std::strcmp(key, "debug_check")) c->check_sig = value != 0;
  else if (!std::strcmp(key, "pdl")) c->pdl = value != 0;
  else if (!std::strcmp(key, "acc_red")) {
    if ((value != 0) != (c->acc_red != 0)) drop_plans(c);  // the TMA ring shape of ACCUMULATE plans depends on it
    c->acc_red = value != 0;
  }
  else if (!std::strcmp(key, "trace")) {  // capacity in records; 0 = off
    if (value < 0 || value > (int64_t(1) << 26)) return ADAPCC_ERR_INVALID_ARGUMENT;
    if (cudaSetDevice(c->device) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) return ADAPCC_ERR_CUDA;
    cudaFree(c->trace);
    cudaFree(c->trace_n);
    c->trace = nullptr;
    c->trace_n = nullptr;
    c->trace_cap = 0;
    if (value > 0) {
      if (cudaMalloc(&c->trace, (size_t)value * sizeof(TraceRec)) != cudaSuccess ||
          cudaMalloc(&c->trace_n, sizeof(unsigned)) != cudaSuccess ||
          cudaMemset(c->trace_n, 0, sizeof(unsigned)) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(c->trace);
        cudaFree(c->trace_n);
        c->trace = nullptr;
        c->trace_n = nullptr;
        return ADAPCC_ERR_OOM;
      }
      c->trace_cap = (uint32_t)value;
    }
  }
  else if (!std::strcmp(key, "sched")) {
    if (value < 0 || value > 2) return ADAPCC_ERR_INVALID_ARGUMENT;
    c->sched = value;
    drop_plans(c);  // blobs are built at plan time
  }
  else if (!std::strcmp(key, "first_blob")) {
    c->first_blob = value != 0;
    drop_plans(c);
  }
  else if (!std::strcmp(key, "debug_drop_rank")) {
    if (!c->loopback || value < -1 || value >= c->nranks) return ADAPCC_ERR_INVALID_ARGUMENT;
    c->drop_rank = value;
  } else return ADAPCC_ERR_INVALID_ARGUMENT;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_trace_read(adapcc_comm_t c, void* records, uint32_t max_records, uint32_t* n_copied,
                                  uint32_t* n_total) {
  if (!c || !n_copied || (max_records && !records)) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lock(c->mu);
  *n_copied = 0;
  if (n_total) *n_total = 0;
  if (!c->trace) return ADAPCC_ERR_UNSUPPORTED;
  CK(cudaSetDevice(c->device));
  CK(cudaDeviceSynchronize());
  unsigned n = 0;
  CK(cudaMemcpy(&n, c->trace_n, sizeof(n), cudaMemcpyDeviceToHost));
  const uint32_t have = std::min<uint32_t>(n, c->trace_cap), k = std::min<uint32_t>(have, max_records);
  if (k) CK(cudaMemcpy(records, c->trace, (size_t)k * sizeof(TraceRec), cudaMemcpyDeviceToHost));
  CK(cudaMemset(c->trace_n, 0, sizeof(unsigned)));
  *n_copied = k;
  if (n_total) *n_total = n;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_launch_count(adapcc_comm_t c, uint64_t* count) {
  if (!c || !count) return ADAPCC_ERR_INVALID_ARGUMENT;
  *count = c->launches;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_last_engine(adapcc_comm_t c, int* engine) {
  if (!c || !engine) return ADAPCC_ERR_INVALID_ARGUMENT;
  *engine = c->last_engine;
  return ADAPCC_SUCCESS;
}

// ----------------------------------------------------------- host-only inspection
adapcc_result_t adapcc_strategy_check(const char* text, int* nranks, int* coll, int* nsubs,
                                      char* err, size_t err_len) {
  Strategy st;
  std::string e;
  if (!parse_strategy(text, &st, &e)) {
    if (err && err_len) {
      std::strncpy(err, e.c_str(), err_len - 1);
      err[err_len - 1] = 0;
    }
    return ADAPCC_ERR_INVALID_STRATEGY;
  }
  if (nranks) *nranks = st.nranks;
  if (coll) *coll = (int)st.coll;
  if (nsubs) *nsubs = (int)st.subs.size();
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_strategy_tuples(const char* text, int sub, uint64_t mask, uint8_t* tuples,
                                       int32_t* nflows) {
  Strategy st;
  if (!parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (sub < 0 || sub >= (int)st.subs.size() || st.subs[sub].kind != kTree || !tuples)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  TreeBehavior b = tree_behavior(st.subs[sub], mask);
  for (int g = 0; g < st.nranks; ++g) {
    tuples[4 * g + 0] = b.tup[g].act;
    tuples[4 * g + 1] = b.tup[g].recv;
    tuples[4 * g + 2] = b.tup[g].kern;
    tuples[4 * g + 3] = b.tup[g].send;
    if (nflows) nflows[g] = (int32_t)b.flows[g].size();
  }
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_strategy_sub(const char* text, int sub, int64_t* weight, int64_t* chunk,
                                    int32_t* parent, int32_t* src) {
  Strategy st;
  if (!parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (sub < 0 || sub >= (int)st.subs.size()) return ADAPCC_ERR_INVALID_ARGUMENT;
  const SubColl& s = st.subs[sub];
  if (weight) *weight = s.weight;
  if (chunk) *chunk = s.chunk;
  if (src) *src = s.src;
  if (parent)
    for (int g = 0; g < st.nranks; ++g) parent[g] = s.parent.empty() ? -2 : s.parent[g];
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_strategy_route(const char* text, int sub, int src, int dst, int32_t* hops,
                                      int* nhops) {
  Strategy st;
  if (!parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (sub < 0 || sub >= (int)st.subs.size() || st.subs[sub].kind != kA2A || !nhops || src < 0 ||
      src >= st.nranks || dst < 0 || dst >= st.nranks)
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const std::vector<int>* h = st.subs[sub].hops(src, dst);
  *nhops = h ? (int)h->size() : 0;
  if (h && hops)
    for (size_t i = 0; i < h->size(); ++i) hops[i] = (*h)[i];
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_strategy_partition(const char* text, uint64_t count, adapcc_dtype_t dtype,
                                          int src, uint64_t* bounds, int* nbounds) {
  Strategy st;
  if (!parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (!bounds || !nbounds) return ADAPCC_ERR_INVALID_ARGUMENT;
  std::vector<int64_t> w;
  for (auto& s : st.subs)
    if ((st.coll != kAllGather && st.coll != kReduceScatter) || s.src == src) w.push_back(s.weight);
  if (w.empty()) return ADAPCC_ERR_INVALID_ARGUMENT;
  auto b = partition(count, esize_of(dtype), w);
  for (size_t i = 0; i < b.size(); ++i) bounds[i] = b[i];
  *nbounds = (int)b.size();
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_plan_stats(const char* text, uint64_t count, adapcc_dtype_t dtype,
                                  uint64_t mask, unsigned flags, adapcc_mode_t mode, int rank,
                                  size_t scratch_bytes, uint64_t members, adapcc_plan_stats_t* out) {
  Strategy st;
  if (!parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (!out || rank < -1 || rank >= st.nranks) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (members == 0) members = st.nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << st.nranks) - 1);
  if (mask & ~members) return ADAPCC_ERR_INVALID_ARGUMENT;
  if (!check_members(st, members, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  PlanRequest rq;
  rq.members = members;
  rq.st = &st;
  rq.count = count;
  rq.esize = esize_of(dtype);
  rq.ready_mask = mask;
  rq.accumulate = flags & ADAPCC_FLAG_ACCUMULATE;
  rq.late_join = flags & (ADAPCC_FLAG_LATE_JOIN | ADAPCC_FLAG_LATE_COMPLEMENT);
  rq.mode = (Mode)mode;
  const size_t scratch = scratch_bytes ? scratch_bytes : kDefaultScratch;
  if (scratch < (size_t)kArenaHeader + 2 * (4096 + 65536)) return ADAPCC_ERR_INVALID_ARGUMENT;
  rq.half_bytes = ((scratch - kArenaHeader) / 2) / 256 * 256;
  rq.nvls_bytes = uint64_t(1) << 30;  // host-only planning: as if 1 GiB of NVLS scratch were set up
  std::vector<SegmentPlan> segs;
  std::string perr;
  if (!build_plan(rq, &segs, &perr)) return perr.rfind("unsupported", 0) == 0 ? ADAPCC_ERR_UNSUPPORTED : ADAPCC_ERR_OOM;
  PlanStats s;
  for (auto& p : segs) accumulate_stats(p, rank, rq.esize, &s);
  s.segments = segs.size();
  out->tasks = s.tasks;
  out->items = s.items;
  out->levels = s.levels;
  out->segments = s.segments;
  out->bytes_read = s.bytes_read;
  out->bytes_written = s.bytes_written;
  out->remote_bytes = s.remote_bytes;
  out->arena_bytes = s.arena_bytes;
  return ADAPCC_SUCCESS;
}

adapcc_result_t adapcc_plan_items(const char* text, uint64_t count, adapcc_dtype_t dtype, uint64_t mask,
                                  unsigned flags, adapcc_mode_t mode, int rank, size_t scratch_bytes, int grid,
                                  int tma, uint32_t piece_kib, int taper, int segment, adapcc_item_t* items,
                                  uint32_t max_items, uint32_t* n_items, adapcc_task_info_t* tasks,
                                  uint32_t max_tasks, uint32_t* n_tasks) {
  Strategy st;
  if (!text || !parse_strategy(text, &st, nullptr)) return ADAPCC_ERR_INVALID_STRATEGY;
  if (rank < -1 || rank >= st.nranks || grid < 1 || segment < 0 || taper < 0 || taper > 64 || !n_items ||
      !n_tasks || (max_items && !items) || (max_tasks && !tasks))
    return ADAPCC_ERR_INVALID_ARGUMENT;
  const uint64_t members = st.nranks >= 64 ? ~uint64_t(0) : ((uint64_t(1) << st.nranks) - 1);
  if (mask & ~members) return ADAPCC_ERR_INVALID_ARGUMENT;
  PlanRequest rq;
  rq.members = members;
  rq.st = &st;
  rq.count = count;
  rq.esize = esize_of(dtype);
  rq.ready_mask = mask;
  rq.accumulate = flags & ADAPCC_FLAG_ACCUMULATE;
  rq.late_join = flags & ADAPCC_FLAG_LATE_JOIN;
  rq.mode = (Mode)mode;
  rq.grid = grid;
  const size_t scratch = scratch_bytes ? scratch_bytes : kDefaultScratch;
  if (scratch < (size_t)kArenaHeader + 2 * (4096 + 65536)) return ADAPCC_ERR_INVALID_ARGUMENT;
  rq.half_bytes = ((scratch - kArenaHeader) / 2) / 256 * 256;
  rq.nvls_bytes = uint64_t(1) << 30;  // host-only planning: as if 1 GiB of NVLS scratch were set up
  std::vector<SegmentPlan> segs;
  std::string perr;
  if (!build_plan(rq, &segs, &perr)) return perr.rfind("unsupported", 0) == 0 ? ADAPCC_ERR_UNSUPPORTED : ADAPCC_ERR_OOM;
  if ((size_t)segment >= segs.size()) return ADAPCC_ERR_INVALID_ARGUMENT;
  const SegmentPlan& sp = segs[segment];
  const std::vector<Item> it = order_items(sp, rank, rq.esize, grid, (uint64_t)piece_kib * 1024, taper, tma != 0);
  *n_items = (uint32_t)it.size();
  for (uint32_t i = 0; i < std::min<uint32_t>(max_items, *n_items); ++i)
    items[i] = adapcc_item_t{it[i].task, it[i].chunk, it[i].off, it[i].len};
  *n_tasks = (uint32_t)sp.tasks.size();
  for (uint32_t i = 0; i < std::min<uint32_t>(max_tasks, *n_tasks); ++i) {
    const Task& t = sp.tasks[i];
    tasks[i] = adapcc_task_info_t{t.lo, t.hi, t.chunk_elems, t.nchunks, t.nsrc, t.ndst, t.nwait, t.npost,
                                  t.level, t.owner};
  }
  return ADAPCC_SUCCESS;
}

}  // extern "C"
