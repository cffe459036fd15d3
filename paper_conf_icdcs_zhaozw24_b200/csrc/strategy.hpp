// Strategy IR: parsed AdapCC strategy + behaviour tuples + partition.
//
// The paper's strategy (§IV-D): M sub-collectives m, each with its own
// graph (a tree for Reduce/Broadcast), data partition S_m (sum S_m = S,
// P:L167), chunk size C_m and aggregation flags a_{m,g},
// shipped to every worker (XML in the paper; our text format is
// DESIGN.md §2).  This is the product-side loader; the CPU oracle has its own
// independent parser (oracle/strategy.py).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace adapcc {

constexpr int kMaxRanks = 64;
constexpr int kMaxSubs = 128;
constexpr int64_t kMaxWeight = int64_t(1) << 24;
constexpr int64_t kMaxChunk = int64_t(1) << 31;

enum Coll : int {
  kAllReduce = 0, kAllGather = 1, kAllToAll = 2,
  kReduce = 3, kBroadcast = 4, kReduceScatter = 5  // NEXT-4 primitives
};
constexpr int kNumColl = 6;
enum SubKind : int { kTree = 0, kBcast = 1, kA2A = 2, kRTree = 3,
                     kNvls = 4 /* allreduce partition reduced by the NVSwitch (multimem, NEXT-2) */ };

// One routed AlltoAll flow (routing variables x^f_ij, eq. 1): block
// src -> dst travels src -> hops[0] -> ... -> hops.back() -> dst.
struct Route {
  int src = -1, dst = -1;
  std::vector<int> hops;
};

struct SubColl {
  SubKind kind = kTree;
  int64_t weight = 0;          // effective integer weight (ring chains: w, others: w*n)
  int64_t chunk = 0;           // C_m, bytes, multiple of 16
  std::vector<int> parent;     // tree / bcast; -1 at the root
  uint64_t noagg = 0;          // bit g: a_{m,g} = 0
  bool relay_store = false;    // tree: pure relays store-and-forward through their arena (relay=store)
  int src = -1;                // bcast: source; rtree: destination block (== root)
  int root = -1;
  std::vector<std::vector<int>> children;  // ascending rank order (reading Q5)
  std::vector<Route> routes;   // a2a: flows that do not go direct (sorted by (src, dst))
  // a2a: relay ranks of flow src -> dst (empty = direct)
  const std::vector<int>* hops(int src, int dst) const;
};

struct Strategy {
  int nranks = 0;
  Coll coll = kAllReduce;
  std::vector<SubColl> subs;
  uint64_t hash = 0;           // FNV-1a of the normalised text
};

// Parse + validate; returns false and fills *err on failure.
bool parse_strategy(const char* text, Strategy* out, std::string* err);

// Fault tolerance (NEXT-3): after faulty ranks are excluded, a
// strategy may still name them, but only where they have nothing to do:
// leaves of every tree / broadcast tree whose source or destination is alive,
// never an AlltoAll relay, never the Reduce root or Broadcast source.
bool check_members(const Strategy& st, uint64_t members, std::string* err);

// Reading Q9: bounds of `count` elements over `weights` (size M -> M+1 bounds).
std::vector<uint64_t> partition(uint64_t count, int esize, const std::vector<int64_t>& weights);

// Behaviour tuple <isActive, hasRecv, hasKernel, hasSend>.
struct Tuple {
  bool act = false, recv = false, kern = false, send = false;
};

// A flow leaving a node (P:L154(3), Fig. 8(b)): rank r's own tensor or the
// aggregate formed at kernel node r.
struct Flow {
  enum Kind : int { kIn = 0, kAgg = 1 } kind;
  int rank;
};

struct TreeBehavior {
  std::vector<Tuple> tup;                 // per rank
  std::vector<std::vector<Flow>> flows;   // per rank, flows emitted upward
  std::vector<int> postorder;             // children before parents
};

TreeBehavior tree_behavior(const SubColl& s, uint64_t ready_mask);

// Ordered inputs folded by kernel node g: own tensor if ready, then the flows
// of its sending children by ascending rank (reading Q5).
std::vector<Flow> kernel_sources(const SubColl& s, const TreeBehavior& b, int g);

}  // namespace adapcc
