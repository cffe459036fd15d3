// Plan compiler (see plan.hpp).  Data movement per collective and mode:
//
// AllReduce, tree m over [lo,hi) ("generate strategies for Reduce and
// execute Broadcast reversely"):
//   DIRECT  kernel node k (non-root): fold(sources(k)) -> slot_k, post flag_k
//           root: fold(sources(root)) (or its single flow / zero) -> every
//           rank's recvbuf (the broadcast collapses to one write per rank
//           because every recvbuf is addressable).
//   STAGED  every flow is pushed by its producer into a landing slot in the
//           arena of its consumer (the kernel node that folds it, P:L263
//           "send one chunk ... an event is then recorded"); the root folds
//           into its own recvbuf and its broadcast slot; every other rank
//           pulls the result from its tree parent's broadcast slot into its
//           recvbuf and, if it has children, into its own broadcast slot
//           (the reversed tree, pipelined per chunk).
//   Pure relays forward by reference: their single incoming flow is
//   pushed straight to their consumer, because on a uniform NVSwitch a
//   store-and-forward hop adds bytes on the relay's ports without adding link
//   capacity.  Relays still receive the result (Q4).
// AllGather: one broadcast tree per source.
// AlltoAll: block d of s lands in block s of d, direct or along the
// flow's route (eq. 1).
#include "plan.hpp"

#include <algorithm>
#include <map>
#include <tuple>

namespace adapcc {
namespace {

constexpr uint64_t kAlign = 256;

uint64_t align_up(uint64_t v, uint64_t a) { return (v + a - 1) / a * a; }

struct Stream {
  BufRef ref{};
  bool wait = false;
  FlagRef flag{};
};

BufRef make_ref(uint8_t kind, int rank, int64_t bias, bool accum = false) {
  BufRef r{};
  r.bias = bias;
  r.kind = kind;
  r.rank = (uint8_t)rank;
  r.accum = accum ? 1 : 0;
  return r;
}

class Builder {
 public:
  Builder(int n, int esize, uint64_t half, uint64_t members, uint64_t unit_cap)
      : n_(n), esize_(esize), half_(half), flag_cap_(flag_region_bytes(half)), members_(members),
        unit_cap_(unit_cap), used_(n, 0), flags_used_(n, 0) {}

  // Pipelining unit (elements) of a sub-collective with chunk C_m: C_m, or a
  // smaller unit when the call is too small to give every CTA work at C_m
  // (reading R8: the strategy's chunk is the largest unit the engine moves
  // between flags; results do not depend on it).
  uint32_t chunk_elems(int64_t chunk_bytes) const {
    const uint64_t b = unit_cap_ ? std::min<uint64_t>((uint64_t)chunk_bytes, unit_cap_) : (uint64_t)chunk_bytes;
    return (uint32_t)(b / esize_);
  }

  bool alive(int g) const { return ((members_ >> g) & 1) != 0; }

  // Each parity half of a rank's arena = [flag region | data region].  Flag
  // words only ever hold epochs (monotonic), so a later plan with a different
  // layout can never mistake an old data byte for a posted flag.
  uint64_t alloc(int r, uint64_t bytes) {
    uint64_t off = flag_cap_ + used_[r];
    used_[r] = align_up(used_[r] + bytes, kAlign);
    return off;
  }
  // a slot preceded by its per-chunk decision words (STAGED late join)
  uint64_t alloc_dec(int r, uint64_t bytes, uint32_t nchunks) {
    const uint64_t d = late_dec_bytes(nchunks);
    return alloc(r, d + bytes) + d;
  }
  FlagRef alloc_flags(int r, uint32_t nchunks) {
    FlagRef f{};
    f.off = flags_used_[r];
    flags_used_[r] = align_up(flags_used_[r] + 8ull * nchunks, 128);
    f.rank = (uint32_t)r;
    return f;
  }
  bool fits() const {
    for (int r = 0; r < n_; ++r)
      if (flags_used_[r] > flag_cap_ || flag_cap_ + used_[r] > half_) return false;
    return nvls_used_ <= nvls_cap_;
  }
  // NVLS scratch: the same offsets on every rank (one multicast address)
  uint64_t nvls_alloc(uint64_t bytes) {
    const uint64_t off = nvls_used_;
    nvls_used_ = align_up(nvls_used_ + bytes, kAlign);
    return off;
  }
  uint64_t nvls_used_ = 0, nvls_cap_ = 0;

  // Slot holding elements [lo,hi) of a stream at rank r: address(e) = base + off + (e-lo)*esize
  Stream slot_stream(int r, uint64_t off, uint64_t lo, const FlagRef* f) {
    Stream s;
    s.ref = make_ref(kBufArena, r, (int64_t)off - (int64_t)(lo * esize_));
    if (f) { s.wait = true; s.flag = *f; }
    return s;
  }

  // late: late-join candidates (root tasks); late_waits: their landing
  // slots' flags (STAGED), waited after the sources' flags; lkind: LateKind
  int add(int owner, uint64_t lo, uint64_t hi, uint32_t ce, uint16_t op,
          const std::vector<Stream>& srcs, const std::vector<BufRef>& dsts,
          const std::vector<FlagRef>& posts, const std::vector<BufRef>& late = {},
          const std::vector<FlagRef>& late_waits = {}, uint8_t lkind = kLateNone) {
    Task t{};
    t.lo = lo;
    t.hi = hi;
    t.chunk_elems = ce;
    t.nchunks = (uint32_t)((hi - lo + ce - 1) / ce);
    t.nsrc = (uint16_t)srcs.size();
    t.ndst = (uint16_t)dsts.size();
    t.op = op;
    t.owner = (uint16_t)owner;
    t.ref0 = (uint32_t)p_.refs.size();
    for (auto& s : srcs) p_.refs.push_back(s.ref);
    for (auto& d : dsts) p_.refs.push_back(d);
    for (auto& l : late) p_.refs.push_back(l);
    t.nlate = (uint16_t)late.size();
    t.flag0 = (uint32_t)p_.flags.size();
    uint32_t level = 0;
    uint16_t nwait = 0;
    for (auto& s : srcs) {
      if (!s.wait) continue;
      p_.flags.push_back(s.flag);
      ++nwait;
      auto it = producer_.find({s.flag.rank, s.flag.off});
      if (it != producer_.end()) level = std::max(level, p_.tasks[it->second].level + 1);
    }
    for (auto& f : late_waits) {
      p_.flags.push_back(f);
      ++nwait;
      auto it = producer_.find({f.rank, f.off});
      if (it != producer_.end()) level = std::max(level, p_.tasks[it->second].level + 1);
    }
    t.nwait = nwait;
    t.nlwait = (uint8_t)late_waits.size();
    t.lkind = lkind;
    for (auto& f : posts) p_.flags.push_back(f);
    t.npost = (uint16_t)posts.size();
    t.level = level;
    const int idx = (int)p_.tasks.size();
    for (auto& f : posts) producer_[{f.rank, f.off}] = idx;
    p_.tasks.push_back(t);
    p_.max_level = std::max(p_.max_level, level);
    return idx;
  }

  // a task with one source stream whose chunk is ready after ALL of `waits`'
  // flags (NVLS: every rank copied its part in)
  int add_multiwait(int owner, uint64_t lo, uint64_t hi, uint32_t ce, uint16_t op, const std::vector<Stream>& waits,
                    const std::vector<BufRef>& dsts, const std::vector<FlagRef>& posts) {
    std::vector<FlagRef> extra;
    for (size_t i = 1; i < waits.size(); ++i) extra.push_back(waits[i].flag);
    const int idx = add(owner, lo, hi, ce, op, {waits[0]}, dsts, posts, {}, extra, kLateNone);
    p_.tasks[idx].nlwait = 0;
    return idx;
  }

  SegmentPlan finish() {
    p_.fits = fits();
    p_.arena_used.resize(n_);
    for (int r = 0; r < n_; ++r) p_.arena_used[r] = flag_cap_ + used_[r];
    return std::move(p_);
  }

  int n_, esize_;
  uint64_t half_, flag_cap_, members_, unit_cap_;
  std::vector<uint64_t> used_, flags_used_;
  SegmentPlan p_;
  std::map<std::pair<uint32_t, uint64_t>, int> producer_;
};

std::vector<int> bfs_order(const SubColl& s) {
  std::vector<int> q = {s.root};
  for (size_t i = 0; i < q.size(); ++i)
    for (int c : s.children[q[i]]) q.push_back(c);
  return q;
}

// ------------------------------------------------------------- AllReduce
// relay=store (relays forward "as intermediaries, relaying tensor
// data from other workers"): a pure relay -- not ready, no kernel, one
// incoming flow (P:L154(2)) -- receives that flow into its own arena and
// forwards it, chunk by chunk, instead of being bypassed.  The behaviour
// tuples are unchanged; for planning the relay's emitted flow becomes its
// stored copy (Flow kAgg at the relay, a one-source "fold" = a byte copy), so
// every consumer still folds the same bytes at the same position.
struct RelayPlan {
  std::vector<uint8_t> store;             // per rank: a store-and-forward relay
  std::vector<std::vector<Flow>> src;     // its single incoming flow
};

RelayPlan store_relays(const SubColl& s, TreeBehavior* b) {
  const int n = (int)s.parent.size();
  RelayPlan rp;
  rp.store.assign(n, 0);
  rp.src.assign(n, {});
  if (!s.relay_store) return rp;
  for (int g : b->postorder) {  // children first: a relay below a relay forwards the stored copy
    const Tuple& t = b->tup[g];
    std::vector<Flow> f;
    if (t.kern) {
      f.push_back({Flow::kAgg, g});
    } else {
      if (t.act) f.push_back({Flow::kIn, g});
      for (int c : s.children[g])
        if (b->tup[c].send) f.insert(f.end(), b->flows[c].begin(), b->flows[c].end());
    }
    if (!t.kern && !t.act && t.recv && t.send && f.size() == 1 && g != s.root) {
      rp.store[g] = 1;
      rp.src[g] = f;
      f = {{Flow::kAgg, g}};
    }
    b->flows[g] = f;
  }
  return rp;
}

// send_bias: byte offset of the tree's block inside every rank's sendbuf
// (ReduceScatter block b); root_only: the result goes to the root's recvbuf
// only (Reduce, ReduceScatter) instead of every rank (AllReduce).
void plan_allreduce_tree(Builder& B, const SubColl& s, uint64_t lo, uint64_t hi, uint64_t mask,
                         bool accumulate, Mode mode, int64_t send_bias = 0, bool root_only = false,
                         bool late_join = false) {
  const int n = B.n_;
  const int es = B.esize_;
  const uint32_t ce = B.chunk_elems(s.chunk);
  const uint32_t nch = (uint32_t)((hi - lo + ce - 1) / ce);
  const uint64_t len = (hi - lo) * es;
  TreeBehavior b = tree_behavior(s, mask);
  const RelayPlan rp = store_relays(s, &b);
  const int root = s.root;

  // sources folded at the root (kernel) or its single flow (no kernel)
  std::vector<Flow> root_src =
      b.tup[root].kern ? kernel_sources(s, b, root) : b.flows[root];
  const bool zero = root_src.empty();
  if (zero && accumulate && !late_join) return;  // recvbuf untouched (reading Q7)

  std::vector<BufRef> recv_all;
  for (int g = 0; g < n; ++g)
    if ((!root_only || g == s.root) && B.alive(g)) recv_all.push_back(make_ref(kBufRecv, g, 0, accumulate));

  if (mode == kDirect) {
    std::map<int, std::pair<uint64_t, FlagRef>> agg_slot;  // kernel node -> slot
    auto stream_of = [&](const Flow& f) {
      if (f.kind == Flow::kIn) { Stream st; st.ref = make_ref(kBufSend, f.rank, send_bias); return st; }
      auto& as = agg_slot.at(f.rank);
      return B.slot_stream(f.rank, as.first, lo, &as.second);
    };
    for (int k : b.postorder) {
      if (!(b.tup[k].kern || rp.store[k]) || k == root) continue;
      uint64_t off = B.alloc(k, len);
      FlagRef fl = B.alloc_flags(k, nch);
      agg_slot[k] = {off, fl};
      std::vector<Stream> srcs;
      for (auto& f : rp.store[k] ? rp.src[k] : kernel_sources(s, b, k)) srcs.push_back(stream_of(f));
      B.add(k, lo, hi, ce, kOpFold, srcs,
            {make_ref(kBufArena, k, (int64_t)off - (int64_t)(lo * es))}, {fl});
    }
    std::vector<Stream> srcs;
    for (auto& f : root_src) srcs.push_back(stream_of(f));
    // late join: every non-ready rank is an optional source of the
    // root's fold, included per piece if it became ready in time
    std::vector<BufRef> late;
    if (late_join)
      for (int g = 0; g < n; ++g)
        if (!((mask >> g) & 1) && B.alive(g)) late.push_back(make_ref(kBufSend, g, send_bias));
    B.add(root, lo, hi, ce, zero ? kOpZero : kOpFold, srcs, recv_all, {}, late);
    return;
  }

  // STAGED: consumers and their landing slots
  struct Dest { int rank; uint64_t off; FlagRef flag; };
  std::map<std::pair<int, int>, Dest> dest_of;  // (flow kind, rank) -> landing at consumer
  std::map<int, std::vector<Stream>> consumer_srcs;
  std::vector<int> consumers;
  for (int k : b.postorder)
    if ((b.tup[k].kern || rp.store[k]) && k != root) consumers.push_back(k);
  consumers.push_back(root);
  for (int c : consumers) {
    const std::vector<Flow> L = (c == root) ? root_src : rp.store[c] ? rp.src[c] : kernel_sources(s, b, c);
    std::vector<Stream> srcs;
    for (const Flow& f : L) {
      if (f.kind == Flow::kIn && f.rank == c) {
        Stream st;
        st.ref = make_ref(kBufSend, c, send_bias);
        srcs.push_back(st);
        continue;
      }
      uint64_t off = B.alloc(c, len);
      FlagRef fl = B.alloc_flags(c, nch);
      dest_of[{(int)f.kind, f.rank}] = {c, off, fl};
      srcs.push_back(B.slot_stream(c, off, lo, &fl));
    }
    consumer_srcs[c] = std::move(srcs);
  }
  // pushes of ready ranks' own tensors (leaves, a=0 nodes, relayed flows)
  for (auto& kv : dest_of) {
    if (kv.first.first != Flow::kIn) continue;
    const int r = kv.first.second;
    const Dest& d = kv.second;
    Stream src;
    src.ref = make_ref(kBufSend, r, send_bias);
    B.add(r, lo, hi, ce, kOpFold, {src},
          {make_ref(kBufArena, d.rank, (int64_t)d.off - (int64_t)(lo * es))}, {d.flag});
  }
  // aggregation kernels (post-order: producers first)
  for (int k : consumers) {
    if (k == root) continue;
    const Dest& d = dest_of.at({(int)Flow::kAgg, k});
    B.add(k, lo, hi, ce, kOpFold, consumer_srcs[k],
          {make_ref(kBufArena, d.rank, (int64_t)d.off - (int64_t)(lo * es))}, {d.flag});
  }
  // late join (NEXT-1) on the STAGED protocol: every non-ready live
  // rank pushes its own chunk straight into a landing slot at the root -- iff
  // it is ready by then (phase 1) / iff it did not in phase 1 (phase 2) -- and
  // says so in the slot's per-chunk decision word; a non-ready root folds its
  // own input when its ready word allows (reading R4: late inputs join at the
  // root, after the regular terms, ascending rank)
  std::vector<BufRef> late_refs;
  std::vector<FlagRef> late_waits;
  if (late_join) {
    for (int g = 0; g < n; ++g) {
      if (((mask >> g) & 1) || !B.alive(g)) continue;
      if (g == root) {
        late_refs.push_back(make_ref(kBufSend, g, send_bias));
        continue;
      }
      const uint64_t off = B.alloc_dec(root, len, nch);
      const FlagRef fl = B.alloc_flags(root, nch);
      const BufRef slot = make_ref(kBufArena, root, (int64_t)off - (int64_t)(lo * es));
      Stream src;
      src.ref = make_ref(kBufSend, g, send_bias);
      B.add(g, lo, hi, ce, kOpFold, {src}, {slot}, {fl}, {}, {}, kLatePush);
      late_refs.push_back(slot);
      late_waits.push_back(fl);
    }
  }
  // root hand-off: own recvbuf + broadcast slot
  std::map<int, std::pair<uint64_t, FlagRef>> down;
  auto add_down_dst = [&](int g, std::vector<BufRef>* dsts, std::vector<FlagRef>* posts) {
    if (s.children[g].empty()) return;
    uint64_t off = late_join ? B.alloc_dec(g, len, nch) : B.alloc(g, len);
    FlagRef fl = B.alloc_flags(g, nch);
    down[g] = {off, fl};
    dsts->push_back(make_ref(kBufArena, g, (int64_t)off - (int64_t)(lo * es)));
    posts->push_back(fl);
  };
  {
    std::vector<BufRef> dsts = {make_ref(kBufRecv, root, 0, accumulate)};
    std::vector<FlagRef> posts;
    if (!root_only) add_down_dst(root, &dsts, &posts);
    B.add(root, lo, hi, ce, zero ? kOpZero : kOpFold, consumer_srcs[root], dsts, posts, late_refs, late_waits,
          late_join ? kLateRoot : kLateNone);
  }
  if (root_only) return;
  // broadcast down the reversed tree, parents before children
  for (int g : bfs_order(s)) {
    if (g == root || !B.alive(g)) continue;  // excluded ranks are leaves (check_members)
    const int p = s.parent[g];
    auto& pd = down.at(p);
    std::vector<Stream> srcs = {B.slot_stream(p, pd.first, lo, &pd.second)};
    std::vector<BufRef> dsts = {make_ref(kBufRecv, g, 0, accumulate)};
    std::vector<FlagRef> posts;
    add_down_dst(g, &dsts, &posts);
    B.add(g, lo, hi, ce, kOpFold, srcs, dsts, posts, {}, {}, late_join ? kLatePull : kLateNone);
  }
}

// ----------------------------------------------------------------- NVLS
// An nvls sub-collective (NEXT-2; the NVSwitch as the aggregation point --
// the B200 counterpart of the paper's switch / NIC nodes of the communication
// graph): every rank copies its partition into its multicast-bound
// scratch (one flag per slice owner), slice owner k sums slice k over all
// ranks' copies in the switch and stores the sum to all of them at once
// (multimem ld_reduce + st, one flag to every rank), and every rank copies
// the sums out to its recvbuf.  Per GPU and direction ~S crosses NVLink
// instead of 2(n-1)/n S for P2P trees.  The switch sums every rank's copy,
// so it needs the whole mask; the sub-16-byte tail of the last partition
// goes through a star tree at rank 0.
void plan_nvls(Builder& B, const SubColl& s, uint64_t lo, uint64_t hi, uint64_t mask, bool accumulate, Mode mode,
               bool late_join, std::string* unsupported) {
  const int n = B.n_;
  const int es = B.esize_;
  const uint64_t all = n >= 64 ? ~uint64_t(0) : ((uint64_t(1) << n) - 1);
  if (B.nvls_cap_ == 0) { *unsupported = "nvls line without NVLS scratch (adapcc_nvls_setup)"; return; }
  if ((mask & all) != all || B.members_ != all) {
    *unsupported = "nvls lines reduce every rank's copy: the whole mask is required";
    return;
  }
  if (late_join) { *unsupported = "late join on nvls lines"; return; }
  const uint64_t unit = 16 / es;
  const uint64_t hal = lo + (hi - lo) / unit * unit;
  if (hal < hi) {  // ragged tail: a star tree rooted at rank 0
    SubColl star;
    star.kind = kTree;
    star.weight = 1;
    star.chunk = s.chunk;
    star.parent.assign(n, 0);
    star.parent[0] = -1;
    star.root = 0;
    star.children.assign(n, {});
    for (int g = 1; g < n; ++g) star.children[0].push_back(g);
    plan_allreduce_tree(B, star, hal, hi, mask, accumulate, mode, 0, false, false);
  }
  if (hal <= lo) return;
  const uint64_t L = hal - lo, bytes = L * es;
  const uint64_t in_off = B.nvls_alloc(bytes), out_off = B.nvls_alloc(bytes);
  const int64_t in_bias = (int64_t)in_off - (int64_t)(lo * es), out_bias = (int64_t)out_off - (int64_t)(lo * es);
  const uint32_t ce = std::max<uint32_t>((uint32_t)unit, B.chunk_elems(s.chunk) / (uint32_t)unit * (uint32_t)unit);
  const uint64_t units = L / unit;
  for (int k = 0; k < n; ++k) {  // slice k: reduced by rank k
    const uint64_t a = lo + units * k / n * unit, b = lo + units * (k + 1) / n * unit;
    if (a >= b) continue;
    const uint32_t nch = (uint32_t)((b - a + ce - 1) / ce);
    std::vector<FlagRef> fin(n), fout(n);
    for (int q = 0; q < n; ++q) {
      fin[q] = B.alloc_flags(k, nch);   // "rank q copied slice k in", at rank k
      fout[q] = B.alloc_flags(q, nch);  // "slice k is summed", at rank q
    }
    for (int q = 0; q < n; ++q) {
      Stream src;
      src.ref = make_ref(kBufSend, q, 0);
      B.add(q, a, b, ce, kOpFold, {src}, {make_ref(kBufNvlsUc, q, in_bias)}, {fin[q]});
    }
    std::vector<Stream> waits;
    for (int q = 0; q < n; ++q) {
      Stream w;
      w.ref = make_ref(kBufNvlsMc, k, in_bias);
      w.wait = true;
      w.flag = fin[q];
      waits.push_back(w);
    }
    // one source stream (the multicast input), waited for through n flags
    B.add_multiwait(k, a, b, ce, kOpNvls, waits, {make_ref(kBufNvlsMc, k, out_bias)}, fout);
    for (int q = 0; q < n; ++q) {
      Stream src;
      src.ref = make_ref(kBufNvlsUc, q, out_bias);
      src.wait = true;
      src.flag = fout[q];
      B.add(q, a, b, ce, kOpFold, {src}, {make_ref(kBufRecv, q, 0, accumulate)}, {});
    }
  }
  B.p_.nvls = true;
}

// ------------------------------------------------------------- AllGather
// slot_bias < 0: AllGather (source s lands in slot s of every recvbuf);
// otherwise Broadcast (lands at that byte offset).
void plan_allgather_tree(Builder& B, const SubColl& s, uint64_t lo, uint64_t hi, uint64_t cnt,
                         uint64_t mask, Mode mode, int64_t slot_bias_override = -1) {
  const int n = B.n_;
  const int es = B.esize_;
  const int src = s.src;
  if (!((mask >> src) & 1)) return;  // non-ready source: slots untouched (Q12)
  const uint32_t ce = B.chunk_elems(s.chunk);
  const uint32_t nch = (uint32_t)((hi - lo + ce - 1) / ce);
  const uint64_t len = (hi - lo) * es;
  const int64_t slot_bias = slot_bias_override >= 0 ? slot_bias_override : (int64_t)(src * cnt * es);
  Stream in;
  in.ref = make_ref(kBufSend, src, 0);
  if (mode == kDirect) {
    std::vector<BufRef> dsts;
    for (int g = 0; g < n; ++g)
      if (B.alive(g)) dsts.push_back(make_ref(kBufRecv, g, slot_bias));
    B.add(src, lo, hi, ce, kOpFold, {in}, dsts, {});
    return;
  }
  std::map<int, std::pair<uint64_t, FlagRef>> down;
  for (int g : bfs_order(s)) {
    if (!B.alive(g)) continue;  // excluded ranks are leaves (check_members)
    std::vector<Stream> srcs;
    if (g == src) {
      srcs.push_back(in);
    } else {
      auto& pd = down.at(s.parent[g]);
      srcs.push_back(B.slot_stream(s.parent[g], pd.first, lo, &pd.second));
    }
    std::vector<BufRef> dsts = {make_ref(kBufRecv, g, slot_bias)};
    std::vector<FlagRef> posts;
    if (!s.children[g].empty()) {
      uint64_t off = B.alloc(g, len);
      FlagRef fl = B.alloc_flags(g, nch);
      down[g] = {off, fl};
      dsts.push_back(make_ref(kBufArena, g, (int64_t)off - (int64_t)(lo * es)));
      posts.push_back(fl);
    }
    B.add(g, lo, hi, ce, kOpFold, srcs, dsts, posts);
  }
}

// -------------------------------------------------------------- AlltoAll
// One flow ("each GPU sends multiple flows to all other GPUs") along
// its route src -> hops -> dst (routing variables x^f_ij, eq. 1).  Relays do
// not aggregate (a_{m,g} = 0 for primitives without aggregation), so
// every hop is chunk-pipelined store-and-forward, h_j = h_i + t_ij (eq. 2):
// the holder pushes the chunk into a landing slot in the next relay's arena
// and posts that chunk's flag.  The last holder writes the destination block
// (DIRECT) or pushes into a landing slot that the destination copies out
// (STAGED).
void plan_flow(Builder& B, int src, int dst, const std::vector<int>* hops, const Stream& in,
               const BufRef& out, uint64_t lo, uint64_t hi, uint32_t ce, Mode mode) {
  const int es = B.esize_;
  const uint32_t nch = (uint32_t)((hi - lo + ce - 1) / ce);
  const uint64_t len = (hi - lo) * es;
  Stream cur = in;
  int at = src;
  auto push = [&](int to) {
    const uint64_t off = B.alloc(to, len);
    const FlagRef fl = B.alloc_flags(to, nch);
    B.add(at, lo, hi, ce, kOpFold, {cur}, {make_ref(kBufArena, to, (int64_t)off - (int64_t)(lo * es))}, {fl});
    cur = B.slot_stream(to, off, lo, &fl);
    at = to;
  };
  if (hops)
    for (int h : *hops) push(h);
  if (mode == kStaged && at != dst) push(dst);
  B.add(at, lo, hi, ce, kOpFold, {cur}, {out}, {});
}

void plan_alltoall_line(Builder& B, const SubColl& s, uint64_t lo, uint64_t hi, uint64_t cnt,
                        uint64_t mask, Mode mode) {
  const int n = B.n_;
  const int es = B.esize_;
  const uint32_t ce = B.chunk_elems(s.chunk);
  for (int src = 0; src < n; ++src) {
    if (!((mask >> src) & 1)) continue;
    for (int d = 0; d < n; ++d) {
      if (!B.alive(d)) continue;
      Stream in;
      in.ref = make_ref(kBufSend, src, (int64_t)(d * cnt * es));
      plan_flow(B, src, d, s.hops(src, d), in, make_ref(kBufRecv, d, (int64_t)(src * cnt * es)), lo, hi,
                ce, mode);
    }
  }
}

// AlltoAllv: every (s, d) block has its own count; each block is split over
// the a2a lines by weight (Q9) and then into segment k of nseg.
void plan_alltoallv(Builder& B, const PlanRequest& rq, uint64_t k, uint64_t nseg) {
  const Strategy& st = *rq.st;
  const int n = st.nranks, es = rq.esize;
  const uint64_t unit = 16 / es;
  std::vector<int64_t> w;
  for (auto& s : st.subs) w.push_back(s.weight);
  for (int src = 0; src < n; ++src) {
    if (!((rq.ready_mask >> src) & 1)) continue;
    for (int d = 0; d < n; ++d) {
      const uint64_t c = rq.counts[(size_t)src * n + d];
      if (!c || !B.alive(d)) continue;
      uint64_t soff = 0, roff = 0;
      for (int j = 0; j < d; ++j) soff += rq.counts[(size_t)src * n + j];
      for (int j = 0; j < src; ++j) roff += rq.counts[(size_t)j * n + d];
      const auto b = partition(c, es, w);
      for (size_t m = 0; m < st.subs.size(); ++m) {
        const uint64_t step = align_up((b[m + 1] - b[m] + nseg - 1) / nseg, unit);
        const uint64_t lo = std::min(b[m + 1], b[m] + k * step), hi = std::min(b[m + 1], b[m] + (k + 1) * step);
        if (lo >= hi) continue;
        const SubColl& s = st.subs[m];
        Stream in;
        in.ref = make_ref(kBufSend, src, (int64_t)(soff * es));
        plan_flow(B, src, d, s.hops(src, d), in, make_ref(kBufRecv, d, (int64_t)(roff * es)), lo, hi,
                  B.chunk_elems(s.chunk), rq.mode);
      }
    }
  }
}

SegmentPlan build_units(const PlanRequest& rq, const std::vector<std::pair<uint64_t, uint64_t>>& ranges,
                        uint64_t seg_k, uint64_t nseg, uint64_t unit_cap);

SegmentPlan build_segment(const PlanRequest& rq,
                          const std::vector<std::pair<uint64_t, uint64_t>>& ranges, uint64_t seg_k,
                          uint64_t nseg) {
  const Strategy& st = *rq.st;
  // unit cap: about two flagged units per CTA over the call's bytes per rank
  // (x n ranks), 4 KiB-aligned, at least 16 KiB
  // and never above 1 MiB: one CTA moves a unit between flags, and larger
  // units serialise a chunk on one SM (measured: ring / double-binary trees
  // lose 40-60 % with 4 MiB units)
  uint64_t unit_cap = 0;
  if (rq.grid > 0) {
    unit_cap = uint64_t(1) << 20;
    if (!rq.counts) {
      const uint64_t per_rank = rq.count * (uint64_t)rq.esize *
                                ((st.coll == kAllToAll || st.coll == kAllGather || st.coll == kReduceScatter) ? st.nranks : 1);
      unit_cap = std::min(unit_cap, std::max<uint64_t>(16384, per_rank * st.nranks / (2ull * rq.grid) / 4096 * 4096));
    }
  }
  SegmentPlan p = build_units(rq, ranges, seg_k, nseg, unit_cap);
  // The cap only matters where units pipeline between flags.  A flag-free
  // plan (DIRECT star / AllGather / AlltoAll) keeps C_m: its work balance
  // comes from pieces (order_items), and capped units would only shrink them
  // (AlltoAll at 1 MiB per rank: 2 item rounds instead of 1, 5.4 -> 7.0 us).
  bool flagged = false;
  for (const Task& t : p.tasks) flagged |= t.nwait != 0 || t.npost != 0;
  if (!flagged && unit_cap) p = build_units(rq, ranges, seg_k, nseg, 0);
  return p;
}

SegmentPlan build_units(const PlanRequest& rq, const std::vector<std::pair<uint64_t, uint64_t>>& ranges,
                        uint64_t seg_k, uint64_t nseg, uint64_t unit_cap) {
  const Strategy& st = *rq.st;
  Builder B(st.nranks, rq.esize, rq.half_bytes, rq.members, unit_cap);
  B.nvls_cap_ = rq.nvls_bytes;
  if (rq.counts) {
    plan_alltoallv(B, rq, seg_k, nseg);
    return B.finish();
  }
  for (size_t m = 0; m < st.subs.size(); ++m) {
    const uint64_t lo = ranges[m].first, hi = ranges[m].second;
    if (lo >= hi) continue;
    const SubColl& s = st.subs[m];
    switch (st.coll) {
      case kAllReduce:
        if (s.kind == kNvls) plan_nvls(B, s, lo, hi, rq.ready_mask, rq.accumulate, rq.mode, rq.late_join, &B.p_.unsupported);
        else plan_allreduce_tree(B, s, lo, hi, rq.ready_mask, rq.accumulate, rq.mode, 0, false, rq.late_join);
        break;
      case kReduce: plan_allreduce_tree(B, s, lo, hi, rq.ready_mask, rq.accumulate, rq.mode, 0, true); break;
      case kReduceScatter:
        if (!B.alive(s.src)) break;  // block of an excluded rank: no destination
        plan_allreduce_tree(B, s, lo, hi, rq.ready_mask, rq.accumulate, rq.mode,
                            (int64_t)((uint64_t)s.src * rq.count * rq.esize), true);
        break;
      case kAllGather: plan_allgather_tree(B, s, lo, hi, rq.count, rq.ready_mask, rq.mode); break;
      case kBroadcast: plan_allgather_tree(B, s, lo, hi, rq.count, rq.ready_mask, rq.mode, 0); break;
      default: plan_alltoall_line(B, s, lo, hi, rq.count, rq.ready_mask, rq.mode); break;
    }
  }
  return B.finish();
}

}  // namespace

uint64_t flag_region_bytes(uint64_t half) {
  uint64_t f = half / 32 / 256 * 256;
  return std::min<uint64_t>(std::max<uint64_t>(f, 4096), uint64_t(32) << 20);
}

std::vector<std::pair<uint64_t, uint64_t>> sub_ranges(const Strategy& st, uint64_t count,
                                                      int esize) {
  std::vector<std::pair<uint64_t, uint64_t>> r(st.subs.size());
  if (st.coll == kAllGather || st.coll == kReduceScatter) {
    for (int src = 0; src < st.nranks; ++src) {
      std::vector<int64_t> w;
      std::vector<size_t> idx;
      for (size_t m = 0; m < st.subs.size(); ++m)
        if (st.subs[m].src == src) { w.push_back(st.subs[m].weight); idx.push_back(m); }
      auto b = partition(count, esize, w);
      for (size_t i = 0; i < idx.size(); ++i) r[idx[i]] = {b[i], b[i + 1]};
    }
    return r;
  }
  std::vector<int64_t> w;
  for (auto& s : st.subs) w.push_back(s.weight);
  auto b = partition(count, esize, w);
  for (size_t m = 0; m < st.subs.size(); ++m) r[m] = {b[m], b[m + 1]};
  return r;
}

bool build_plan(const PlanRequest& rq, std::vector<SegmentPlan>* segs, std::string* err) {
  segs->clear();
  const auto full = sub_ranges(*rq.st, rq.count, rq.esize);
  const uint64_t unit = 16 / rq.esize;
  for (uint64_t nseg = 1;; nseg *= 2) {
    std::vector<SegmentPlan> out;
    bool fits = true;
    uint64_t max_step = 0;
    for (uint64_t k = 0; k < nseg && fits; ++k) {
      std::vector<std::pair<uint64_t, uint64_t>> rr(full.size());
      for (size_t m = 0; m < full.size(); ++m) {
        const uint64_t lo = full[m].first, hi = full[m].second;
        const uint64_t step = align_up((hi - lo + nseg - 1) / nseg, unit);
        max_step = std::max(max_step, step);
        const uint64_t a = std::min(hi, lo + k * step), b = std::min(hi, lo + (k + 1) * step);
        rr[m] = {a, b};
      }
      SegmentPlan p = build_segment(rq, rr, k, nseg);
      if (!p.unsupported.empty()) {
        if (err) *err = "unsupported: " + p.unsupported;
        return false;
      }
      if (rq.counts) {
        uint64_t cmax = 0;
        const int n = rq.st->nranks;
        for (int i = 0; i < n * n; ++i) cmax = std::max<uint64_t>(cmax, rq.counts[i]);
        max_step = std::max(max_step, align_up((cmax + nseg - 1) / nseg, unit));
      }
      fits = fits && p.fits;
      if (!p.tasks.empty()) out.push_back(std::move(p));
    }
    if (fits) {
      *segs = std::move(out);
      return true;
    }
    if (max_step <= unit) {  // cannot split further
      if (err) *err = "scratch arena too small for this strategy";
      return false;
    }
  }
}

std::vector<Item> order_items(const SegmentPlan& p, int rank, int esize, int grid,
                              uint64_t piece_bytes, int taper, bool tma, bool acc_red) {
  // Work balance: tasks that post no flags are cut into pieces of roughly
  // equal traffic.
  // streams of a task: sources + destinations, an accumulating destination
  // twice (recv is read and written)
  auto streams_of = [&](const Task& T) {
    uint64_t s = (uint64_t)T.nsrc + T.ndst;
    for (uint32_t k = 0; k < T.ndst; ++k) s += p.refs[T.ref0 + T.nsrc + k].accum ? 1 : 0;
    return std::max<uint64_t>(1, s);
  };
  uint64_t total = 0;
  for (const Task& T : p.tasks)
    if (rank < 0 || T.owner == rank) total += (T.hi - T.lo) * esize * streams_of(T);
  // Measured on B200 (profiles/sweep_r01.json, profiles/pieces_r01.json):
  // ~512 KiB of traffic per item (32 KiB per stream for a 16-stream fold) is
  // the sweet spot of large calls -- smaller items pay the per-item claim/sync
  // overhead, larger ones lose bandwidth.
  // Pieces are sized so that every CTA gets the same number m of items: a
  // CTA streams a piece at a roughly fixed rate, so a call ends when the CTA
  // with the most items does (8 MiB per rank, TMA: 1.7 items per CTA left half
  // the grid idle for a whole item at the end).
  const uint64_t g = (uint64_t)std::max(grid, 1);
  // Phase 2 by bulk reduce-adds (acc_red) streams best at ~256 KiB per item
  // (16 / 25 / 64 / 100 / 256 MiB per rank: +0.2 / +1.0 / +1.5 / +1.5 / +1.3 %
  // with the taper below, profiles/acc_pieces_r02.json)
  const uint64_t cap = acc_red ? 256 * 1024 : 512 * 1024, floor_bytes = tma ? 256 * 1024 : 16 * 1024;
  const uint64_t m = std::max<uint64_t>(1, (total + g * cap - 1) / (g * cap));
  const uint64_t target =
      piece_bytes ? piece_bytes : std::min<uint64_t>(std::max<uint64_t>(total / (m * g), floor_bytes), cap);
  const uint64_t align = 512;  // elements: keeps every piece 16-byte aligned
  struct Key { uint64_t a; uint32_t level, task, chunk, off, len; };
  std::vector<Key> keys;
  // Claim order: key (chunk + level x lag).  Any lag >= 1 claims an item after
  // the same chunk's items one level down (its only dependencies), which keeps
  // the persistent grid deadlock-free.  The lag spaces a dependency about two
  // in-flight windows (grid x queue depth) ahead of its consumer, so a claimed
  // item rarely waits: lag = ceil(2 x grid / items per (chunk, level)).
  uint64_t lag = 1;
  for (uint32_t t = 0; t < p.tasks.size(); ++t) {
    const Task& T = p.tasks[t];
    if (rank >= 0 && T.owner != rank) continue;
    const uint64_t streams = streams_of(T);
    for (uint32_t c = 0; c < T.nchunks; ++c) {
      const uint64_t c0 = T.lo + (uint64_t)c * T.chunk_elems;
      const uint64_t clen = std::min<uint64_t>(T.hi, c0 + T.chunk_elems) - c0;
      // a flag-free chunk is cut into at most floor(traffic / target) equal
      // pieces of >= `target` bytes: with target = total / grid a mid-size
      // call then has at most one item per CTA (measured: 304 items of 14 KiB
      // per stream on 296 CTAs 14.9 us, 256 items of 16 KiB 10.5 us)
      uint64_t piece = clen;
      if (T.npost == 0) {
        const uint64_t cnt = std::max<uint64_t>(1, clen * streams * esize / target);
        piece = std::max<uint64_t>(align, ((clen + cnt - 1) / cnt + align - 1) / align * align);
      }
      for (uint64_t off = 0; off < clen; off += piece)
        keys.push_back({(uint64_t)c, T.level, t, c, (uint32_t)off,
                        (uint32_t)std::min<uint64_t>(piece, clen - off)});
    }
  }
  if (p.max_level > 0 && !keys.empty()) {
    std::vector<uint64_t> chunks_at(p.max_level + 1, 0);
    for (const Key& k : keys) chunks_at[k.level] = std::max<uint64_t>(chunks_at[k.level], (uint64_t)k.chunk + 1);
    uint64_t slots = 0;
    for (uint64_t v : chunks_at) slots += v;
    const uint64_t per = std::max<uint64_t>(1, keys.size() / std::max<uint64_t>(1, slots));
    lag = std::max<uint64_t>(1, (2ull * std::max(grid, 1) + per - 1) / per);
  }
  for (Key& k : keys) k.a = (uint64_t)k.chunk + (uint64_t)k.level * lag;
  std::sort(keys.begin(), keys.end(), [](const Key& x, const Key& y) {
    return std::tie(x.a, x.level, x.task, x.chunk, x.off) <
           std::tie(y.a, y.level, y.task, y.chunk, y.off);
  });
  // Tail taper: CTAs claim items dynamically, so a launch ends when its last
  // items finish; with uniform pieces the grid idles for about half an item
  // at the end.  The last ~2 x grid items of flag-free tasks are cut into
  // `taper` consecutive sub-pieces (same key position, so the claim order
  // stays topological: sub-pieces wait on the same flags and post none).
  // taper 0 = automatic: halve only items of >= 384 KiB of traffic (measured,
  // profiles/taper_*_r01.json: +1-3 % from 16 MiB per rank up, where pieces
  // are 448-512 KiB; halving ~110-230 KiB pieces costs more in per-item
  // overhead than the shorter tail saves).
  // Automatic taper only from m >= 3 items per CTA: with one or two balanced
  // rounds the last round is already even, and halving its items only adds
  // per-item overhead (8 MiB per rank, m = 2: 26.3 us tapered, 24.8 us not;
  // 16 MiB, m = 4: 46.0 vs 46.3 us, profiles/ab/taper_r01.txt).
  bool auto_taper = taper <= 0;
  if (auto_taper) taper = (piece_bytes || m >= 3 || acc_red) ? 2 : 1;
  if (auto_taper && acc_red) auto_taper = false;  // (its 256 KiB items are all halved, whatever their size)
  std::vector<uint8_t> split(keys.size(), 0);
  if (taper > 1) {
    uint64_t want = 2ull * std::max(grid, 1);
    for (size_t i = keys.size(); i-- > 0 && want > 0;) {
      const Task& T = p.tasks[keys[i].task];
      if (T.npost != 0 || keys[i].len < (uint64_t)taper * align) continue;
      if (auto_taper && (uint64_t)keys[i].len * esize * streams_of(T) < (384u << 10)) continue;
      split[i] = 1;
      --want;
    }
  }
  std::vector<Item> items;
  items.reserve(keys.size());
  for (size_t i = 0; i < keys.size(); ++i) {
    const Key& k = keys[i];
    if (!split[i]) {
      items.push_back({k.task, k.chunk, k.off, k.len});
      continue;
    }
    const uint32_t sub = (uint32_t)((k.len + (uint64_t)taper * align - 1) / ((uint64_t)taper * align) * align);
    for (uint32_t o = 0; o < k.len; o += sub)
      items.push_back({k.task, k.chunk, k.off + o, std::min<uint32_t>(sub, k.len - o)});
  }
  return items;
}

void accumulate_stats(const SegmentPlan& p, int rank, int esize, PlanStats* s) {
  for (const Task& t : p.tasks) {
    if (rank >= 0 && t.owner != rank) continue;
    const uint64_t bytes = (t.hi - t.lo) * esize;
    s->tasks += 1;
    s->items += t.nchunks;
    s->levels = std::max<uint64_t>(s->levels, t.level + 1);
    for (int i = 0; i < t.nsrc; ++i) {
      const BufRef& r = p.refs[t.ref0 + i];
      s->bytes_read += bytes;
      if (r.rank != t.owner) s->remote_bytes += bytes;
    }
    for (int i = 0; i < t.ndst; ++i) {
      const BufRef& r = p.refs[t.ref0 + t.nsrc + i];
      s->bytes_written += bytes;
      if (r.accum) s->bytes_read += bytes;
      if (r.rank != t.owner) s->remote_bytes += bytes * (r.accum ? 2 : 1);
    }
  }
  for (uint64_t u : p.arena_used) s->arena_bytes = std::max(s->arena_bytes, u);
}

}  // namespace adapcc
