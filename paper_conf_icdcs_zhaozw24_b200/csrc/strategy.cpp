// Strategy text loader and tree behaviour (product side; see strategy.hpp).
#include "strategy.hpp"

#include <algorithm>
#include <cstring>
#include <map>

namespace adapcc {
namespace {

bool is_space(char c) { return c == ' ' || c == '\t' || c == '\r' || c == '\v' || c == '\f'; }

std::vector<std::string> split_ws(const std::string& s) {
  std::vector<std::string> out;
  size_t i = 0;
  while (i < s.size()) {
    while (i < s.size() && is_space(s[i])) ++i;
    size_t j = i;
    while (j < s.size() && !is_space(s[j])) ++j;
    if (j > i) out.emplace_back(s.substr(i, j - i));
    i = j;
  }
  return out;
}

// Integer grammar -?[0-9]+ (DESIGN.md §2); rejects overflow past 2^62.
bool parse_int(const std::string& t, int64_t* v) {
  size_t i = 0;
  bool neg = false;
  if (i < t.size() && t[i] == '-') { neg = true; ++i; }
  if (i == t.size()) return false;
  int64_t acc = 0;
  for (; i < t.size(); ++i) {
    if (t[i] < '0' || t[i] > '9') return false;
    if (acc > (int64_t(1) << 58)) return false;
    acc = acc * 10 + (t[i] - '0');
  }
  *v = neg ? -acc : acc;
  return true;
}

bool parse_list(const std::string& t, std::vector<int64_t>* out) {
  out->clear();
  if (t.empty()) return true;
  size_t a = 0;
  while (true) {
    size_t b = t.find(',', a);
    std::string tok = t.substr(a, b == std::string::npos ? std::string::npos : b - a);
    int64_t v;
    if (!parse_int(tok, &v)) return false;
    out->push_back(v);
    if (b == std::string::npos) break;
    a = b + 1;
  }
  return true;
}

bool fail(std::string* err, const std::string& msg) {
  if (err) *err = msg;
  return false;
}

// Tree checks: n entries, one root, parents in range, no self loop, acyclic.
bool check_tree(const std::vector<int64_t>& p, int n, std::string* err) {
  if ((int)p.size() != n) return fail(err, "parent list length != nranks");
  int roots = 0;
  for (int g = 0; g < n; ++g) {
    if (p[g] == -1) { ++roots; continue; }
    if (p[g] < 0 || p[g] >= n) return fail(err, "parent out of range");
    if (p[g] == g) return fail(err, "self loop in tree");
  }
  if (roots != 1) return fail(err, "tree needs exactly one root");
  // colour walk: 0 = unknown, 1 = on current path, 2 = reaches root
  std::vector<int> state(n, 0);
  for (int g = 0; g < n; ++g) {
    std::vector<int> path;
    int x = g;
    while (x != -1 && state[x] == 0) {
      state[x] = 1;
      path.push_back(x);
      x = (int)p[x];
    }
    if (x != -1 && state[x] == 1) return fail(err, "cycle in tree");
    for (int y : path) state[y] = 2;
  }
  return true;
}

void finish_tree(SubColl* s, int n) {
  s->children.assign(n, {});
  for (int g = 0; g < n; ++g) {
    if (s->parent[g] == -1) s->root = g;
    else s->children[s->parent[g]].push_back(g);  // g ascending => children ascending
  }
}

// route=<s>:<d>:<h1>,<h2>,..[;<s>:<d>:<h>,..]: each entry is one
// flow's path (eq. 1: leaves src, enters dst, conserved at every relay).
bool parse_routes(const std::string& v, int n, std::vector<Route>* out, std::string* err) {
  size_t a = 0;
  while (true) {
    size_t b = v.find(';', a);
    const std::string ent = v.substr(a, b == std::string::npos ? std::string::npos : b - a);
    const size_t c1 = ent.find(':');
    const size_t c2 = c1 == std::string::npos ? c1 : ent.find(':', c1 + 1);
    if (c2 == std::string::npos) return fail(err, "route entry must be src:dst:hops");
    int64_t sv = 0, dv = 0;
    std::vector<int64_t> hv;
    if (!parse_int(ent.substr(0, c1), &sv) || !parse_int(ent.substr(c1 + 1, c2 - c1 - 1), &dv) ||
        !parse_list(ent.substr(c2 + 1), &hv))
      return fail(err, "bad route entry");
    if (sv < 0 || sv >= n || dv < 0 || dv >= n) return fail(err, "route rank out of range");
    if (sv == dv) return fail(err, "route src == dst");
    if (hv.empty()) return fail(err, "route needs at least one relay");
    Route r;
    r.src = (int)sv;
    r.dst = (int)dv;
    uint64_t seen = (uint64_t(1) << sv) | (uint64_t(1) << dv);
    for (int64_t h : hv) {
      if (h < 0 || h >= n) return fail(err, "route relay out of range");
      if ((seen >> h) & 1) return fail(err, "route visits a rank twice");
      seen |= uint64_t(1) << h;
      r.hops.push_back((int)h);
    }
    for (const Route& o : *out)
      if (o.src == r.src && o.dst == r.dst) return fail(err, "two routes for one flow");
    out->push_back(std::move(r));
    if (b == std::string::npos) break;
    a = b + 1;
  }
  std::sort(out->begin(), out->end(), [](const Route& x, const Route& y) {
    return x.src != y.src ? x.src < y.src : x.dst < y.dst;
  });
  return true;
}

uint64_t fnv1a(const std::string& s) {
  uint64_t h = 1469598103934665603ull;
  for (unsigned char c : s) { h ^= c; h *= 1099511628211ull; }
  return h;
}

}  // namespace

bool parse_strategy(const char* text, Strategy* out, std::string* err) {
  if (!text) return fail(err, "null strategy text");
  // 1. logical lines without comments and surrounding blanks
  std::vector<std::vector<std::string>> lines;
  std::string norm;
  {
    const char* p = text;
    while (*p) {
      const char* e = p;
      while (*e && *e != '\n') ++e;
      std::string line(p, e - p);
      size_t hash = line.find('#');
      if (hash != std::string::npos) line.resize(hash);
      auto toks = split_ws(line);
      if (!toks.empty()) {
        for (auto& t : toks) { norm += t; norm += ' '; }
        norm += '\n';
        lines.push_back(std::move(toks));
      }
      p = *e ? e + 1 : e;
    }
  }
  if (lines.empty() || lines[0].size() != 2 || lines[0][0] != "adapcc-strategy" ||
      lines[0][1] != "1")
    return fail(err, "first line must be 'adapcc-strategy 1'");

  int n = -1;
  int coll = -1;
  struct Raw { std::string head; std::map<std::string, std::string> kv; };
  std::vector<Raw> raws;
  for (size_t li = 1; li < lines.size(); ++li) {
    const auto& t = lines[li];
    if (t[0] == "nranks") {
      int64_t v;
      if (n != -1 || t.size() != 2 || !parse_int(t[1], &v)) return fail(err, "bad nranks line");
      if (v < 1 || v > kMaxRanks) return fail(err, "nranks out of range");
      n = (int)v;
      continue;
    }
    if (t[0] == "collective") {
      if (coll != -1 || t.size() != 2) return fail(err, "bad collective line");
      if (t[1] == "allreduce") coll = kAllReduce;
      else if (t[1] == "allgather") coll = kAllGather;
      else if (t[1] == "alltoall") coll = kAllToAll;
      else if (t[1] == "reduce") coll = kReduce;
      else if (t[1] == "broadcast") coll = kBroadcast;
      else if (t[1] == "reducescatter") coll = kReduceScatter;
      else return fail(err, "unknown collective");
      continue;
    }
    if (t[0] != "tree" && t[0] != "ring" && t[0] != "bcast" && t[0] != "a2a" && t[0] != "rtree" && t[0] != "nvls")
      return fail(err, "unknown directive " + t[0]);
    Raw r;
    r.head = t[0];
    for (size_t k = 1; k < t.size(); ++k) {
      size_t eq = t[k].find('=');
      if (eq == std::string::npos) return fail(err, "expected key=value");
      std::string key = t[k].substr(0, eq);
      if (r.kv.count(key)) return fail(err, "repeated key " + key);
      r.kv[key] = t[k].substr(eq + 1);
    }
    raws.push_back(std::move(r));
  }
  if (n == -1 || coll == -1) return fail(err, "missing nranks or collective");
  if (raws.empty()) return fail(err, "no sub-collective lines");

  Strategy st;
  st.nranks = n;
  st.coll = (Coll)coll;
  for (const Raw& r : raws) {
    const bool ok_kind = (coll == kAllReduce && (r.head == "tree" || r.head == "ring" || r.head == "nvls")) ||
                         (coll == kAllGather && r.head == "bcast") ||
                         (coll == kAllToAll && r.head == "a2a") ||
                         (coll == kReduce && r.head == "tree") ||
                         (coll == kBroadcast && r.head == "bcast") ||
                         (coll == kReduceScatter && r.head == "rtree");
    if (!ok_kind) return fail(err, "directive " + r.head + " not valid for this collective");
    std::vector<std::string> required = {"weight", "chunk"};
    std::vector<std::string> optional;
    if (r.head == "tree") { required.push_back("parent"); optional.push_back("noagg"); optional.push_back("relay"); }
    if (r.head == "rtree") { required.push_back("parent"); required.push_back("dst"); optional.push_back("noagg"); }
    if (r.head == "ring") required.push_back("order");
    if (r.head == "bcast") { required.push_back("parent"); required.push_back("src"); }
    if (r.head == "a2a") optional.push_back("route");
    for (auto& k : required)
      if (!r.kv.count(k)) return fail(err, r.head + ": missing key " + k);
    for (auto& kv : r.kv) {
      bool known = std::find(required.begin(), required.end(), kv.first) != required.end() ||
                   std::find(optional.begin(), optional.end(), kv.first) != optional.end();
      if (!known) return fail(err, r.head + ": unknown key " + kv.first);
    }
    int64_t w, c;
    if (!parse_int(r.kv.at("weight"), &w)) return fail(err, "bad weight");
    if (!parse_int(r.kv.at("chunk"), &c)) return fail(err, "bad chunk");
    if (w < 0 || w > kMaxWeight) return fail(err, "weight out of range");
    if (c < 16 || c % 16 != 0 || c > kMaxChunk) return fail(err, "chunk must be a multiple of 16 in [16, 2^31]");

    if (r.head == "ring") {
      std::vector<int64_t> order;
      if (!parse_list(r.kv.at("order"), &order)) return fail(err, "bad ring order");
      std::vector<int64_t> sorted = order;
      std::sort(sorted.begin(), sorted.end());
      bool perm = (int)sorted.size() == n;
      for (int i = 0; perm && i < n; ++i) perm = sorted[i] == i;
      if (!perm) return fail(err, "ring order must be a permutation of 0..n-1");
      // reading Q13: chain m has root order[m], leaf order[m+1]
      for (int m = 0; m < n; ++m) {
        SubColl s;
        s.kind = kTree;
        s.weight = w;
        s.chunk = c;
        s.parent.assign(n, -1);
        for (int j = 1; j < n; ++j)
          s.parent[order[(m + j) % n]] = (int)order[(m + j + 1) % n];
        s.parent[order[m]] = -1;
        finish_tree(&s, n);
        st.subs.push_back(std::move(s));
      }
      continue;
    }
    SubColl s;
    s.weight = w * n;
    s.chunk = c;
    if (r.head == "nvls") {  // the switch reduces and multicasts: no graph to give
      s.kind = kNvls;
      st.subs.push_back(std::move(s));
      continue;
    }
    if (r.head == "a2a") {
      s.kind = kA2A;
      if (r.kv.count("route") && !parse_routes(r.kv.at("route"), n, &s.routes, err)) return false;
      st.subs.push_back(std::move(s));
      continue;
    }
    std::vector<int64_t> parent;
    if (!parse_list(r.kv.at("parent"), &parent)) return fail(err, "bad parent list");
    if (!check_tree(parent, n, err)) return false;
    s.parent.assign(parent.begin(), parent.end());
    finish_tree(&s, n);
    if (r.head == "tree" || r.head == "rtree") {
      s.kind = r.head == "tree" ? kTree : kRTree;
      if (s.kind == kRTree) {
        int64_t dst;
        if (!parse_int(r.kv.at("dst"), &dst) || dst < 0 || dst >= n) return fail(err, "bad rtree dst");
        if (s.root != dst) return fail(err, "rtree root must be its dst");
        s.src = (int)dst;
      }
      if (r.kv.count("relay")) {
        const std::string& v = r.kv.at("relay");
        if (v != "store" && v != "bypass") return fail(err, "relay must be store or bypass");
        s.relay_store = v == "store";
      }
      if (r.kv.count("noagg")) {
        std::vector<int64_t> na;
        if (!parse_list(r.kv.at("noagg"), &na)) return fail(err, "bad noagg list");
        for (int64_t g : na) {
          if (g < 0 || g >= n) return fail(err, "noagg rank out of range");
          if (s.noagg >> g & 1) return fail(err, "duplicate noagg rank");
          if (g == s.root) return fail(err, "noagg may not contain the root");
          s.noagg |= uint64_t(1) << g;
        }
      }
    } else {
      s.kind = kBcast;
      int64_t src;
      if (!parse_int(r.kv.at("src"), &src) || src < 0 || src >= n) return fail(err, "bad bcast src");
      if (s.root != src) return fail(err, "bcast root must be its src");
      s.src = (int)src;
    }
    st.subs.push_back(std::move(s));
  }
  if ((int)st.subs.size() > kMaxSubs) return fail(err, "too many sub-collectives");
  if (coll == kAllGather || coll == kReduceScatter) {
    for (int src = 0; src < n; ++src) {
      int64_t tot = 0;
      int lines_for_src = 0;
      for (auto& s : st.subs)
        if (s.src == src) { tot += s.weight; ++lines_for_src; }
      if (lines_for_src == 0 || tot == 0) return fail(err, "block without a positive-weight line");
    }
  } else {
    for (auto& s : st.subs) {
      if (coll == kReduce && s.root != st.subs[0].root) return fail(err, "reduce trees must share one root");
      if (coll == kBroadcast && s.src != st.subs[0].src) return fail(err, "broadcast lines must share one src");
    }
    int64_t tot = 0;
    for (auto& s : st.subs) tot += s.weight;
    if (tot == 0) return fail(err, "total weight must be > 0");
  }
  st.hash = fnv1a(norm);
  *out = std::move(st);
  return true;
}

bool check_members(const Strategy& st, uint64_t members, std::string* err) {
  const int n = st.nranks;
  auto alive = [&](int g) { return ((members >> g) & 1) != 0; };
  for (const SubColl& s : st.subs) {
    if (s.kind == kNvls) {  // the multicast team is every rank of the communicator
      if (members != (n >= 64 ? ~uint64_t(0) : ((uint64_t(1) << n) - 1)))
        return fail(err, "an nvls line needs every rank (the multicast team)");
      continue;
    }
    if (s.kind == kA2A) {
      for (const Route& r : s.routes)
        for (int h : r.hops)
          if (!alive(h)) return fail(err, "an excluded rank cannot relay AlltoAll flows");
      continue;
    }
    if (st.coll == kReduce && !alive(s.root)) return fail(err, "the Reduce root was excluded");
    if (st.coll == kBroadcast && !alive(s.src)) return fail(err, "the Broadcast source was excluded");
    // an AllGather source / ReduceScatter block owner that was excluded: the
    // sub-collective is skipped (never ready / no destination)
    if ((s.kind == kBcast || s.kind == kRTree) && !alive(s.src)) continue;
    for (int g = 0; g < n; ++g)
      if (!alive(g) && !s.children[g].empty())
        return fail(err, "an excluded rank must be a leaf of every tree");
  }
  return true;
}

const std::vector<int>* SubColl::hops(int s, int d) const {
  for (const Route& r : routes)
    if (r.src == s && r.dst == d) return &r.hops;
  return nullptr;
}

std::vector<uint64_t> partition(uint64_t count, int esize, const std::vector<int64_t>& weights) {
  const uint64_t unit = 16 / esize;
  const unsigned __int128 U = count / unit;
  unsigned __int128 W = 0;
  for (int64_t w : weights) W += (uint64_t)w;
  std::vector<uint64_t> b(weights.size() + 1);
  unsigned __int128 prefix = 0;
  for (size_t m = 0; m < weights.size(); ++m) {
    b[m] = (uint64_t)((U * prefix) / W) * unit;
    prefix += (uint64_t)weights[m];
  }
  b[weights.size()] = count;
  return b;
}

TreeBehavior tree_behavior(const SubColl& s, uint64_t ready_mask) {
  const int n = (int)s.parent.size();
  TreeBehavior b;
  b.tup.assign(n, Tuple{});
  b.flows.assign(n, {});
  // iterative post-order from the root (children ascending)
  std::vector<std::pair<int, size_t>> stack = {{s.root, 0}};
  while (!stack.empty()) {
    auto& top = stack.back();
    const int g = top.first;
    if (top.second < s.children[g].size()) {
      int c = s.children[g][top.second++];
      stack.push_back({c, 0});
      continue;
    }
    stack.pop_back();
    b.postorder.push_back(g);
    Tuple& t = b.tup[g];
    t.act = (ready_mask >> g) & 1;
    int in_flows = 0;
    for (int c : s.children[g])
      if (b.tup[c].send) { t.recv = true; in_flows += (int)b.flows[c].size(); }
    const bool agg = !((s.noagg >> g) & 1);
    // no kernel if (1) nothing received, (2) relay with one incoming
    // flow, (3) a_{m,g} = 0
    t.kern = t.recv && agg && !(!t.act && in_flows == 1);
    // P:L155-157
    t.send = (t.act || t.recv) && g != s.root;
    if (t.kern) {
      b.flows[g].push_back({Flow::kAgg, g});
    } else {
      if (t.act) b.flows[g].push_back({Flow::kIn, g});
      for (int c : s.children[g])
        if (b.tup[c].send)
          b.flows[g].insert(b.flows[g].end(), b.flows[c].begin(), b.flows[c].end());
    }
  }
  return b;
}

std::vector<Flow> kernel_sources(const SubColl& s, const TreeBehavior& b, int g) {
  std::vector<Flow> src;
  if (b.tup[g].act) src.push_back({Flow::kIn, g});
  for (int c : s.children[g])
    if (b.tup[c].send) src.insert(src.end(), b.flows[c].begin(), b.flows[c].end());
  return src;
}

}  // namespace adapcc
