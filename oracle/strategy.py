"""Strategy text v1: parser, validator, ring expansion, partition, chunking.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Independent of the C++
loader in paper_conf_icdcs_zhaozw24_b200/csrc/strategy.cpp; both follow the
format specification in DESIGN.md §2.

The paper's strategy is "M parallel sub-collectives", each with its own
communication graph, a data partition S_m with sum S_m = S and a chunk size
C_m (§IV-D, Fig. 8); aggregation flags a_{m,g}
(P:L184); the paper serialises strategies as XML whose schema it does not give
(P:L233), so the text format here is our own.

Format (one directive per line, '#' starts a comment):

    adapcc-strategy 1
    nranks <n>                                  1 <= n <= 64
    collective allreduce|allgather|alltoall
    tree  weight=<w> chunk=<C> parent=<p_0,..,p_{n-1}> [noagg=<g,..>] [relay=store|bypass]   (allreduce)
    ring  weight=<w> chunk=<C> order=<r_0,..,r_{n-1}>                     (allreduce)
    bcast src=<s> weight=<w> chunk=<C> parent=<p_0,..,p_{n-1}>           (allgather, broadcast)
    a2a   weight=<w> chunk=<C> [route=<s>:<d>:<h1>,..[;<s>:<d>:<h>,..]]  (alltoall)
    rtree dst=<b> weight=<w> chunk=<C> parent=<...> [noagg=<g,..>]       (reducescatter)
    nvls  weight=<w> chunk=<C>                                            (allreduce)
  collective reduce uses tree lines sharing one root; broadcast uses bcast
  lines sharing one src (NEXT-4 primitives: Reduce / Broadcast, P:L165,
  ReduceScatter, P:L154(1)).

An nvls line reduces its partition through the NVSwitch (multimem
ld_reduce / st, NEXT-2): the switch is the aggregation point, every rank
receives the result (reading R9: the summation order is the switch's).

An a2a route entry s:d:h1,..,hk sends flow s -> d along s, h1, .., hk, d
(routing variables x^f_ij of eq. 1); flows without an entry go
direct.

Readings: Q9 partition, Q10 chunk, Q13 ring expansion.
"""

import re
from dataclasses import dataclass, field

MAX_RANKS = 64
MAX_SUBS = 128
MAX_WEIGHT = 1 << 24
MAX_CHUNK = 1 << 31
ESIZE = {"f32": 4, "bf16": 2, "i32": 4}


class StrategyError(ValueError):
    """Malformed or invalid strategy text."""


@dataclass
class Sub:
    """One sub-collective m after ring expansion."""
    kind: str                 # 'tree' | 'nvls' (allreduce), 'bcast' (allgather), 'a2a', 'rtree'
    weight: int               # effective integer weight (see expand_weights)
    chunk: int                # C_m in bytes
    parent: list = None       # parent[g], -1 at the root (tree / bcast)
    noagg: frozenset = frozenset()   # ranks g with a_{m,g} = 0
    src: int = -1             # bcast: source (== root); rtree: destination block (== root)
    routes: dict = field(default_factory=dict)   # a2a: (s, d) -> tuple of relay ranks
    relay: str = "bypass"     # tree: how a pure relay forwards its single flow (data path only:
                              # the bytes arrive unchanged either way, so results do not depend on it)

    @property
    def root(self):
        return self.parent.index(-1)

    def children(self, g):
        """Children of g in ascending rank order (reading Q5)."""
        return [c for c in range(len(self.parent)) if self.parent[c] == g]


@dataclass
class Strategy:
    nranks: int
    collective: str
    subs: list = field(default_factory=list)


_INT_RE = re.compile(r"-?[0-9]+")


def _int(tok, what):
    """Integers are ``-?[0-9]+``; no '+', '_' or whitespace."""
    if not _INT_RE.fullmatch(tok):
        raise StrategyError(f"bad integer for {what}: {tok!r}")
    return int(tok, 10)


def _intlist(tok, what):
    if tok == "":
        return []
    return [_int(t, what) for t in tok.split(",")]


def _check_tree(parent, n, what):
    if len(parent) != n:
        raise StrategyError(f"{what}: parent has {len(parent)} entries, nranks={n}")
    roots = [g for g in range(n) if parent[g] == -1]
    if len(roots) != 1:
        raise StrategyError(f"{what}: need exactly one root, found {len(roots)}")
    for g, p in enumerate(parent):
        if p == -1:
            continue
        if not (0 <= p < n):
            raise StrategyError(f"{what}: parent[{g}]={p} out of range")
        if p == g:
            raise StrategyError(f"{what}: self loop at {g}")
    # every node must reach the root: walk at most n steps
    for g in range(n):
        x, steps = g, 0
        while parent[x] != -1:
            x = parent[x]
            steps += 1
            if steps > n:
                raise StrategyError(f"{what}: cycle through rank {g}")


def _routes(tok, n):
    """route=s:d:h1,h2;... -> {(s, d): (h1, h2)}.  Eq. 1 asks that a
    flow leave its source once, enter its destination once and be conserved
    at every other node; a simple path s, h1, .., hk, d (all ranks distinct,
    k >= 1) is exactly such a flow without cycles."""
    out = {}
    if tok is None:
        return out
    for ent in tok.split(";"):
        parts = ent.split(":")
        if len(parts) != 3:
            raise StrategyError(f"route entry {ent!r} is not src:dst:hops")
        s, d = _int(parts[0], "route src"), _int(parts[1], "route dst")
        hops = _intlist(parts[2], "route hops")
        path = [s] + hops + [d]
        if any(not (0 <= g < n) for g in path):
            raise StrategyError(f"route {ent!r} has a rank out of range")
        if s == d:
            raise StrategyError("route src == dst")
        if not hops:
            raise StrategyError("route needs at least one relay")
        if len(set(path)) != len(path):
            raise StrategyError(f"route {ent!r} visits a rank twice")
        if (s, d) in out:
            raise StrategyError(f"two routes for flow {s}->{d}")
        out[(s, d)] = tuple(hops)
    return out


def flow_path(sub, s, d):
    """Nodes of flow s -> d in a2a sub-collective `sub`: [s, h1, .., hk, d]."""
    return [s] + list(sub.routes.get((s, d), ())) + [d]


def parse(text):
    """Parse and validate strategy text; returns Strategy with rings expanded.

    Ring expansion (reading Q13): ``ring order=r_0..r_{n-1}`` becomes n chain
    trees; tree m has root r_m, leaf r_{m+1}, and parent[r_{m+j}] = r_{m+j+1}
    for j = 1..n-1 (indices mod n).  A ring of weight w contributes w/n per
    chain; to keep integers every tree/bcast/a2a weight is multiplied by n and
    each chain gets weight w (only weight ratios enter the partition, Q9).
    """
    lines = []
    for raw in text.splitlines():
        s = raw.split("#", 1)[0].strip()
        if s:
            lines.append(s)
    if not lines or lines[0].split() != ["adapcc-strategy", "1"]:
        raise StrategyError("first line must be 'adapcc-strategy 1'")
    n = None
    coll = None
    raw_subs = []
    for s in lines[1:]:
        toks = s.split()
        head = toks[0]
        if head == "nranks":
            if n is not None or len(toks) != 2:
                raise StrategyError("bad or repeated nranks line")
            n = _int(toks[1], "nranks")
            if not (1 <= n <= MAX_RANKS):
                raise StrategyError(f"nranks {n} out of range")
            continue
        if head == "collective":
            if coll is not None or len(toks) != 2:
                raise StrategyError("bad or repeated collective line")
            coll = toks[1]
            if coll not in ("allreduce", "allgather", "alltoall", "reduce", "broadcast",
                            "reducescatter"):
                raise StrategyError(f"unknown collective {coll!r}")
            continue
        if head not in ("tree", "ring", "bcast", "a2a", "rtree", "nvls"):
            raise StrategyError(f"unknown directive {head!r}")
        kv = {}
        for t in toks[1:]:
            if "=" not in t:
                raise StrategyError(f"expected key=value, got {t!r}")
            k, v = t.split("=", 1)
            if k in kv:
                raise StrategyError(f"repeated key {k!r}")
            kv[k] = v
        raw_subs.append((head, kv))
    if n is None or coll is None:
        raise StrategyError("missing nranks or collective line")
    allowed = {"allreduce": ("tree", "ring", "nvls"), "allgather": ("bcast",), "alltoall": ("a2a",),
               "reduce": ("tree",), "broadcast": ("bcast",), "reducescatter": ("rtree",)}[coll]
    keys = {"tree": {"weight", "chunk", "parent"}, "ring": {"weight", "chunk", "order"},
            "bcast": {"src", "weight", "chunk", "parent"}, "a2a": {"weight", "chunk"},
            "rtree": {"dst", "weight", "chunk", "parent"}, "nvls": {"weight", "chunk"}}
    optional = {"tree": {"noagg", "relay"}, "ring": set(), "bcast": set(), "a2a": {"route"},
                "rtree": {"noagg"}, "nvls": set()}
    if not raw_subs:
        raise StrategyError("no sub-collective lines")
    st = Strategy(nranks=n, collective=coll)
    for head, kv in raw_subs:
        if head not in allowed:
            raise StrategyError(f"directive {head!r} not valid for {coll}")
        missing = keys[head] - set(kv)
        extra = set(kv) - keys[head] - optional[head]
        if missing or extra:
            raise StrategyError(f"{head}: missing {sorted(missing)} extra {sorted(extra)}")
        w = _int(kv["weight"], "weight")
        c = _int(kv["chunk"], "chunk")
        if not (0 <= w <= MAX_WEIGHT):
            raise StrategyError(f"weight {w} out of range")
        if c < 16 or c % 16 != 0 or c > MAX_CHUNK:
            raise StrategyError(f"chunk {c} must be a positive multiple of 16 <= 2^31")
        if head in ("tree", "rtree"):
            parent = _intlist(kv["parent"], "parent")
            _check_tree(parent, n, head)
            noagg = _intlist(kv.get("noagg", ""), "noagg")
            if len(set(noagg)) != len(noagg):
                raise StrategyError("duplicate rank in noagg")
            for g in noagg:
                if not (0 <= g < n):
                    raise StrategyError(f"noagg rank {g} out of range")
                if parent[g] == -1:
                    raise StrategyError("noagg may not contain the root")
            if head == "rtree":
                dst = _int(kv["dst"], "dst")
                if not (0 <= dst < n) or parent[dst] != -1:
                    raise StrategyError("rtree root must be its dst")
                st.subs.append(Sub("rtree", w * n, c, parent, frozenset(noagg), dst))
            else:
                relay = kv.get("relay", "bypass")
                if relay not in ("store", "bypass"):
                    raise StrategyError("relay must be store or bypass")
                st.subs.append(Sub("tree", w * n, c, parent, frozenset(noagg), relay=relay))
        elif head == "ring":
            order = _intlist(kv["order"], "order")
            if sorted(order) != list(range(n)):
                raise StrategyError("ring order must be a permutation of 0..n-1")
            for m in range(n):
                parent = [None] * n
                parent[order[m]] = -1
                for j in range(1, n):
                    parent[order[(m + j) % n]] = order[(m + j + 1) % n]
                st.subs.append(Sub("tree", w, c, parent, frozenset()))
        elif head == "bcast":
            src = _int(kv["src"], "src")
            if not (0 <= src < n):
                raise StrategyError(f"bcast src {src} out of range")
            parent = _intlist(kv["parent"], "parent")
            _check_tree(parent, n, "bcast")
            if parent[src] != -1:
                raise StrategyError("bcast root must be its src")
            st.subs.append(Sub("bcast", w * n, c, parent, frozenset(), src))
        elif head == "nvls":
            st.subs.append(Sub("nvls", w * n, c))
        else:
            st.subs.append(Sub("a2a", w * n, c, routes=_routes(kv.get("route"), n)))
    if len(st.subs) > MAX_SUBS:
        raise StrategyError(f"{len(st.subs)} sub-collectives > {MAX_SUBS}")
    if coll in ("allgather", "reducescatter"):
        for s in range(n):
            ws = [sb.weight for sb in st.subs if sb.src == s]
            if not ws or sum(ws) == 0:
                raise StrategyError(f"{coll} block {s} has no positive-weight line")
    else:
        if coll == "reduce" and len({sb.root for sb in st.subs}) != 1:
            raise StrategyError("reduce trees must share one root")
        if coll == "broadcast" and len({sb.src for sb in st.subs}) != 1:
            raise StrategyError("broadcast lines must share one src")
        if sum(sb.weight for sb in st.subs) == 0:
            raise StrategyError("total weight must be > 0")
    return st


def partition(count, esize, weights):
    """Split ``count`` elements into len(weights) contiguous ranges (reading Q9).

    P:L167 only says sum_m S_m = S.  Rule: unit u = 16/esize elements,
    U = floor(count/u), W = sum(w); b_m = floor(U * sum_{j<m} w_j / W) * u for
    m < M, b_M = count (the last range also takes the ragged tail).
    Returns the M+1 bounds.  Python integers: exact.
    """
    u = 16 // esize
    U = count // u
    W = sum(weights)
    bounds = []
    acc = 0
    for w in weights:
        bounds.append((U * acc // W) * u)
        acc += w
    bounds.append(count)
    return bounds


def chunks(lo, hi, chunk_bytes, esize):
    """Chunks of C_m bytes over [lo, hi) (reading Q10); last may be short."""
    ce = chunk_bytes // esize
    out = []
    a = lo
    while a < hi:
        out.append((a, min(hi, a + ce)))
        a += ce
    return out
