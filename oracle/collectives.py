"""Collective semantics under a strategy and a ready mask -- TEST INFRASTRUCTURE ONLY.

Ranks are simulated: ``xs[r]`` is rank r's 1-D send tensor (numpy), ``None``
allowed for a non-ready rank (its tensor is never read, reading Q11).
dtypes: 'f32' (np.float32), 'bf16' (np.uint16 bit patterns, see oracle.bf16),
'i32' (np.int32).

AllReduce has two definitions here:
  * ``allreduce`` replays the strategy's reduction order exactly (DESIGN.md
    §3 c-2): per tree, bottom-up behaviour tuples, every kernel
    node folds its own tensor (if ready) then its children's flows in
    ascending rank order, in the working precision (fp32 adds; bf16 widened to
    fp32 and rounded once per kernel node with RNE, Q6; int32 wraps, Q15); the
    root's result is broadcast to ALL ranks, relays included (Q4,
    "execute Broadcast reversely" P:L165).
  * ``allreduce_exact`` is the plain definition y = sum_{r in R} x_r in fp64
    ("aggregated tensor"), used to bound the replay's rounding.
AllGather ("one Broadcast on each GPU") and AlltoAll (P:L169,
P:L209-211) move bytes only; their oracle is the plain index definition and
the strategy can only be validated, not change the result (Q12 for masks).
"""

import numpy as np

from . import bf16 as _bf
from .strategy import parse, partition, ESIZE
from .tuples import behavior

_NP = {"f32": np.float32, "bf16": np.uint16, "i32": np.int32}


def _fold(terms, dtype):
    """Left-to-right fold of >= 2 equal-length arrays in the working precision."""
    if dtype == "f32":
        acc = terms[0].astype(np.float32, copy=True)
        for t in terms[1:]:
            acc = acc + t                     # one IEEE fp32 RNE add per element
        return acc
    if dtype == "bf16":
        acc = _bf.to_f32(terms[0])
        for t in terms[1:]:
            acc = acc + _bf.to_f32(t)         # fp32 accumulation
        return _bf.from_f32_rne(acc)          # one rounding per kernel node
    if dtype == "i32":
        acc = terms[0].astype(np.int64)
        for t in terms[1:]:
            acc = (acc + t.astype(np.int64)) & 0xFFFFFFFF   # mod 2^32
        return acc.astype(np.uint32).view(np.int32)
    raise ValueError(dtype)


def _accumulate(prev, res, dtype):
    """recvbuf += result with one rounding (flag ACCUMULATE, phase 2)."""
    return _fold([prev, res], dtype)


def _zero(k, dtype):
    return np.zeros(k, dtype=_NP[dtype])       # +0 bits for every dtype (Q7)


def allreduce(xs, strategy_text, ready, dtype, accumulate=False, y_prev=None):
    """Replay AllReduce along the strategy; returns a list of n arrays.

    xs           : list of n arrays (None for non-ready ranks) of equal length.
    ready        : iterable of ready ranks R.
    accumulate   : y_g <- y_prev_g + result (phase 2); y_prev required.
    """
    st = parse(strategy_text)
    if st.collective != "allreduce":
        raise ValueError("strategy is not an allreduce strategy")
    n = st.nranks
    ready = set(ready)
    lens = {len(x) for x in xs if x is not None}
    if y_prev is not None:
        lens |= {len(y) for y in y_prev}
    assert len(lens) == 1, "all tensors must have the same length"
    count = lens.pop()
    if accumulate:
        ys = [np.array(y_prev[g], dtype=_NP[dtype], copy=True) for g in range(n)]
    else:
        ys = [np.empty(count, dtype=_NP[dtype]) for _ in range(n)]
    bounds = partition(count, ESIZE[dtype], [s.weight for s in st.subs])
    for m, sub in enumerate(st.subs):
        lo, hi = bounds[m], bounds[m + 1]
        if lo == hi:
            continue
        res = _tree_result([x[lo:hi] if x is not None else None for x in xs], sub, ready, dtype)
        for g in range(n):
            if accumulate:
                if res is not None:
                    ys[g][lo:hi] = _accumulate(ys[g][lo:hi], res, dtype)
            else:
                ys[g][lo:hi] = res if res is not None else _zero(hi - lo, dtype)
    return ys


def _nvls_result(vals, ready, dtype):
    """An nvls sub-collective (reading R9): the NVSwitch sums the ready ranks'
    values in an order it does not disclose (PTX multimem.ld_reduce), so the
    oracle is the plain definition -- the exact sum (fp64 accumulation of the
    fp32 / bf16-widened values), rounded once to the working precision (RNE);
    int32 wraps mod 2^32.  GPU parity on fp32 / bf16 is a tolerance check
    against this (nvls_tolerance); int32 is bit-exact."""
    ready = sorted(r for r in ready if vals[r] is not None)
    if not ready:
        return None
    if dtype == "i32":
        tot = np.zeros(len(vals[ready[0]]), dtype=np.int64)
        for r in ready:
            tot = tot + vals[r].astype(np.int64)
        return (tot & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    acc = np.zeros(len(vals[ready[0]]), dtype=np.float64)
    for r in ready:
        acc = acc + (_bf.to_f32(vals[r]) if dtype == "bf16" else vals[r]).astype(np.float64)
    f32 = acc.astype(np.float32)
    return _bf.from_f32_rne(f32) if dtype == "bf16" else f32


def nvls_tolerance(dtype, k):
    """Normwise bound |y - exact| <= tol * sum_r |x_r| for a switch reduction
    of k terms in any order: fp32 adds: (k-1) u + u (the final rounding),
    u = 2^-24; bf16 with fp32 accumulation (.acc::f32) and one rounding to
    bf16: (k-1) 2^-24 + 2^-8.  int32: 0 (exact)."""
    if dtype == "i32":
        return 0.0
    u = 2.0 ** -24
    return (max(k - 1, 0) + 1) * u if dtype == "f32" else max(k - 1, 0) * u + 2.0 ** -8


def _tree_result(vals, sub, ready, dtype):
    """Result of one reduce tree over the elements in ``vals`` (vals[r]: rank r's
    values, None if not ready): bottom-up tuples, fold at every
    kernel node (own first, then sending children ascending, Q5), the root's
    aggregate or its single flow; None when no ready rank is in the tree.
    An nvls sub-collective reduces through the switch (_nvls_result)."""
    if sub.kind == "nvls":
        return _nvls_result(vals, ready, dtype)
    tup, flows = behavior(sub.parent, ready, sub.noagg)
    agg_val = {}

    def value(f):
        kind, r = f
        return vals[r] if kind == "in" else agg_val[r]

    order = []

    def visit(g):
        for c in sub.children(g):
            visit(c)
        order.append(g)

    visit(sub.root)
    for g in order:
        if tup[g][2]:
            terms = [vals[g]] if tup[g][0] else []
            for c in sub.children(g):
                if tup[c][3]:
                    terms += [value(f) for f in flows[c]]
            agg_val[g] = _fold(terms, dtype)
    root = sub.root
    if tup[root][2]:
        return agg_val[root]
    fl = flows[root]
    assert len(fl) <= 1, "a non-kernel root emits at most one flow"
    return np.array(value(fl[0]), copy=True) if fl else None


def allreduce_elements(vals, idx, count, strategy_text, ready, dtype, accumulate=False,
                       y_prev=None):
    """AllReduce result at selected element indices only (for sampled parity at
    full size): vals[r] holds rank r's inputs AT ``idx``; each element is
    reduced by the tree whose partition contains it (Q9), exactly as in
    ``allreduce``.  Returns the (broadcast-identical) result at idx; +0 where
    no rank is ready.  With ``accumulate``, y_prev (values at idx of one
    rank's recvbuf) is combined as in ``allreduce``."""
    st = parse(strategy_text)
    ready = set(ready)
    idx = np.asarray(idx, dtype=np.int64)
    bounds = partition(count, ESIZE[dtype], [s.weight for s in st.subs])
    out = np.array(y_prev, copy=True) if accumulate else _zero(len(idx), dtype)
    for m, sub in enumerate(st.subs):
        sel = np.nonzero((idx >= bounds[m]) & (idx < bounds[m + 1]))[0]
        if len(sel) == 0:
            continue
        res = _tree_result([v[sel] if v is not None else None for v in vals], sub, ready, dtype)
        if res is not None:
            out[sel] = _accumulate(out[sel], res, dtype) if accumulate else res
    return out


def allreduce_exact(xs, ready, dtype, count=None):
    """Plain definition: sum over ready ranks, fp64 for floats, mod 2^32 for int32.

    Returns float64 (f32/bf16) or int32 (i32) array.
    """
    ready = sorted(set(ready))
    if not ready:
        return np.zeros(count, dtype=np.float64 if dtype != "i32" else np.int32)
    if dtype == "i32":
        tot = np.zeros(len(xs[ready[0]]), dtype=np.int64)   # |sum| < 64 * 2^31: exact
        for r in ready:
            tot = tot + xs[r].astype(np.int64)
        return (tot & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    vals = [(_bf.to_f32(xs[r]) if dtype == "bf16" else xs[r]).astype(np.float64)
            for r in ready]
    return np.sum(np.stack(vals), axis=0)


def allgather(xs, strategy_text, ready, dtype, y_prev):
    """y_g[s*cnt:(s+1)*cnt] = x_s for every g and every ready s; other slots
    untouched (Q12).  y_prev: list of n arrays of n*cnt elements."""
    st = parse(strategy_text)
    if st.collective != "allgather":
        raise ValueError("strategy is not an allgather strategy")
    n = st.nranks
    ys = [np.array(y_prev[g], copy=True) for g in range(n)]
    for s in sorted(set(ready)):
        cnt = len(xs[s])
        for g in range(n):
            ys[g][s * cnt:(s + 1) * cnt] = xs[s]
    return ys


def alltoall(xs, strategy_text, ready, dtype, y_prev):
    """y_d[s*cnt:(s+1)*cnt] = x_s[d*cnt:(d+1)*cnt] for every d and ready s
    (including s == d); blocks from non-ready sources untouched (Q12)."""
    st = parse(strategy_text)
    if st.collective != "alltoall":
        raise ValueError("strategy is not an alltoall strategy")
    n = st.nranks
    ys = [np.array(y_prev[g], copy=True) for g in range(n)]
    for s in sorted(set(ready)):
        cnt = len(xs[s]) // n
        for d in range(n):
            ys[d][s * cnt:(s + 1) * cnt] = xs[s][d * cnt:(d + 1) * cnt]
    return ys


# ---------------------------------------------------------------- NEXT-4 primitives
def reduce(xs, strategy_text, ready, dtype, accumulate=False, y_prev=None):
    """Reduce: the trees' common root r receives sum_{R} x replayed along the
    trees (AdapCC "generate[s] strategies for Reduce"; the root GPU of
    each sub-collective "aggregates gradients").  Every other
    rank's recvbuf is untouched (returned as y_prev[g], or None)."""
    st = parse(strategy_text)
    if st.collective != "reduce":
        raise ValueError("strategy is not a reduce strategy")
    n = st.nranks
    ready = set(ready)
    root = st.subs[0].root
    lens = {len(x) for x in xs if x is not None}
    if y_prev is not None:
        lens |= {len(y_prev[root])}
    count = lens.pop()
    ys = [None if y_prev is None else np.array(y_prev[g], copy=True) for g in range(n)]
    y = np.array(y_prev[root], copy=True) if accumulate else np.empty(count, dtype=_NP[dtype])
    bounds = partition(count, ESIZE[dtype], [s.weight for s in st.subs])
    for m, sub in enumerate(st.subs):
        lo, hi = bounds[m], bounds[m + 1]
        if lo == hi:
            continue
        res = _tree_result([x[lo:hi] if x is not None else None for x in xs], sub, ready, dtype)
        if accumulate:
            if res is not None:
                y[lo:hi] = _accumulate(y[lo:hi], res, dtype)
        else:
            y[lo:hi] = res if res is not None else _zero(hi - lo, dtype)
    ys[root] = y
    return ys


def broadcast(xs, strategy_text, ready, dtype, y_prev):
    """Broadcast from the common src s of the bcast lines: y_g = x_s for every
    g when s is ready; otherwise every recvbuf is untouched (Q12)."""
    st = parse(strategy_text)
    if st.collective != "broadcast":
        raise ValueError("strategy is not a broadcast strategy")
    src = st.subs[0].src
    ys = [np.array(y, copy=True) for y in y_prev]
    if src in set(ready):
        for g in range(st.nranks):
            ys[g][:] = xs[src]
    return ys


def reducescatter(xs, strategy_text, ready, dtype, accumulate=False, y_prev=None):
    """ReduceScatter: rank b receives block b (cnt = len(x)/n elements) of
    sum_{R} x, replayed along the rtree lines of block b (rooted at b); the
    block's elements are partitioned over its lines by weight (Q9)."""
    st = parse(strategy_text)
    if st.collective != "reducescatter":
        raise ValueError("strategy is not a reducescatter strategy")
    n = st.nranks
    ready = set(ready)
    total = {len(x) for x in xs if x is not None}
    cnt = (total.pop() // n) if total else len(y_prev[0])
    ys = []
    for b in range(n):
        y = np.array(y_prev[b], copy=True) if accumulate else np.empty(cnt, dtype=_NP[dtype])
        lines = [sb for sb in st.subs if sb.src == b]
        bounds = partition(cnt, ESIZE[dtype], [sb.weight for sb in lines])
        for i, sub in enumerate(lines):
            lo, hi = bounds[i], bounds[i + 1]
            if lo == hi:
                continue
            res = _tree_result([x[b * cnt + lo:b * cnt + hi] if x is not None else None for x in xs],
                               sub, ready, dtype)
            if accumulate:
                if res is not None:
                    y[lo:hi] = _accumulate(y[lo:hi], res, dtype)
            else:
                y[lo:hi] = res if res is not None else _zero(hi - lo, dtype)
        ys.append(y)
    return ys


# --------------------------------------------------------- NEXT-1: late join
def _root_terms(vals, sub, ready, dtype):
    """The values a tree's root folds (kernel root: own tensor if ready, then the
    sending children's flows; non-kernel root: its single flow, or nothing),
    with every non-root kernel node's aggregate computed as in _tree_result."""
    tup, flows = behavior(sub.parent, ready, sub.noagg)
    agg_val = {}

    def value(f):
        kind, r = f
        return vals[r] if kind == "in" else agg_val[r]

    order = []

    def visit(g):
        for c in sub.children(g):
            visit(c)
        order.append(g)

    visit(sub.root)
    root = sub.root
    for g in order:
        if tup[g][2] and g != root:
            terms = [vals[g]] if tup[g][0] else []
            for c in sub.children(g):
                if tup[c][3]:
                    terms += [value(f) for f in flows[c]]
            agg_val[g] = _fold(terms, dtype)
    if tup[root][2]:
        terms = [vals[root]] if tup[root][0] else []
        for c in sub.children(root):
            if tup[c][3]:
                terms += [value(f) for f in flows[c]]
        return terms
    return [value(f) for f in flows[root]]


def allreduce_late(xs, strategy_text, ready, dtype, included, phase=1, y_prev=None, members=None):
    """Late join with a uniform inclusion set.

    phase 1: every tree's root folds its regular terms followed by the inputs
             of the late ranks in ``included`` (ascending rank): one rounding;
             a single term without late inputs is copied unchanged; no term -> +0.
    phase 2: y_prev + fold(inputs of the late ranks NOT in ``included``,
             ascending), one rounding for the sum and one for the addition
             (the ACCUMULATE rule); nothing left -> y_prev unchanged.
    Late ranks = ranks not in ``ready``; ``included`` must be a subset.
    members: the live ranks after a fault exclusion (faulty
    workers leave the group) -- excluded ranks are never late and never
    contribute; None = every rank."""
    st = parse(strategy_text)
    n = st.nranks
    ready = set(ready)
    late = sorted((set(range(n)) if members is None else set(members)) - ready)
    included = sorted(set(included))
    assert set(included) <= set(late)
    lens = {len(x) for x in xs if x is not None}
    count = lens.pop()
    bounds = partition(count, ESIZE[dtype], [s.weight for s in st.subs])
    if phase == 2:
        rest = [r for r in late if r not in included]
        ys = [np.array(y, copy=True) for y in y_prev]
        if not rest:
            return ys
        add = xs[rest[0]].copy() if len(rest) == 1 else _fold([xs[r] for r in rest], dtype)
        return [_accumulate(y, add, dtype) for y in ys]
    ys = [np.empty(count, dtype=_NP[dtype]) for _ in range(n)]
    for m, sub in enumerate(st.subs):
        lo, hi = bounds[m], bounds[m + 1]
        if lo == hi:
            continue
        vals = [x[lo:hi] if x is not None else None for x in xs]
        terms = _root_terms(vals, sub, ready, dtype) + [xs[r][lo:hi] for r in included]
        if not terms:
            res = _zero(hi - lo, dtype)
        elif len(terms) == 1:
            res = np.array(terms[0], copy=True)
        else:
            res = _fold(terms, dtype)
        for g in range(n):
            ys[g][lo:hi] = res
    return ys


def alltoallv(xs, counts, strategy_text, ready, dtype, y_prev):
    """AlltoAllv (NEXT-4): counts[s][d] elements of rank s's packed sendbuf
    (destination order) land in rank d's packed recvbuf (source order), for
    every ready s; other blocks untouched.  Pure index definition."""
    st = parse(strategy_text)
    if st.collective != "alltoall":
        raise ValueError("strategy is not an alltoall strategy")
    n = st.nranks
    ys = [np.array(y, copy=True) for y in y_prev]
    for s in sorted(set(ready)):
        for d in range(n):
            soff = sum(counts[s][:d])
            roff = sum(counts[j][d] for j in range(s))
            c = counts[s][d]
            ys[d][roff:roff + c] = xs[s][soff:soff + c]
    return ys
