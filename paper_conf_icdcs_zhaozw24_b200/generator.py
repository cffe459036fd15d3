"""Strategy generator: emits strategy text v1.

Stand-in for the paper's Synthesizer (§IV-D).  The MILP solved
with Gurobi is out of scope (NP-hard, licensed solver); the strategy
is an INPUT of the hot path.  This module produces the families the bench and
tests use -- star trees, complementary binary trees, rings (chains), per-source
broadcast trees, direct AlltoAll -- and link-bandwidth / ready-mask weighted
star trees from the paper's own link-load model applied to one NVSwitch:

  Reduce with aggregation at the root: one flow per (ready sender, tree)
  (N_{ij} = 1); Broadcast: one flow per edge; the
  profiled bandwidth of a link is shared by its flows (eq. 3).

For star tree m with weight w_m (fraction of the tensor) under ready set R
(k = |R|), the bytes each GPU g moves per byte of tensor are
  egress_g  = [g in R] (1 - w_g) + (n - 1) w_g
  ingress_g = (k - [g in R]) w_g + (1 - w_g)
and the generator minimises max_g max(egress_g, ingress_g) / b_g (b_g: the
GPU's NVLink bandwidth, uniform 900 GB/s by default) -- a small LP.
"""

DEFAULT_CHUNK = 262144


def _header(n, coll):
    return f"adapcc-strategy 1\nnranks {n}\ncollective {coll}\n"


def _join(v):
    return ",".join(str(int(x)) for x in v)


def star_parent(n, root):
    return [-1 if g == root else root for g in range(n)]


def chain_parent(order):
    """order[0] is the leaf, order[-1] the root."""
    p = [None] * len(order)
    for i, g in enumerate(order):
        p[g] = order[i + 1] if i + 1 < len(order) else -1
    return p


def binary_tree_parent(order):
    """Heap-shaped binary tree over `order` (order[0] is the root)."""
    p = [None] * len(order)
    for i, g in enumerate(order):
        p[g] = -1 if i == 0 else order[(i - 1) // 2]
    return p


# ------------------------------------------------------------------- allreduce
def allreduce_trees(parents, weights=None, chunk=DEFAULT_CHUNK, noaggs=None, relay=None):
    """relay: None (the default, bypass) or 'store' / 'bypass' on every tree line."""
    n = len(parents[0])
    weights = weights if weights is not None else [1] * len(parents)
    noaggs = noaggs or [()] * len(parents)
    out = _header(n, "allreduce")
    for p, w, na in zip(parents, weights, noaggs):
        out += f"tree weight={int(w)} chunk={int(chunk)} parent={_join(p)}"
        if na:
            out += f" noagg={_join(na)}"
        if relay:
            out += f" relay={relay}"
        out += "\n"
    return out


def allreduce_stars(n, chunk=DEFAULT_CHUNK, roots=None, weights=None):
    """M star trees rooted at `roots` (default: every rank) -- the B200 analogue
    of M parallel sub-collectives (M sweep of Fig. 19(a))."""
    roots = list(range(n)) if roots is None else list(roots)
    return allreduce_trees([star_parent(n, r) for r in roots], weights, chunk)


def allreduce_double_binary(n, chunk=DEFAULT_CHUNK):
    """Two complementary heap trees (NCCL-style double binary tree)."""
    a = list(range(n))
    b = [(g + n // 2) % n for g in range(n)][::-1]
    return allreduce_trees([binary_tree_parent(a), binary_tree_parent(b)], [1, 1], chunk)


def allreduce_ring(n, chunk=DEFAULT_CHUNK, order=None, weight=1):
    order = list(range(n)) if order is None else list(order)
    return _header(n, "allreduce") + f"ring weight={int(weight)} chunk={int(chunk)} order={_join(order)}\n"


def star_loads(n, ready, w, bw=None):
    """Per-GPU (egress, ingress) bytes per tensor byte and the max time factor."""
    ready = set(ready)
    k = len(ready)
    bw = bw or [1.0] * n
    eg = [((g in ready) * (1 - w[g]) + (n - 1) * w[g]) for g in range(n)]
    ig = [((k - (g in ready)) * w[g] + (1 - w[g])) for g in range(n)]
    t = max(max(e, i) / b for e, i, b in zip(eg, ig, bw))
    return eg, ig, t


def mask_aware_star_weights(n, ready, bw=None, relays_as_roots=True, scale=1 << 16):
    """Fractions w_m minimising the max per-GPU time under the load model above.

    relays_as_roots=False forces w = 0 on non-ready roots (relays as leaves);
    returns (integer weights, fractions, time factor)."""
    ready = set(ready)
    bw = bw or [1.0] * n
    if not ready:
        w = [1.0 / n] * n
    else:
        w = _solve_lp(n, ready, bw, relays_as_roots)
    ints = [int(round(x * scale)) for x in w]
    if sum(ints) == 0:
        ints = [1] * n
    return ints, w, star_loads(n, ready, w, bw)[2]


def _solve_lp(n, ready, bw, relays_as_roots):
    """Min-max weights by water-filling (no solver needed): GPU g's time
    s_g(w) = max(egress_g(w), ingress_g(w)) / b_g is affine-increasing in its
    own weight w (star_loads), so the lexicographic min-max allocation under
    sum w = 1 raises a common level L until the weights w_g(L) = the largest w
    with s_g(w) <= L (0 if g's base load already exceeds L; 0 for relays when
    they may not root) sum to 1.  Among the min-max optima it is the one that
    evens out every non-bottleneck GPU (an LP vertex would pile the weight
    onto a few of them when a slow GPU's own slice sets the maximum)."""
    ready = set(ready)
    k = len(ready)
    terms = []   # per g: [(c, d)] with load = c + d w for egress and ingress
    for g in range(n):
        r = g in ready
        terms.append([(1.0 if r else 0.0, (n - 1) - (1.0 if r else 0.0)),      # egress
                      (1.0, (k - (1.0 if r else 0.0)) - 1.0)])                  # ingress
    ub = [1.0 if (g in ready or relays_as_roots) else 0.0 for g in range(n)]

    def w_at(L):
        out = []
        for g in range(n):
            w = ub[g]
            for c, d in terms[g]:
                if c > L * bw[g]:
                    w = 0.0
                elif d > 0:
                    w = min(w, (L * bw[g] - c) / d)
            out.append(max(0.0, w))
        return out

    lo, hi = 0.0, 1.0
    while sum(w_at(hi)) < 1.0:
        hi *= 2.0
        if hi > 1e12:
            return _two_class(n, ready, relays_as_roots)
    for _ in range(200):
        mid = 0.5 * (lo + hi)
        if sum(w_at(mid)) < 1.0:
            lo = mid
        else:
            hi = mid
    w = w_at(hi)
    tot = sum(w)
    return [x / tot for x in w]


def _two_class(n, ready, relays_as_roots):
    k = len(ready)
    best = None
    steps = 20000
    for i in range(steps + 1):
        wa = i / steps / k
        wr = (1 - k * wa) / (n - k) if n > k else 0.0
        if n > k and not relays_as_roots:
            if abs(1 - k * wa) > 1e-12:
                continue
            wr = 0.0
        if wr < -1e-12:
            continue
        w = [wa if g in ready else wr for g in range(n)]
        t = star_loads(n, ready, w)[2]
        if best is None or t < best[0]:
            best = (t, w)
    return best[1]


def allreduce_mask_aware_stars(n, ready, chunk=DEFAULT_CHUNK, bw=None, relays_as_roots=True):
    ints, _, _ = mask_aware_star_weights(n, ready, bw, relays_as_roots)
    return allreduce_stars(n, chunk, weights=ints)


# ------------------------------------------------------------------- allgather
def allreduce_nvls(n, chunk=DEFAULT_CHUNK, nvls_weight=1, star_weight=0):
    """NVLS switch reduction (NEXT-2): one nvls line (the NVSwitch reduces and
    multicasts its partition) plus, with star_weight > 0, n star trees sharing
    the rest (weights are per line, reading Q9)."""
    lines = [f"nvls weight={nvls_weight} chunk={chunk}"]
    if star_weight:
        for m in range(n):
            lines.append(f"tree weight={star_weight} chunk={chunk} parent={_join(star_parent(n, m))}")
    return _header(n, "allreduce") + "\n".join(lines) + "\n"


def allgather_stars(n, chunk=DEFAULT_CHUNK):
    """One Broadcast per source, each a star from the source."""
    out = _header(n, "allgather")
    for s in range(n):
        out += f"bcast src={s} weight=1 chunk={int(chunk)} parent={_join(star_parent(n, s))}\n"
    return out


def allgather_chains(n, chunk=1 << 20):
    out = _header(n, "allgather")
    for s in range(n):
        order = [(s + k) % n for k in range(n - 1, -1, -1)]
        out += f"bcast src={s} weight=1 chunk={int(chunk)} parent={_join(chain_parent(order))}\n"
    return out


# -------------------------------------------------------------------- alltoall
def alltoall_direct(n, chunk=1 << 20, lines=1):
    return _header(n, "alltoall") + "".join(
        f"a2a weight=1 chunk={int(chunk)}\n" for _ in range(lines))


def alltoall_routed(n, lines, chunk=1 << 20):
    """AlltoAll with explicit routes (routing variables x^f_ij, eq. 1).
    lines: list of (weight, {(s, d): [h1, ..]}) -- one a2a line each; flows
    absent from a line's dict go direct."""
    out = _header(n, "alltoall")
    for w, routes in lines:
        out += f"a2a weight={int(w)} chunk={int(chunk)}"
        if routes:
            out += " route=" + ";".join(f"{s}:{d}:{_join(h)}" for (s, d), h in sorted(routes.items()))
        out += "\n"
    return out


def alltoall_detour(n, slow_edges, chunk=1 << 20, direct_weight=0, routed_weight=1):
    """Route AlltoAll around slow links (the synthesizer's routing decision,
    P:L171, under the load model of P:L209-211): every flow s -> d whose direct
    edge is slow takes a two-hop path s -> h -> d through the relay h whose two
    edges carry the fewest flows so far (both fast).  direct_weight > 0 adds a
    direct a2a line, so that routed_weight : direct_weight of every block is
    detoured and the rest still uses the slow edge (multi-path split)."""
    slow = set(slow_edges)
    load = {(i, j): 1 for i in range(n) for j in range(n) if i != j and (i, j) not in slow}
    routes = {}
    for (s, d) in sorted(slow):
        best = None
        for h in range(n):
            if h in (s, d) or (s, h) in slow or (h, d) in slow:
                continue
            cost = max(load[(s, h)], load[(h, d)])
            if best is None or cost < best[0]:
                best = (cost, h)
        if best is None:
            continue                       # no fast detour: stays direct
        h = best[1]
        load[(s, h)] += 1
        load[(h, d)] += 1
        routes[(s, d)] = [h]
    lines = [(routed_weight, routes)] + ([(direct_weight, {})] if direct_weight else [])
    return alltoall_routed(n, lines, chunk)


def survivor_stars(n, alive, chunk=DEFAULT_CHUNK):
    """AllReduce strategy after a fault exclusion (NEXT-3): one
    star per live rank with equal weights; excluded ranks are leaves of every
    star (the only place adapcc_exclude lets a strategy name them)."""
    out = _header(n, "allreduce")
    for r in sorted(alive):
        out += f"tree weight=1 chunk={int(chunk)} parent={_join(star_parent(n, r))}\n"
    return out


# ----------------------------------------------------- NEXT-4 primitives
def reduce_trees(parents, weights=None, chunk=DEFAULT_CHUNK, noaggs=None):
    """Reduce: every tree must be rooted at the Reduce root."""
    n = len(parents[0])
    weights = weights if weights is not None else [1] * len(parents)
    noaggs = noaggs or [()] * len(parents)
    out = _header(n, "reduce")
    for p, w, na in zip(parents, weights, noaggs):
        out += f"tree weight={int(w)} chunk={int(chunk)} parent={_join(p)}"
        if na:
            out += f" noagg={_join(na)}"
        out += "\n"
    return out


def broadcast_trees(root, parents, weights=None, chunk=DEFAULT_CHUNK):
    n = len(parents[0])
    weights = weights if weights is not None else [1] * len(parents)
    return _header(n, "broadcast") + "".join(
        f"bcast src={root} weight={int(w)} chunk={int(chunk)} parent={_join(p)}\n"
        for p, w in zip(parents, weights))


def reducescatter_stars(n, chunk=DEFAULT_CHUNK):
    """One star per block b rooted at b (b's block is reduced at b)."""
    return _header(n, "reducescatter") + "".join(
        f"rtree dst={b} weight=1 chunk={int(chunk)} parent={_join(star_parent(n, b))}\n" for b in range(n))


def reducescatter_trees(lines, n, chunk=DEFAULT_CHUNK):
    """lines: list of (dst, parent, weight)."""
    return _header(n, "reducescatter") + "".join(
        f"rtree dst={d} weight={int(w)} chunk={int(chunk)} parent={_join(p)}\n" for d, p, w in lines)
