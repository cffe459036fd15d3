"""Link profiler and strategy cost model (NEXT-2, §IV-B, §IV-D).

alpha-beta profiling: on a link, sending a piece of size s n times
takes n(alpha + beta s); sending n*s at once takes alpha + beta n s; several
(n, s) pairs give alpha and beta.  Probe rounds between instances follow the
round-robin schedule of Fig. 5(b): in round i instance k
probes (k + i) % N, so every round is a permutation (one flow per port).

Cost model of a reduce tree, used to choose chunk sizes:
  t_ij   = alpha_ij + beta~_ij C_m                   (chunk time on edge i -> j)
  beta~_ij = beta_ij * sum_m N^m_ij                  (eq. 3, bandwidth sharing)
  N^m_ij = 1 when i aggregates; |F^i_m| + sum_k N^m_ki otherwise;
           1 for Broadcast
  h_j    = max over in-flows (h_i + t_ij) with aggregation, h_i + t_ij without
           (eq. 2, garbled; reading Q18)
  T_f    = h_dst + ceil(S_m / C_m) * T_bottle, T_bottle = max edge gap on the
           path (eqs. 5, 6); the strategy's time is max_f T_f (eq. 4)
AlltoAll: N_ij = number of flows (all lines) traversing (i, j);
relays do not aggregate, so a flow's first chunk reaches its destination at
h = sum of t_ij along its route (eq. 2, a = 0) and the flow ends at
h + ceil(S_m / C_m) * (its slowest edge) (eqs. 5, 6).
AllReduce = the Reduce trees followed by their reversed Broadcast, pipelined
chunk by chunk: per tree T = h_root + depth_bcast_time +
ceil(S_m / C_m) * max(bottleneck of both stages) -- reading R6.
Trees are read through the product's strategy loader (host-only C ABI).
"""

import math

from . import adapcc as _A

# ---------------------------------------------------------------- profiler


def solve_alpha_beta(t_many, t_once, n, s):
    """Closed form from the two probes of P:L113:
    t_many = n (alpha + beta s), t_once = alpha + beta n s
    => alpha = (t_many - t_once) / (n - 1), beta = (t_once - alpha) / (n s)."""
    alpha = (t_many - t_once) / (n - 1)
    beta = (t_once - alpha) / (n * s)
    return alpha, beta


def fit_alpha_beta(samples):
    """Least squares over (messages, bytes_each, seconds) samples of the model
    t = messages * alpha + messages * bytes_each * beta ("several
    measurements are performed under different values of n and s")."""
    a11 = a12 = a22 = b1 = b2 = 0.0
    for m, s, t in samples:
        x1, x2 = float(m), float(m) * float(s)
        a11 += x1 * x1
        a12 += x1 * x2
        a22 += x2 * x2
        b1 += x1 * t
        b2 += x2 * t
    det = a11 * a22 - a12 * a12
    return (b1 * a22 - b2 * a12) / det, (a11 * b2 - a12 * b1) / det


def probe_rounds(n_instances):
    """Fig. 5(b): N-1 rounds; in round i instance k probes (k + i) % N."""
    return [[(k, (k + i) % n_instances) for k in range(n_instances)] for i in range(1, n_instances)]


def probe_link(copy_fn, sizes=(1 << 16, 1 << 20), repeats=(1, 8), timer=None):
    """Measure one link with the paper's two probe shapes.  copy_fn(nbytes)
    performs one transfer and returns its duration in seconds (or timer()
    measures it).  Returns (alpha, beta, samples)."""
    samples = []
    for s in sizes:
        for n in repeats:
            t = sum(copy_fn(s) for _ in range(n))        # n pieces of s
            samples.append((n, s, t))
            t1 = copy_fn(n * s)                          # one piece of n*s
            samples.append((1, n * s, t1))
    alpha, beta = fit_alpha_beta(samples)
    return alpha, beta, samples


def profile_links(comm, sizes=(1 << 16, 1 << 22), repeats=(1, 8), engine="sm", iters=20, gather=None):
    """Per-link alpha / beta on the device, through
    adapcc_link_probe (graph-captured messages, so alpha is the device's
    per-message cost rather than host launch noise).

    Multi-process: the N-1 rounds of Fig. 5(b) (probe_rounds): in round i rank
    k probes (k + i) % N while every other rank probes its own partner (one
    flow per port); per link the paper's two shapes, m messages of s
    and one message of m*s, for every (s, m), least-squares fit.
    `gather(obj) -> list per rank` shares the rows (default: the
    torch.distributed default group).  Loopback (n virtual ranks on one GPU):
    virtual rank 0 probes each q in turn; every "link" is the HBM copy path.
    Also times the fan-out 1 -> all others at the largest size (the N>1 bench's
    P2P ceiling).  Returns a JSON-able dict."""
    n, me = comm.nranks, comm.rank
    rounds = [[(0, q)] for q in range(1, n)] if comm.loopback else probe_rounds(n)
    rows = {}
    for rnd in rounds:
        mine = rnd if comm.loopback else [p for p in rnd if p[0] == me]
        for (i, j) in mine:
            samples = []
            for s in sizes:
                for m in repeats:
                    for msgs, nb in ((m, s), (1, m * s)):
                        t = comm.link_probe({j}, nb, messages=msgs, engine=engine, iters=iters,
                                            src=i if comm.loopback else -1)
                        samples.append((msgs, nb, t))
            a, b = fit_alpha_beta(samples)
            rows[(i, j)] = {"alpha_s": a, "beta_s_per_byte": b, "samples": samples}
    # fan-out 1 -> n-1 (rank 0 sends, the others only take part)
    big = max(sizes) * max(repeats)
    fan_dst = set(range(1, n)) if (comm.loopback or me == 0) else set()
    t_fan = comm.link_probe(fan_dst, big, engine=engine, iters=max(2, iters // 4), src=0 if comm.loopback else -1)
    mine = {"rows": {f"{i}->{j}": v for (i, j), v in rows.items()},
            "fanout": {"src": 0, "bytes_per_dst": big, "seconds": t_fan} if fan_dst else None}
    if comm.loopback:
        per_rank = [mine]
    else:
        if gather is None:
            import torch.distributed as dist

            def gather(obj):
                out = [None] * dist.get_world_size()
                dist.all_gather_object(out, obj)
                return out
        per_rank = gather(mine)
    alpha = [[None] * n for _ in range(n)]
    beta = [[None] * n for _ in range(n)]
    samples = {}
    for pr in per_rank:
        for key, v in pr["rows"].items():
            i, j = (int(x) for x in key.split("->"))
            alpha[i][j], beta[i][j] = v["alpha_s"], v["beta_s_per_byte"]
            samples[key] = v["samples"]
    fan = [pr["fanout"] for pr in per_rank if pr["fanout"]]
    gbps = [[(1.0 / b / 1e9 if b and b > 0 else None) for b in row] for row in beta]
    return {"n": n, "engine": engine, "loopback": comm.loopback, "sizes": list(sizes), "repeats": list(repeats),
            "alpha_us": [[(a * 1e6 if a is not None else None) for a in row] for row in alpha],
            "beta_GBps": gbps, "samples": samples,
            "fanout": [{"src": f["src"], "dsts": n - 1, "bytes_per_dst": f["bytes_per_dst"], "seconds": f["seconds"],
                        "GBps_per_dst": f["bytes_per_dst"] / f["seconds"] / 1e9 if f["seconds"] else None,
                        "GBps_out": (n - 1) * f["bytes_per_dst"] / f["seconds"] / 1e9 if f["seconds"] else None}
                       for f in fan]}


def links_to_model(profile):
    """alpha[i][j] (s) and beta[i][j] (s/byte) matrices for the cost model;
    links the profile did not measure take the mean of the measured ones."""
    n = profile["n"]
    a_all = [a for row in profile["alpha_us"] for a in row if a is not None]
    g_all = [g for row in profile["beta_GBps"] for g in row if g]
    a0 = (sum(a_all) / len(a_all)) * 1e-6 if a_all else 3e-6
    b0 = 1.0 / ((sum(g_all) / len(g_all)) * 1e9) if g_all else 1.0 / 770e9
    alpha = [[(profile["alpha_us"][i][j] * 1e-6 if profile["alpha_us"][i][j] is not None else a0) for j in range(n)]
             for i in range(n)]
    beta = [[(1.0 / (profile["beta_GBps"][i][j] * 1e9) if profile["beta_GBps"][i][j] else b0) for j in range(n)]
            for i in range(n)]
    return alpha, beta


def per_gpu_bandwidth(profile):
    """Per-GPU link bandwidth (GB/s) for generator.mask_aware_star_weights(bw=):
    the slowest measured outgoing link of each GPU (one NVSwitch port each)."""
    n = profile["n"]
    out = []
    for i in range(n):
        g = [profile["beta_GBps"][i][j] for j in range(n) if j != i and profile["beta_GBps"][i][j]]
        out.append(min(g) if g else None)
    known = [x for x in out if x]
    fill = sum(known) / len(known) if known else 1.0
    return [x if x else fill for x in out]


def chunk_from_profile(profile, S, text_for_chunk=None, candidates=(1 << 14, 1 << 16, 1 << 18, 1 << 20, 1 << 22)):
    """The cost model's chunk for S bytes per rank on the profiled links
    (default strategy: n star trees), plus the predicted times."""
    from . import generator as G
    n = profile["n"]
    alpha, beta = links_to_model(profile)
    fn = text_for_chunk or (lambda c: G.allreduce_stars(n, chunk=c))
    return best_chunk(fn, S, alpha, beta, candidates)


def adapt_strategy(comm, tensor_bytes, ready=None, profile=None, engine="sm", set_default_chunk=True,
                   **probe_kw):
    """The paper's adaptation loop (P:L109-115 profiling -> P:L176-231 strategy
    -> P:L341-343 swap without restart) in one call: profile the links (or use
    `profile`), weight the n star trees by the measured per-GPU bandwidth and
    the ready set (generator.mask_aware_star_weights, the link-load model of
    P:L194-215), pick the chunk with the cost model (eqs. 2-6) and install
    the result with set_strategy (stream-ordered, reading a10).  Collective in
    multi-process mode (profiling probes every link).  Returns (text,
    profile, chunk)."""
    from . import generator as G
    prof = profile or profile_links(comm, engine=engine, **probe_kw)
    n = comm.nranks
    R = set(range(n)) if ready is None else set(ready)
    bw = per_gpu_bandwidth(prof)
    ints, _, _ = G.mask_aware_star_weights(n, R, bw=bw)
    chunk, _ = chunk_from_profile(prof, tensor_bytes,
                                  text_for_chunk=lambda c: G.allreduce_stars(n, chunk=c, weights=ints))
    text = G.allreduce_stars(n, chunk=chunk, weights=ints)
    comm.set_strategy("allreduce", text)
    if set_default_chunk:
        comm.config("default_chunk", chunk)
    return text, prof, chunk


# -------------------------------------------------------------- cost model
def _trees(text):
    n, coll, nsubs = _A.strategy_check(text)
    subs = []
    for m in range(nsubs):
        w, chunk, parent, src = _A.strategy_sub(text, m)
        subs.append((w, chunk, parent))
    return n, subs


def link_loads(parent, noagg=frozenset(), broadcast=False):
    """N_ij for every tree edge (child -> parent) of one sub-collective."""
    n = len(parent)
    children = {g: [c for c in range(n) if parent[c] == g] for g in range(n)}
    loads = {}

    def out_flows(g):   # flows sent from g to its parent
        if broadcast or g not in noagg:
            return 1
        return 1 + sum(out_flows(c) for c in children[g])

    for g in range(n):
        if parent[g] != -1:
            loads[(g, parent[g])] = out_flows(g)
    return loads


def tree_time(parent, S_m, C_m, alpha, beta, shared_loads=None, noagg=frozenset()):
    """T of one Reduce tree (eqs. 2, 5, 6).  alpha[i][j], beta[i][j] per link
    (seconds, seconds per byte); shared_loads[(i, j)] = sum_m N^m_ij over all
    sub-collectives (eq. 3), defaults to this tree's own loads."""
    n = len(parent)
    loads = shared_loads or link_loads(parent, noagg)
    root = parent.index(-1)
    children = {g: [c for c in range(n) if parent[c] == g] for g in range(n)}

    def t(i, j):
        return alpha[i][j] + beta[i][j] * loads.get((i, j), 1) * C_m

    h = {}
    bottle = 0.0

    def ready(g):   # eq. 2 with aggregation: wait for the slowest in-flow
        nonlocal bottle
        if g in h:
            return h[g]
        best = 0.0
        for c in children[g]:
            best = max(best, ready(c) + t(c, g))
            bottle = max(bottle, t(c, g))
        h[g] = best
        return best

    h_root = ready(root)
    chunks = max(1, math.ceil(S_m / C_m))
    return h_root + chunks * bottle, h_root, bottle


def allreduce_time(text, S, alpha, beta, esize=4):
    """Predicted AllReduce time of a strategy for S bytes per rank: every tree
    reduces its partition and broadcasts it back along the reversed edges, both
    stages pipelined; the trees run concurrently sharing links (eq. 3)."""
    n, subs = _trees(text)
    W = sum(w for w, _, _ in subs)
    shared = {}
    for _, _, parent in subs:
        for e, v in link_loads(parent).items():
            shared[e] = shared.get(e, 0) + v
            shared[(e[1], e[0])] = shared.get((e[1], e[0]), 0) + 1   # broadcast back
    worst = 0.0
    for w, chunk, parent in subs:
        S_m = S * w / W
        if S_m <= 0:
            continue
        t_red, h_red, b_red = tree_time(parent, S_m, chunk, alpha, beta, shared)
        rev = {(j, i): 1 for (i, j) in link_loads(parent)}
        # broadcast stage: same tree, edges reversed, depth h_bcast
        depth = _depth(parent)
        t_edge = max((alpha[j][i] + beta[j][i] * shared.get((j, i), 1) * chunk for (j, i) in rev), default=0.0)
        h_b = depth * t_edge
        chunks = max(1, math.ceil(S_m / chunk))
        worst = max(worst, h_red + h_b + chunks * max(b_red, t_edge))
    return worst


def alltoall_paths(text):
    """Per a2a line m: (weight, chunk, {(s, d): [s, h1, .., d]}) read through
    the product's loader (adapcc_strategy_route)."""
    n, coll, nsubs = _A.strategy_check(text)
    out = []
    for m in range(nsubs):
        w, chunk, _, _ = _A.strategy_sub(text, m)
        paths = {(s, d): [s] + _A.strategy_route(text, m, s, d) + [d]
                 for s in range(n) for d in range(n) if s != d}
        out.append((w, chunk, paths))
    return n, out


def alltoall_link_loads(text, ready=None):
    """N_ij = sum over all lines' flows of x^f_ij (P:L209-211 with eq. 3's
    sum over sub-collectives).  ready: sources that send (default all)."""
    n, lines = alltoall_paths(text)
    src = set(range(n)) if ready is None else set(ready)
    loads = {}
    for _, _, paths in lines:
        for (s, _), p in paths.items():
            if s not in src:
                continue
            for e in zip(p[:-1], p[1:]):
                loads[e] = loads.get(e, 0) + 1
    return loads


def alltoall_time(text, S, alpha, beta, ready=None):
    """Predicted AlltoAll time, S bytes per (source, destination) block split
    over the a2a lines by weight; flows of every line share links (eq. 3)."""
    n, lines = alltoall_paths(text)
    src = set(range(n)) if ready is None else set(ready)
    loads = alltoall_link_loads(text, ready)
    W = sum(w for w, _, _ in lines)
    worst = 0.0
    for w, chunk, paths in lines:
        S_m = S * w / W
        if S_m <= 0:
            continue
        chunks = max(1, math.ceil(S_m / chunk))
        for (s, _), p in paths.items():
            if s not in src:
                continue
            ts = [alpha[i][j] + beta[i][j] * loads[(i, j)] * chunk for i, j in zip(p[:-1], p[1:])]
            worst = max(worst, sum(ts) + chunks * max(ts))
    return worst


def _depth(parent):
    d = 0
    for g in range(len(parent)):
        k, x = 0, g
        while parent[x] != -1:
            x, k = parent[x], k + 1
        d = max(d, k)
    return d


def best_chunk(text_for_chunk, S, alpha, beta, candidates=(1 << 14, 1 << 16, 1 << 18, 1 << 20, 1 << 22)):
    """Chunk size C minimising the predicted time ("identifies optimized chunk
    size to pipeline the transmission").  text_for_chunk(C) -> strategy."""
    scored = [(allreduce_time(text_for_chunk(c), S, alpha, beta), c) for c in candidates]
    return min(scored)[1], scored


def uniform_links(n, alpha, beta):
    """NVSwitch: every GPU pair has the same alpha, beta."""
    return [[alpha] * n for _ in range(n)], [[beta] * n for _ in range(n)]
