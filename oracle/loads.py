"""Link loads of AlltoAll strategies (§IV-D "Bandwidth Sharing").

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Routing (eq. 1): x^f_ij = 1 iff flow f traverses edge (i, j); every
flow leaves its source once, enters its destination once and is conserved at
every other node.  For AlltoAll "flows carry different parameters, and the
link load sums all traversing flows":  N^m_ij = sum_f x^f_ij.
Flows of AlltoAll: "each GPU sends multiple flows to all other GPUs",
i.e. one flow per ordered pair s != d; a block a rank keeps (s == d) crosses
no edge.  Under a ready mask only ready sources send.
"""

from .strategy import ESIZE, flow_path, parse, partition


def flow_edges(sub, s, d):
    """x^f_ij of flow s -> d as the list of edges (i, j) it traverses."""
    p = flow_path(sub, s, d)
    return list(zip(p[:-1], p[1:]))


def alltoall_link_loads(strategy_text, ready=None):
    """N^m_ij per a2a sub-collective m: list of {(i, j): count}."""
    st = parse(strategy_text)
    if st.collective != "alltoall":
        raise ValueError("alltoall strategy expected")
    n = st.nranks
    srcs = range(n) if ready is None else sorted(ready)
    out = []
    for sub in st.subs:
        N = {}
        for s in srcs:
            for d in range(n):
                if d == s:
                    continue
                for e in flow_edges(sub, s, d):
                    N[e] = N.get(e, 0) + 1
        out.append(N)
    return out


def alltoall_edge_bytes(strategy_text, count, dtype, ready):
    """Bytes every directed edge (i, j) carries in one AlltoAll of `count`
    elements per peer block: each block is split over the a2a lines by weight
    (partition, reading Q9) and line m's share travels along line m's route."""
    st = parse(strategy_text)
    es = ESIZE[dtype]
    b = partition(count, es, [sb.weight for sb in st.subs])
    out = {}
    for m, sub in enumerate(st.subs):
        nbytes = (b[m + 1] - b[m]) * es
        if nbytes == 0:
            continue
        for s in sorted(ready):
            for d in range(st.nranks):
                if d == s:
                    continue
                for e in flow_edges(sub, s, d):
                    out[e] = out.get(e, 0) + nbytes
    return out
