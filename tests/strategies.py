"""Strategy-text builders for tests (plain string formatting; no method arithmetic).

Kept in tests/ so that the oracle tests do not depend on the product's
generator; the product generator is tested separately against the oracle's
parser (tests/test_generator.py).
"""


def header(n, coll):
    return f"adapcc-strategy 1\nnranks {n}\ncollective {coll}\n"


def tree_line(parent, weight=1, chunk=262144, noagg=()):
    s = f"tree weight={weight} chunk={chunk} parent={','.join(map(str, parent))}"
    if noagg:
        s += " noagg=" + ",".join(map(str, noagg))
    return s + "\n"


def allreduce_trees(parents, weights=None, chunk=262144, noaggs=None):
    n = len(parents[0])
    weights = weights or [1] * len(parents)
    noaggs = noaggs or [()] * len(parents)
    return header(n, "allreduce") + "".join(
        tree_line(p, w, chunk, na) for p, w, na in zip(parents, weights, noaggs))


def star(n, root):
    return [-1 if g == root else root for g in range(n)]


def chain(order):
    """order[0] is the leaf ... order[-1] the root."""
    n = len(order)
    p = [None] * n
    for i, g in enumerate(order):
        p[g] = order[i + 1] if i + 1 < n else -1
    return p


def allreduce_stars(n, chunk=262144, weights=None):
    return allreduce_trees([star(n, m) for m in range(n)], weights, chunk)


def allreduce_ring(n, chunk=262144, weight=1, order=None):
    order = order if order is not None else list(range(n))
    return header(n, "allreduce") + (
        f"ring weight={weight} chunk={chunk} order={','.join(map(str, order))}\n")


def allgather_stars(n, chunk=262144, weight=1):
    return header(n, "allgather") + "".join(
        f"bcast src={s} weight={weight} chunk={chunk} parent={','.join(map(str, star(n, s)))}\n"
        for s in range(n))


def allgather_chains(n, chunk=1 << 20):
    out = header(n, "allgather")
    for s in range(n):
        order = [(s + k) % n for k in range(n - 1, -1, -1)]   # ..., s+1, s  (s is root)
        out += (f"bcast src={s} weight=1 chunk={chunk} "
                f"parent={','.join(map(str, chain(order)))}\n")
    return out


def alltoall_direct(n, chunk=1 << 20, lines=1):
    return header(n, "alltoall") + "".join(
        f"a2a weight=1 chunk={chunk}\n" for _ in range(lines))


def all_rooted_trees(n):
    """Every rooted labelled tree on n nodes as a parent array (n^(n-1) of them)."""
    import itertools
    out = []
    for cand in itertools.product(range(-1, n), repeat=n):
        if cand.count(-1) != 1 or any(cand[g] == g for g in range(n)):
            continue
        ok = True
        for g in range(n):
            x, k = g, 0
            while cand[x] != -1 and k <= n:
                x, k = cand[x], k + 1
            if k > n:
                ok = False
                break
        if ok:
            out.append(list(cand))
    return out
