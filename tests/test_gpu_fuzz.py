"""Randomised GPU parity sweep (-m gpu): random trees (shape, root, noagg),
weights, chunk sizes, counts (1 element .. 3 M, ragged), masks, dtypes,
plans (DIRECT / STAGED), kernels (LDG, TMA, auto), LDG schedules, PDL on/off
and piece sizes, every collective the
loopback communicator offers; bit-exact against the oracle.  Seeded: a
failure names its case and reproduces."""

import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests.gpu_util import bits, empty_dev, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _random_tree(rng, n):
    """Random labelled tree: random attachment order, random root."""
    order = [int(v) for v in rng.permutation(n)]
    parent = [-1] * n
    for i in range(1, n):
        parent[order[i]] = order[int(rng.integers(0, i))]
    return parent


def _case(seed, large=False, n=None):
    rng = np.random.default_rng(seed + (100_000 if large else 0))
    n = int(rng.integers(2, 9)) if n is None else n
    coll = ["allreduce", "allreduce", "allgather", "alltoall", "reducescatter"][int(rng.integers(0, 5))]
    dtype = ["f32", "bf16", "i32"][int(rng.integers(0, 3))]
    big = rng.random() < 0.3
    count = int(np.exp(rng.uniform(0, np.log(3e6 if big else 2e4))))
    if large:
        count = int(np.exp(rng.uniform(np.log(2e5), np.log(4e6))))
    if coll in ("alltoall", "allgather", "reducescatter"):
        count = max(1, count // n)
    chunk = 16 * int(np.exp(rng.uniform(np.log(4), np.log((8 << 20) // 16))))
    if large:
        chunk = 16 * int(np.exp(rng.uniform(np.log(4096), np.log((8 << 20) // 16))))
    mode = ["direct", "staged"][int(rng.integers(0, 2))]
    engine = int(rng.integers(0, 3))
    if engine == 2 and np.random.default_rng(seed + (8_300_000 if large else 8_200_000)).random() < 0.5:
        engine = 3   # flat kernel (its own stream: the other draws keep their values)
    ready = {g for g in range(n) if rng.random() < 0.75}
    if rng.random() < 0.2:
        ready = set(range(n))
    m = int(rng.integers(1, 4))
    # r02 knobs from their own stream: relay=store on allreduce trees, bulk reduce-add ACCUMULATE on/off
    r3 = np.random.default_rng(seed + (8_100_000 if large else 8_000_000))
    relay = "store" if r3.random() < 0.3 else None
    acc_red = int(r3.integers(0, 2))
    if coll == "allreduce":
        parents = [_random_tree(rng, n) for _ in range(m)]
        noaggs = [[g for g in range(n) if p[g] != -1 and rng.random() < 0.25] for p in parents]
        text = G.allreduce_trees(parents, [int(rng.integers(1, 5)) for _ in range(m)], chunk, noaggs, relay=relay)
    elif coll == "allgather":
        text = G._header(n, "allgather")
        for s in range(n):
            for _ in range(int(rng.integers(1, 3))):
                p = _random_tree(rng, n)
                # re-root at s: swap labels of the root and s
                r = p.index(-1)
                sw = {r: s, s: r}
                q = [-1] * n
                for g in range(n):
                    pg = p[g]
                    q[sw.get(g, g)] = -1 if pg == -1 else sw.get(pg, pg)
                text += f"bcast src={s} weight={int(rng.integers(1, 4))} chunk={chunk} parent={G._join(q)}\n"
    elif coll == "alltoall":
        lines = []
        for _ in range(m):
            routes = {}
            for s in range(n):
                for d in range(n):
                    if s != d and n > 2 and rng.random() < 0.3:
                        others = [g for g in range(n) if g not in (s, d)]
                        k = int(rng.integers(1, min(3, len(others)) + 1))
                        routes[(s, d)] = [int(v) for v in rng.choice(others, k, replace=False)]
            lines.append((int(rng.integers(1, 4)), routes))
        text = G.alltoall_routed(n, lines, chunk)
    else:
        text = G._header(n, "reducescatter")
        for b in range(n):
            p = _random_tree(rng, n)
            r = p.index(-1)
            sw = {r: b, b: r}
            q = [-1] * n
            for g in range(n):
                pg = p[g]
                q[sw.get(g, g)] = -1 if pg == -1 else sw.get(pg, pg)
            text += f"rtree dst={b} weight=1 chunk={chunk} parent={G._join(q)}\n"
    # launch knobs from their own stream (the cases above stay as they were):
    # LDG schedule (dynamic claims / static blobs), programmatic dependent
    # launch, work-piece size (0 = automatic)
    r2 = np.random.default_rng(seed + (7_100_000 if large else 7_000_000))
    knobs = dict(sched=int(r2.choice([0, 2])), pdl=int(r2.integers(0, 2)),
                 piece_kib=int(r2.choice([0, 0, 16, 48, 512])))
    return dict(n=n, coll=coll, dtype=dtype, count=count, mode=mode, engine=engine, ready=ready, text=text,
                seed=seed, acc_red=acc_red, **knobs)


def _eq(a, b):
    return np.array_equal(bits(a), bits(b))


FUZZ_CASES = int(os.environ.get("ADAPCC_FUZZ_CASES", "1000"))  # widen the sweep for one-off soak runs


@pytest.mark.parametrize("seed", range(FUZZ_CASES))
def test_fuzz(seed):
    _run(_case(seed))


@pytest.mark.parametrize("seed", range(60))
def test_fuzz_large(seed):
    """Large counts and chunks: multi-tile items in both kernels."""
    _run(_case(seed, large=True))


def _run(c):
    seed = c["seed"]
    n, dtype, count, R, text = c["n"], c["dtype"], c["count"], c["ready"], c["text"]
    es = 4 if dtype != "bf16" else 2
    per_rank = count * (n if c["coll"] in ("alltoall", "reducescatter") else 1)
    out_per_rank = count * (n if c["coll"] in ("alltoall", "allgather") else 1)
    scratch = 4 * max(per_rank, out_per_rank) * es + (32 << 20)
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=scratch, mode=c["mode"])
    comm.config("timeout_ms", 20000)
    comm.config("engine", c["engine"])
    for k in ("sched", "pdl", "piece_kib", "acc_red"):
        comm.config(k, c[k])
    comm.set_strategy(c["coll"], text)
    xs = rank_tensors(dtype, per_rank, n, base=5000 + seed)
    prev = [rank_tensors(dtype, out_per_rank, 1, base=6000 + 7 * seed + g)[0] for g in range(n)]
    dx = [to_dev(x, dtype) if g in R else None for g, x in enumerate(xs)]
    dy = [to_dev(p, dtype) for p in prev]
    if c["coll"] == "allreduce":
        acc = seed % 3 == 0
        comm.allreduce_lb(dx, dy, ready=R, accumulate=acc)
        exp = oc.allreduce(xs, text, R, dtype, accumulate=acc, y_prev=prev)
    elif c["coll"] == "allgather":
        comm.allgather_lb(dx, dy, ready=R)
        exp = oc.allgather(xs, text, R, dtype, prev)
    elif c["coll"] == "alltoall":
        comm.alltoall_lb(dx, dy, ready=R)
        exp = oc.alltoall(xs, text, R, dtype, prev)
    else:
        comm.reducescatter_lb(dx, dy, ready=R)
        exp = oc.reducescatter(xs, text, R, dtype, y_prev=prev)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0, c
    for g in range(n):
        assert _eq(to_host(dy[g], dtype), exp[g]), (g, {k: v for k, v in c.items() if k != "text"}, text)
    comm.finalize()


# ------------------------------------------------------------- late join (NEXT-1)
@pytest.mark.parametrize("seed", range(200))
def test_fuzz_late_join(seed):
    """Random trees / noagg / weights / chunks / counts / ready sets, both
    plans and kernels: a random subset L of the late ranks signals before
    phase 1 (so every piece includes exactly L), phase 2 adds the rest;
    both phases bit-exact against oracle.allreduce_late (R4, R10)."""
    rng = np.random.default_rng(9_000_000 + seed)
    n = int(rng.integers(3, 9))
    dtype = ["f32", "bf16", "i32"][int(rng.integers(0, 3))]
    count = int(np.exp(rng.uniform(np.log(50), np.log(2e6))))
    chunk = 16 * int(np.exp(rng.uniform(np.log(64), np.log((4 << 20) // 16))))
    mode = ["direct", "staged"][int(rng.integers(0, 2))]
    engine = int(rng.integers(0, 3))
    m = int(rng.integers(1, 4))
    parents = [_random_tree(rng, n) for _ in range(m)]
    noaggs = [[g for g in range(n) if p[g] != -1 and rng.random() < 0.2] for p in parents]
    text = G.allreduce_trees(parents, [int(rng.integers(1, 5)) for _ in range(m)], chunk, noaggs)
    late = sorted(int(g) for g in rng.choice(n, int(rng.integers(1, n)), replace=False))
    R = set(range(n)) - set(late)
    L = {g for g in late if rng.random() < 0.5}
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=8 * count * 4 + (32 << 20), mode=mode)
    comm.config("timeout_ms", 20000)
    comm.config("engine", engine)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors(dtype, count, n, base=9100 + seed)
    dx = [to_dev(x, dtype) for x in xs]
    dy = [empty_dev(count, dtype) for _ in range(n)]
    t = comm.late_ticket() + 1
    for g in L:
        comm.signal_ready(g, ticket=t)
    comm.allreduce_lb(dx, dy, ready=R, late="join")
    torch.cuda.synchronize()
    e1 = oc.allreduce_late(xs, text, R, dtype, L, phase=1)
    case = dict(seed=seed, n=n, dtype=dtype, count=count, mode=mode, engine=engine, late=late, L=sorted(L))
    for g in range(n):
        assert _eq(to_host(dy[g], dtype), e1[g]), ("phase 1", g, case, text)
    comm.allreduce_lb(dx, dy, ready=R, late="complement")
    torch.cuda.synchronize()
    e2 = oc.allreduce_late(xs, text, R, dtype, L, phase=2, y_prev=e1)
    assert comm.get_async_error() == 0, case
    for g in range(n):
        assert _eq(to_host(dy[g], dtype), e2[g]), ("phase 2", g, case, text)
    comm.finalize()


# ------------------------------------------------------------- NVLS (NEXT-2)
@pytest.mark.parametrize("seed", range(60))
def test_fuzz_nvls_emulated(seed):
    """Random mixtures of nvls lines and trees on the loopback-emulated switch:
    int32 exact, fp32 / bf16 within the switch's any-order bound (R9)."""
    from oracle import bf16 as obf
    rng = np.random.default_rng(9_500_000 + seed)
    n = int(rng.integers(2, 9))
    dtype = ["f32", "bf16", "i32"][int(rng.integers(0, 3))]
    count = int(np.exp(rng.uniform(np.log(20), np.log(2e6))))
    chunk = 16 * int(np.exp(rng.uniform(np.log(64), np.log((2 << 20) // 16))))
    mode = ["direct", "staged"][int(rng.integers(0, 2))]
    lines = [f"nvls weight={int(rng.integers(1, 6))} chunk={chunk}" for _ in range(int(rng.integers(1, 3)))]
    for _ in range(int(rng.integers(0, 3))):
        lines.append(f"tree weight={int(rng.integers(1, 4))} chunk={chunk} parent={G._join(_random_tree(rng, n))}")
    order = [int(i) for i in rng.permutation(len(lines))]
    text = G._header(n, "allreduce") + "\n".join(lines[i] for i in order) + "\n"
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=8 * count * 4 + (32 << 20), mode=mode)
    ok, why = comm.nvls_setup(2 * count * 4 + (1 << 20))
    assert ok, why
    comm.set_strategy("allreduce", text)
    xs = rank_tensors(dtype, count, n, base=9600 + seed)
    dy = [empty_dev(count, dtype) for _ in range(n)]
    comm.allreduce_lb([to_dev(x, dtype) for x in xs], dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    exp = oc.allreduce(xs, text, set(range(n)), dtype)
    got = [to_host(y, dtype) for y in dy]
    case = dict(seed=seed, n=n, dtype=dtype, count=count, mode=mode)
    for g in range(n):
        if dtype == "i32":
            assert np.array_equal(got[g], exp[g]), (g, case, text)
        else:
            f = (lambda a: obf.to_f32(a).astype(np.float64)) if dtype == "bf16" else (lambda a: a.astype(np.float64))
            den = np.sum(np.abs(np.stack([f(x) for x in xs])), axis=0) + 1e-30
            # tree partitions replay bit-exactly within the same bound; nvls ones are order-free
            assert np.max(np.abs(f(got[g]) - f(exp[g])) / den) <= 2 * oc.nvls_tolerance(dtype, n) + 1e-12, (g, case)
    comm.finalize()
