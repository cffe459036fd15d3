"""Late join (NEXT-1) on the GPU vs the late-join oracle (-m gpu).

Deterministic cases: the late ranks signal before phase 1 (every piece folds
them) or never (phase 2 adds them all).  Racing case: a late rank signals from
a side stream while phase 1 runs; the inclusion is then timing-dependent, so
every work piece (the plan's unit of inclusion, from adapcc_plan_items) must
match the oracle for ONE inclusion set, the same set explaining both the
phase-1 and the final value of all its elements (the oracle never consumes
the GPU's decisions), and the race must produce a mixed outcome; int32
finals are exact."""

import itertools

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests import strategies as S  # noqa: E402
from tests.gpu_util import bits, empty_dev, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _comm(n, engine, mode="direct"):
    c = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=64 << 20)
    c.config("engine", engine)
    c.config("timeout_ms", 20000)
    return c


@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
@pytest.mark.parametrize("case", ["all", "none", "one"])
def test_late_join_deterministic(engine, dtype, case, mode):
    """STAGED: late ranks push their chunks to the roots themselves;
    DIRECT: roots read them.  Both kernels."""
    n, count = 8, 200_003
    R, late = {0, 1, 2, 4, 5, 7}, [3, 6]
    text = S.allreduce_trees([S.star(n, m) for m in range(n)] + [S.chain([0, 1, 2, 3, 4, 5, 6, 7])],
                             chunk=16384)
    xs = rank_tensors(dtype, count, n)
    comm = _comm(n, engine, mode)
    comm.set_strategy("allreduce", text)
    dx = [to_dev(x, dtype) for x in xs]
    dy = [empty_dev(count, dtype) for _ in range(n)]
    if case in ("all", "one"):
        t = comm.late_ticket() + 1          # the ticket the next LATE_JOIN call will use
        for r in (late if case == "all" else late[:1]):
            comm.signal_ready(r, ticket=t)
    comm.allreduce_lb(dx, dy, ready=R, late="join")
    torch.cuda.synchronize()
    # "one": rank 3 joins every piece, rank 6 none -> phase 2 runs every root piece, adding only 6
    L = set(late) if case == "all" else {late[0]} if case == "one" else set()
    e1 = oc.allreduce_late(xs, text, R, dtype, L, phase=1)
    assert all(np.array_equal(bits(to_host(y, dtype)), bits(e)) for y, e in zip(dy, e1))
    comm.allreduce_lb(dx, dy, ready=R, late="complement")
    torch.cuda.synchronize()
    e2 = oc.allreduce_late(xs, text, R, dtype, L, phase=2, y_prev=e1)
    assert all(np.array_equal(bits(to_host(y, dtype)), bits(e)) for y, e in zip(dy, e2))
    assert comm.get_async_error() == 0
    comm.finalize()


def _piece_ranges(text, count, dtype, R, grid, engine, mode="direct"):
    """Element ranges [a, b) of the work pieces of the LATE_JOIN plan the
    kernel runs (same grid, same item cutting): the unit of inclusion.
    STAGED: the root tasks' chunks (a star root writes its recv and its
    broadcast slot)."""
    mask = sum(1 << r for r in R)
    items, tasks = pkg.adapcc.plan_items(text, count, dtype, mask, grid, tma=engine == 1,
                                         late="join", mode=mode)
    if mode == "staged":
        items = items[(tasks[items["task"]]["ndst"] == 2) & (tasks[items["task"]]["nwait"] >= 1)]
    t = tasks[items["task"]]
    a = t["lo"] + items["chunk"].astype(np.uint64) * t["chunk_elems"] + items["off"]
    return np.stack([a, a + items["len"]], axis=1).astype(np.int64)


@pytest.mark.parametrize("engine,mode", [(0, "direct"), (1, "direct"), (0, "staged"), (1, "staged")])
@pytest.mark.parametrize("dtype", ["f32", "i32"])
def test_late_join_racing_signal(engine, dtype, mode):
    """Rank 3 signals from a side stream while phase 1 runs.  Per work piece
    (chunks "with the same offset" join), ONE inclusion set must
    explain every element of the piece in both phases; across lags the race
    must produce a mixed outcome (some pieces with rank 3, some without)."""
    n, count, grid = 8, 4_000_003, 32
    R, late = {0, 1, 2, 4, 5, 7}, [3, 6]
    text = G.allreduce_stars(n, chunk=65536)
    xs = rank_tensors(dtype, count, n)
    comm = _comm(n, engine, mode)
    comm.config("max_ctas", grid)       # the piece cut below uses the same grid
    comm.set_strategy("allreduce", text)
    dx = [to_dev(x, dtype) for x in xs]
    dy = [empty_dev(count, dtype) for _ in range(n)]
    comm.allreduce_lb(dx, dy)  # warm-up (plans, clocks)
    torch.cuda.synchronize()
    pieces = _piece_ranges(text, count, dtype, R, grid, engine, mode)
    covered = np.zeros(count, np.int32)
    for a, b in pieces:
        covered[a:b] += 1
    assert (covered == 1).all(), "pieces must tile the tensor"
    options = [set(c) for k in range(3) for c in itertools.combinations(late, k)]
    expect = []
    for L in options:
        p1 = oc.allreduce_late(xs, text, R, dtype, L, phase=1)[0]
        p2 = oc.allreduce_late(xs, text, R, dtype, L, phase=2, y_prev=[p1])[0]
        expect.append((bits(p1), bits(p2)))
    side, main = torch.cuda.Stream(), torch.cuda.Stream()
    main.wait_stream(torch.cuda.current_stream())
    outcomes = set()
    # grid 32: phase 1 runs for hundreds of microseconds, so a lag sweep lands
    # the signal inside it despite the host's launch jitter
    for lag in (20_000, 50_000, 100_000, 200_000, 400_000, 800_000, 1_600_000):
        t = comm.late_ticket() + 1
        start = torch.cuda.Event()
        start.record(main)
        side.wait_event(start)
        with torch.cuda.stream(side):
            torch.cuda._sleep(lag)             # rank 3 finishes "compute" while phase 1 runs
            comm.signal_ready(3, ticket=t, stream=side)
        comm.allreduce_lb(dx, dy, ready=R, late="join", stream=main)
        main.synchronize()
        y1 = [to_host(y, dtype) for y in dy]
        comm.allreduce_lb(dx, dy, ready=R, late="complement", stream=main)
        main.synchronize()
        y2 = [to_host(y, dtype) for y in dy]
        side.synchronize()
        assert comm.get_async_error() == 0
        for g in range(1, n):                   # broadcast identity
            assert np.array_equal(bits(y1[g]), bits(y1[0])) and np.array_equal(bits(y2[g]), bits(y2[0]))
        match = [(bits(y1[0]) == e1) & (bits(y2[0]) == e2) for e1, e2 in expect]
        csum = [np.concatenate([[0], np.cumsum(m)]) for m in match]
        for a, b in pieces:
            fits = [k for k in range(len(options)) if csum[k][b] - csum[k][a] == b - a]
            assert fits, f"piece [{a},{b}) not explained by one inclusion set (lag {lag})"
            outcomes.add(3 in options[fits[0]] if len(fits) == 1 else None)
        if dtype == "i32":
            assert np.array_equal(y2[0], oc.allreduce_exact(xs, set(range(n)), "i32"))
        if True in outcomes and False in outcomes:
            break
    assert True in outcomes and False in outcomes, f"no mixed outcome in any lag: {outcomes}"
    torch.cuda.synchronize()
    comm.finalize()


@pytest.mark.parametrize("engine", [0, 1])
def test_late_join_interleaved_plans(engine):
    """Phase-1 / phase-2 pairs of two plans interleave on one stream
    (phase 1 A, phase 1 B, phase 2 A, phase 2 B): each phase 2 complements
    its own plan's phase 1.  A second phase 2 adds nothing."""
    n = 8
    R, late = {0, 1, 2, 4, 5, 7}, [3, 6]
    text = G.allreduce_stars(n, chunk=65536)
    comm = _comm(n, engine)
    comm.set_strategy("allreduce", text)
    cA, cB = 1_000_003, 600_011
    xA, xB = rank_tensors("i32", cA, n), rank_tensors("i32", cB, n, base=1500)
    dA, dB = [to_dev(x, "i32") for x in xA], [to_dev(x, "i32") for x in xB]
    yA, yB = [empty_dev(cA, "i32") for _ in range(n)], [empty_dev(cB, "i32") for _ in range(n)]
    tA = comm.late_ticket() + 1
    comm.signal_ready(3, ticket=tA)             # rank 3 joins A's phase 1, not B's (ticket tA + 1)
    comm.allreduce_lb(dA, yA, ready=R, late="join")
    comm.allreduce_lb(dB, yB, ready=R, late="join")
    torch.cuda.synchronize()
    eA1 = oc.allreduce_late(xA, text, R, "i32", {3}, phase=1)
    eB1 = oc.allreduce_late(xB, text, R, "i32", set(), phase=1)
    assert all(np.array_equal(to_host(y, "i32"), e) for y, e in zip(yA, eA1))
    assert all(np.array_equal(to_host(y, "i32"), e) for y, e in zip(yB, eB1))
    comm.allreduce_lb(dA, yA, ready=R, late="complement")
    comm.allreduce_lb(dB, yB, ready=R, late="complement")
    comm.allreduce_lb(dA, yA, ready=R, late="complement")   # nothing left to add
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    fA, fB = oc.allreduce_exact(xA, set(range(n)), "i32"), oc.allreduce_exact(xB, set(range(n)), "i32")
    assert all(np.array_equal(to_host(y, "i32"), fA) for y in yA)
    assert all(np.array_equal(to_host(y, "i32"), fB) for y in yB)
    comm.finalize()


@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("engine", [0, 1])
def test_late_join_graph_replay(engine, mode):
    """Phase 1 + phase 2 captured in one CUDA graph (the ticket is baked in) and replayed: every replay
    rebuilds phase 1's list of incomplete pieces from scratch (phase 2 empties its list when it ends),
    so rank 6 is added exactly once per replay (int32, exact) while rank 3 joins every piece."""
    n, count = 8, 300_007
    R, late = {0, 1, 2, 4, 5, 7}, [3, 6]
    text = G.allreduce_stars(n, chunk=65536)
    xs = rank_tensors("i32", count, n)
    comm = _comm(n, engine, mode)
    comm.set_strategy("allreduce", text)
    dx = [to_dev(x, "i32") for x in xs]
    dy = [empty_dev(count, "i32") for _ in range(n)]
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        comm.allreduce_lb(dx, dy, ready=R, late="join")       # plan built outside the capture
        comm.allreduce_lb(dx, dy, ready=R, late="complement")
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            t = comm.late_ticket() + 1
            comm.signal_ready(late[0], ticket=t, stream=s)
            comm.allreduce_lb(dx, dy, ready=R, late="join", stream=s)
            comm.allreduce_lb(dx, dy, ready=R, late="complement", stream=s)
    full = oc.allreduce(xs, text, set(range(n)), "i32")
    for _ in range(3):
        for y in dy:
            y.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert comm.get_async_error() == 0
        for y, e in zip(dy, full):
            assert np.array_equal(bits(to_host(y, "i32")), bits(e))
    comm.finalize()


def test_late_join_rejects_aliased_late_input():
    """A late rank's input is read after phase 1 wrote its recvbuf: in-place
    late join would fold the phase-1 result instead of the gradient."""
    n = 4
    comm = _comm(n, 0)
    xs = [torch.ones(4096, device="cuda") for _ in range(n)]
    ys = [torch.empty_like(x) for x in xs]
    ys[3] = xs[3]                                   # rank 3 (late) in place
    with pytest.raises(pkg.AdapccError) as e:
        comm.allreduce_lb(xs, ys, ready={0, 1, 2}, late="join")
    assert e.value.code == pkg.adapcc.INVALID_ARGUMENT
    ys[3] = torch.empty_like(xs[3])
    ys[0] = xs[0]                                   # a ready rank in place is fine
    comm.allreduce_lb(xs, ys, ready={0, 1, 2}, late="join")
    torch.cuda.synchronize()
    comm.finalize()
