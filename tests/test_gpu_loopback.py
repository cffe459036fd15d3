"""GPU parity: the CUDA engine through the C ABI vs the CPU oracle (-m gpu).

Loopback mode hosts n virtual ranks on one B200; DIRECT runs the single-copy
plan, STAGED runs exactly the multi-process protocol (landing slots, broadcast
slots, per-chunk flags).  Bar (BASELINE north star): bit-exact for int32,
AllGather and AlltoAll, and for fp32 / bf16 because the oracle replays the
strategy's reduction order; additionally within 1e-6 (fp32) / 1e-2 (bf16,
star trees) relative error of the fp64 definition.
"""

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

MODES = ["direct", "staged"]
ENGINES = [0, 1, 3]   # 0: LDG/STG fold kernel, 1: TMA bulk-copy pipeline kernel, 3: flat (flag-free plans; others fall back)


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _comm(n, mode, scratch=64 << 20, engine=2):
    c = pkg.Communicator.loopback(n, device=0, scratch_bytes=scratch, mode=mode)
    c.config("timeout_ms", 20000)
    c.config("engine", engine)
    return c


def _run_allreduce(comm, xs, dtype, ready, accumulate=False, prev=None, in_place=False):
    n = comm.nranks
    count = len(next(x for x in xs if x is not None)) if any(x is not None for x in xs) else len(prev[0])
    dx = [to_dev(x, dtype) if x is not None else None for x in xs]
    if in_place:
        dy = dx
    elif prev is not None:
        dy = [to_dev(p, dtype) for p in prev]
    else:
        dy = [empty_dev(count, dtype) for _ in range(n)]
    comm.allreduce_lb(dx, dy, ready=ready, accumulate=accumulate)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    return [to_host(y, dtype) for y in dy]


def _assert_bits(got, exp, ctx):
    for g, (a, b) in enumerate(zip(got, exp)):
        ba, bb = bits(a), bits(b)
        if not np.array_equal(ba, bb):
            bad = np.nonzero(ba != bb)[0]
            raise AssertionError(f"{ctx}: rank {g}: {len(bad)} mismatches, first at {bad[:5]}: "
                                 f"got {ba[bad[:5]]} exp {bb[bad[:5]]}")


ALLREDUCE_STRATS = {
    "stars8": lambda n: G.allreduce_stars(n, chunk=4096),
    "stars2roots": lambda n: G.allreduce_stars(n, chunk=8192, roots=[0, 1], weights=[3, 1]),
    "ring": lambda n: G.allreduce_ring(n, chunk=2048),
    "dbinary": lambda n: G.allreduce_double_binary(n, chunk=1024),
    "mixed_noagg": lambda n: S.allreduce_trees(
        [S.chain(list(range(n))), S.star(n, n - 1), [1] + [-1] + [0] * (n - 2)],
        weights=[2, 1, 3], chunk=1024, noaggs=[(), (), (0, 2)]),
}


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
@pytest.mark.parametrize("strat", list(ALLREDUCE_STRATS))
@pytest.mark.parametrize("engine", ENGINES)
def test_allreduce_parity(mode, dtype, strat, engine):
    n = 8 if strat != "mixed_noagg" else 5
    count = 100_003  # ragged: not a multiple of any vector width
    text = ALLREDUCE_STRATS[strat](n)
    comm = _comm(n, mode, engine=engine)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors(dtype, count, n)
    for mask in ((1 << n) - 1, 0b10110111 & ((1 << n) - 1), 0b1, 1 << (n - 1)):
        R = {r for r in range(n) if mask >> r & 1}
        xr = [x if r in R else None for r, x in enumerate(xs)]
        got = _run_allreduce(comm, xr, dtype, R)
        exp = oc.allreduce(xs, text, R, dtype)
        _assert_bits(got, exp, f"{strat}/{mode}/{dtype}/mask={mask:#x}")
        if dtype == "f32" or (dtype == "bf16" and strat.startswith("stars")):
            ex = oc.allreduce_exact(xs, R, dtype)
            g0 = got[0].astype(np.float64) if dtype == "f32" else \
                (got[0].astype(np.uint32) << 16).view(np.float32).astype(np.float64)
            den = np.max(np.abs(ex)) + 1e-30
            tol = 1e-6 if dtype == "f32" else 1e-2
            assert np.max(np.abs(g0 - ex)) / den <= tol
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("engine", ENGINES)
def test_c1_config_bit_exact(mode, engine):
    """BASELINE config C1: fp32 1M elements, 2 ranks, single tree, chunk 256 KB."""
    n, count = 2, 1 << 20
    text = S.allreduce_trees([[-1, 0]], chunk=262144)
    comm = _comm(n, mode, engine=engine)
    comm.set_strategy("allreduce", text)
    for dtype, dist in (("f32", "normal"), ("i32", "int")):
        xs = rank_tensors(dtype, count, n, dist=dist)
        got = _run_allreduce(comm, xs, dtype, {0, 1})
        _assert_bits(got, oc.allreduce(xs, text, {0, 1}, dtype), f"C1/{mode}/{dtype}")
    comm.finalize()


@pytest.mark.parametrize("acc_red", [1, 0])
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
@pytest.mark.parametrize("engine", ENGINES + [2])
def test_phase1_phase2_accumulate(mode, dtype, engine, acc_red):
    """C3 shape (reduced): stragglers {3,6} relay in phase 1, join with ACCUMULATE
    (TMA kernel: bulk reduce-add into recv, or the shared-memory read-modify-write;
    engine 2 = auto: this small DIRECT phase 2 runs on the flat kernel)."""
    n, count = 8, 65_537
    R1, R2 = {0, 1, 2, 4, 5, 7}, {3, 6}
    xs = rank_tensors(dtype, count, n)
    t1 = G.allreduce_mask_aware_stars(n, R1, chunk=8192)
    t2 = G.allreduce_mask_aware_stars(n, R2, chunk=8192)
    comm = _comm(n, mode, engine=engine)
    comm.config("acc_red", acc_red)
    comm.set_strategy("allreduce", t1)
    y1 = _run_allreduce(comm, [x if r in R1 else None for r, x in enumerate(xs)], dtype, R1)
    e1 = oc.allreduce(xs, t1, R1, dtype)
    _assert_bits(y1, e1, "phase1")
    comm.set_strategy("allreduce", t2)
    y2 = _run_allreduce(comm, [x if r in R2 else None for r, x in enumerate(xs)], dtype, R2,
                        accumulate=True, prev=y1)
    _assert_bits(y2, oc.allreduce(xs, t2, R2, dtype, accumulate=True, y_prev=e1), "phase2")
    if engine == 2 and mode == "direct":
        assert comm.last_engine() == 3   # auto: small flag-free ACCUMULATE -> flat kernel
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("engine", ENGINES)
def test_empty_mask_and_in_place(mode, engine):
    n, count = 4, 3001
    comm = _comm(n, mode, engine=engine)
    xs = rank_tensors("f32", count, n)
    text = G.allreduce_stars(n, chunk=512)
    comm.set_strategy("allreduce", text)
    got = _run_allreduce(comm, xs, "f32", set())
    _assert_bits(got, [np.zeros(count, np.float32)] * n, "empty")
    prev = [x.copy() for x in xs]
    got = _run_allreduce(comm, [None] * n, "f32", set(), accumulate=True, prev=prev)
    _assert_bits(got, prev, "empty-accumulate")
    got = _run_allreduce(comm, xs, "f32", {0, 2, 3}, in_place=True)
    _assert_bits(got, oc.allreduce(xs, text, {0, 2, 3}, "f32"), "in-place")
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["bf16", "f32"])
@pytest.mark.parametrize("strat", ["stars", "chains"])
@pytest.mark.parametrize("engine", ENGINES)
def test_allgather_parity(mode, dtype, strat, engine):
    n, cnt = 6, 10_001
    text = (G.allgather_stars(n, chunk=4096) if strat == "stars"
            else G.allgather_chains(n, chunk=2048))
    comm = _comm(n, mode, engine=engine)
    comm.set_strategy("allgather", text)
    xs = rank_tensors(dtype, cnt, n)
    for R in (set(range(n)), {1, 4}):
        prev = [rank_tensors(dtype, n * cnt, 1, base=77 + g)[0] for g in range(n)]
        dx = [to_dev(x, dtype) for x in xs]
        dy = [to_dev(p, dtype) for p in prev]
        comm.allgather_lb(dx, dy, ready=R)
        torch.cuda.synchronize()
        got = [to_host(y, dtype) for y in dy]
        _assert_bits(got, oc.allgather(xs, text, R, dtype, prev), f"allgather/{strat}/{mode}")
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["bf16", "i32"])
@pytest.mark.parametrize("engine", ENGINES)
def test_alltoall_parity(mode, dtype, engine):
    n, cnt = 8, 4099
    text = G.alltoall_direct(n, chunk=2048, lines=3)
    comm = _comm(n, mode, engine=engine)
    comm.set_strategy("alltoall", text)
    xs = rank_tensors(dtype, n * cnt, n)
    for R in (set(range(n)), {0, 5, 6}):
        prev = [rank_tensors(dtype, n * cnt, 1, base=300 + g)[0] for g in range(n)]
        dx = [to_dev(x, dtype) for x in xs]
        dy = [to_dev(p, dtype) for p in prev]
        comm.alltoall_lb(dx, dy, ready=R)
        torch.cuda.synchronize()
        got = [to_host(y, dtype) for y in dy]
        _assert_bits(got, oc.alltoall(xs, text, R, dtype, prev), f"alltoall/{mode}")
    comm.finalize()


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("mode", MODES)
def test_strategy_swap_mid_stream(mode, engine):
    """C5 shape (reduced): AllGather stream with a strategy swap at call 6 of 12,
    all calls enqueued back to back on one stream."""
    n, cnt = 4, 6400
    comm = _comm(n, mode, engine=engine)
    t_a, t_b = G.allgather_stars(n, chunk=4096), G.allgather_chains(n, chunk=8192)
    comm.set_strategy("allgather", t_a)
    xs_all, outs = [], []
    for call in range(12):
        if call == 6:
            comm.set_strategy("allgather", t_b)
        xs = rank_tensors("bf16", cnt, n, base=5000 + 10 * call)
        dx = [to_dev(x, "bf16") for x in xs]
        dy = [empty_dev(n * cnt, "bf16") for _ in range(n)]
        comm.allgather_lb(dx, dy)
        xs_all.append(xs)
        outs.append((dx, dy))
    torch.cuda.synchronize()
    for call, (xs, (_, dy)) in enumerate(zip(xs_all, outs)):
        exp = np.concatenate(xs)
        for y in dy:
            assert np.array_equal(to_host(y, "bf16"), exp), call
    comm.finalize()


@pytest.mark.parametrize("engine", ENGINES)
def test_segmented_call_when_arena_small(engine):
    n, count = 4, 1 << 20
    comm = _comm(n, "staged", scratch=1 << 20, engine=engine)
    text = G.allreduce_stars(n, chunk=16384)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors("f32", count, n)
    before = comm.launch_count()
    got = _run_allreduce(comm, xs, "f32", set(range(n)))
    assert comm.launch_count() - before > 1
    _assert_bits(got, oc.allreduce(xs, text, set(range(n)), "f32"), "segmented")
    comm.finalize()


@pytest.mark.parametrize("engine", ENGINES)
def test_watchdog_reports_timeout(engine):
    n = 4
    comm = _comm(n, "staged", engine=engine)
    comm.config("timeout_ms", 300)
    comm.config("debug_drop_rank", 2)
    xs = [to_dev(x, "f32") for x in rank_tensors("f32", 4096, n)]
    ys = [empty_dev(4096, "f32") for _ in range(n)]
    comm.allreduce_lb(xs, ys)
    torch.cuda.synchronize()
    assert comm.get_async_error() == pkg.adapcc.TIMEOUT
    with pytest.raises(pkg.AdapccError) as e:
        comm.allreduce_lb(xs, ys)
    assert e.value.code == pkg.adapcc.TIMEOUT
    comm.finalize()


def test_argument_errors():
    n = 2
    comm = _comm(n, "direct")
    x = [torch.zeros(64, device="cuda") for _ in range(n)]
    y = [torch.zeros(64, device="cuda") for _ in range(n)]
    with pytest.raises(pkg.AdapccError) as e:
        comm.allreduce_lb(x, y, ready=0b100)          # bit >= nranks
    assert e.value.code == pkg.adapcc.INVALID_ARGUMENT
    with pytest.raises(pkg.AdapccError) as e:
        comm.allreduce_lb([t[1:] for t in x], [t[1:] for t in y])   # misaligned
    assert e.value.code == pkg.adapcc.INVALID_ARGUMENT
    with pytest.raises(pkg.AdapccError) as e:
        comm.set_strategy("allreduce", G.allreduce_stars(3))     # wrong nranks
    assert e.value.code == pkg.adapcc.INVALID_STRATEGY
    with pytest.raises(pkg.AdapccError) as e:
        comm.alltoall_lb(x, x)                                    # aliasing
    assert e.value.code == pkg.adapcc.INVALID_ARGUMENT
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("engine", ENGINES)
def test_cuda_graph_capture_and_replay(mode, engine):
    """Calls are capturable once their plan is cached (warm-up call first)."""
    n, count = 4, 50_001
    comm = _comm(n, mode, engine=engine)
    text = G.allreduce_stars(n, chunk=16384)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors("f32", count, n)
    dx = [to_dev(x, "f32") for x in xs]
    dy = [empty_dev(count, "f32") for _ in range(n)]
    comm.allreduce_lb(dx, dy)          # warm-up builds and uploads the plan
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        comm.allreduce_lb(dx, dy)
        comm.allreduce_lb(dx, dy)
    exp = oc.allreduce(xs, text, set(range(n)), "f32")
    for rep in range(3):   # epochs advance on the device: replays never see stale flags
        for t in dy:
            t.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert comm.get_async_error() == 0
        _assert_bits([to_host(t, "f32") for t in dy], exp, f"graph replay {rep}")
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("n", [2, 3, 5])
def test_tma_large_items(mode, dtype, n):
    """Items whose shared-memory tile exceeds one consumer round: K = 2, 3
    folds and the K = 1 accumulate copy of phase 2 with 64 KiB stages (DIRECT
    plans), chunks of 4 MiB so every item spans many tiles."""
    count = (3 << 20) + 5
    es = 4 if dtype == "f32" else 2
    comm = _comm(n, mode, scratch=3 * count * es + (64 << 20), engine=1)
    xs = rank_tensors(dtype, count, n)
    for text in (G.allreduce_stars(n, chunk=4 << 20), G.allreduce_ring(n, chunk=4 << 20)):
        comm.set_strategy("allreduce", text)
        got = _run_allreduce(comm, xs, dtype, set(range(n)))
        _assert_bits(got, oc.allreduce(xs, text, set(range(n)), dtype), f"large/{n}/{mode}")
        # phase 1 without rank 0, phase 2 = rank 0 alone with ACCUMULATE (K = 1 + accumulate)
        R1 = set(range(1, n))
        p1 = _run_allreduce(comm, [x if r in R1 else None for r, x in enumerate(xs)], dtype, R1)
        got = _run_allreduce(comm, [xs[0]] + [None] * (n - 1), dtype, {0}, accumulate=True, prev=p1)
        exp1 = oc.allreduce(xs, text, R1, dtype)
        _assert_bits(got, oc.allreduce(xs, text, {0}, dtype, accumulate=True, y_prev=exp1), f"large-acc/{n}/{mode}")
    assert comm.last_engine() == 1
    comm.finalize()


def _subnormal_case(dtype, count, rng):
    """prev / x pairs whose sums are subnormal, start subnormal, or cancel to
    +-0 (reading Q16: IEEE, no flush to zero)."""
    if dtype == "f32":
        tiny = np.float32(1.1754944e-38)   # smallest normal
        prev = (rng.integers(-40, 40, count).astype(np.float32) * np.float32(2.0 ** -140)) + \
            np.where(rng.random(count) < 0.5, tiny, -tiny).astype(np.float32)
        x = (rng.integers(-40, 40, count).astype(np.float32) * np.float32(2.0 ** -141)) - prev * np.float32(0.75)
        return prev.astype(np.float32), x.astype(np.float32)
    # bf16 bit patterns: exponent field 0 or 1 (subnormal / smallest normals), random signs
    def pat():
        e = rng.integers(0, 2, count).astype(np.uint16) << 7
        m = rng.integers(0, 128, count).astype(np.uint16)
        s = (rng.integers(0, 2, count).astype(np.uint16) << 15)
        return (s | e | m).astype(np.uint16)
    return pat(), pat()


@pytest.mark.parametrize("acc_red", [1, 0])
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("engine", ENGINES)
def test_accumulate_subnormals_ieee(dtype, engine, acc_red):
    """ACCUMULATE (phase 2) where recv, the result and recv + result are
    subnormal: the engine (incl. the L2 bulk reduce-add) must not flush to
    zero -- bit-exact with the oracle's IEEE replay (reading Q16).  K = 1
    (single late rank) and K = 2 (two late ranks, folded first)."""
    n, count = 3, (1 << 20) + 37
    rng = np.random.default_rng(5)
    prev, x1 = _subnormal_case(dtype, count, rng)
    _, x2 = _subnormal_case(dtype, count, rng)
    xs = [None, x1, x2]
    text = G.allreduce_stars(n, chunk=65536)
    comm = _comm(n, "direct", engine=engine)
    comm.config("acc_red", acc_red)
    comm.set_strategy("allreduce", text)
    for R in ({1}, {1, 2}):
        got = _run_allreduce(comm, [x if r in R else None for r, x in enumerate(xs)], dtype, R,
                             accumulate=True, prev=[prev] * n)
        _assert_bits(got, oc.allreduce(xs, text, R, dtype, accumulate=True, y_prev=[prev] * n),
                     f"subnormal/{dtype}/{sorted(R)}")
    assert comm.get_async_error() == 0
    comm.finalize()


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("n", [9, 16, 64])
def test_wide_rank_counts(n, mode, engine):
    """More than 8 ranks: the kernels instantiated for 64-entry pointer arrays
    (<= 8 ranks launch the narrow parameter block, launch.hpp)."""
    count = 10_007
    comm = _comm(n, mode, scratch=16 << 20, engine=engine)
    xs = rank_tensors("i32", count, n)
    text = G.allreduce_stars(n, chunk=8192)
    comm.set_strategy("allreduce", text)
    R = set(range(n)) - {n // 2}
    got = _run_allreduce(comm, xs, "i32", R)
    _assert_bits(got, oc.allreduce(xs, text, R, "i32"), f"wide/{n}")
    cnt = 257
    ag = G.allgather_stars(n, chunk=4096)
    comm.set_strategy("allgather", ag)
    xg = rank_tensors("f32", cnt, n)
    dy = [empty_dev(n * cnt, "f32") for _ in range(n)]
    comm.allgather_lb([to_dev(x, "f32") for x in xg], dy)
    torch.cuda.synchronize()
    full = np.concatenate(xg)
    for g in range(n):
        assert np.array_equal(bits(to_host(dy[g], "f32")), bits(full)), g
    assert comm.get_async_error() == 0
    comm.finalize()


@pytest.mark.parametrize("relay", ["store", "bypass"])
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
def test_relay_store_bit_exact(relay, mode, engine, dtype):
    """relay=store: pure relays forward through their own arena,
    chunk by chunk; the result is bit-identical to the oracle (and to the
    bypass data path) for chains of relays, binary trees and stars."""
    n, count = 7, 300_007
    parents = [[-1, 0, 1, 2, 3, 4, 5], [-1, 0, 0, 1, 1, 2, 2], S.star(n, 3)]
    text = G.allreduce_trees(parents, weights=[3, 2, 1], chunk=32768, relay=relay)
    comm = _comm(n, mode, scratch=128 << 20, engine=engine)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors(dtype, count, n)
    for R in ({0, 6}, {0, 3, 4}, set(range(n)) - {1, 2, 5}, {6}):
        got = _run_allreduce(comm, xs, dtype, R)
        _assert_bits(got, oc.allreduce(xs, text, R, dtype), f"relay={relay}/{sorted(R)}")
    comm.finalize()
