"""GPU parity of routed AlltoAll (SURVEY §8(a) a9 "direct or along a route",
P:L171 eq. 1) and routed AlltoAllv, loopback n virtual ranks (-m gpu).

Bit-exact against the oracle's definition (routes change the path, never the
bytes: "flows carry different parameters")."""

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from oracle import loads as OL  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import moe_counts, rank_tensors  # noqa: E402
from tests.gpu_util import bits, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _comm(n, mode, engine, scratch=64 << 20):
    c = pkg.Communicator.loopback(n, device=0, scratch_bytes=scratch, mode=mode)
    c.config("timeout_ms", 20000)
    c.config("engine", engine)
    return c


def _strategies(n):
    ring_routes = {(g, (g + 1) % n): [(g + 2) % n, (g + 3) % n] for g in range(n)}   # 2 relays each
    long_route = {(0, n - 1): list(range(1, n - 1))}                                   # n-2 relays
    return {
        "detour": G.alltoall_detour(n, [(0, 1), (1, 0), (2, 5), (7, 3), (4, 6)], chunk=4096),
        "split": G.alltoall_routed(n, [(3, ring_routes), (1, {}), (2, long_route)], chunk=2048),
        "all_routed": G.alltoall_routed(
            n, [(1, {(s, d): [next(h for h in range(n) if h not in (s, d))]
                     for s in range(n) for d in range(n) if s != d})], chunk=8192),
    }


@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_routed_alltoall_parity(mode, dtype, engine):
    n, cnt = 8, 5003                        # ragged: not a multiple of any chunk
    comm = _comm(n, mode, engine)
    xs = rank_tensors(dtype, n * cnt, n)
    for name, text in _strategies(n).items():
        comm.set_strategy("alltoall", text)
        for R in (set(range(n)), {0, 2, 7}, {3}):
            prev = [rank_tensors(dtype, n * cnt, 1, base=400 + g)[0] for g in range(n)]
            dx = [to_dev(x, dtype) for x in xs]
            dy = [to_dev(p, dtype) for p in prev]
            comm.alltoall_lb(dx, dy, ready=R)
            torch.cuda.synchronize()
            exp = oc.alltoall(xs, text, R, dtype, prev)
            for g in range(n):
                assert np.array_equal(bits(to_host(dy[g], dtype)), bits(exp[g])), (name, mode, R, g)
    assert comm.get_async_error() == 0
    comm.finalize()


@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_routed_alltoall_stats_match_loads(mode):
    """The plan the GPU ran moves exactly the oracle's per-edge bytes."""
    n, cnt = 8, 5003
    text = _strategies(n)["split"]
    R = set(range(n))
    EB = OL.alltoall_edge_bytes(text, cnt, "f32", R)
    for r in range(n):
        st = pkg.adapcc.plan_stats(text, cnt, "f32", (1 << n) - 1, False, mode, r, 64 << 20)
        assert st["remote_bytes"] == sum(v for (i, _), v in EB.items() if i == r)


@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_routed_alltoallv_skewed(mode, engine):
    n = 8
    counts = moe_counts(n, 256, 1024, zipf_a=1.2)
    rng = np.random.default_rng(3)
    xs = []
    for s in range(n):
        xs.append(rank_tensors("bf16", int(sum(counts[s])), 1, base=7000 + s)[0])
    recv = [sum(counts[s][d] for s in range(n)) for d in range(n)]
    comm = _comm(n, mode, engine, scratch=4 * max(recv) * 2 + (64 << 20))
    text = _strategies(n)["split"]
    comm.set_strategy("alltoall", text)
    for R in (set(range(n)), set(int(g) for g in rng.choice(n, 4, replace=False))):
        prev = [rank_tensors("bf16", r, 1, base=7100 + d)[0] for d, r in enumerate(recv)]
        dx = [to_dev(x, "bf16") for x in xs]
        dy = [to_dev(p, "bf16") for p in prev]
        comm.alltoallv_lb(dx, dy, counts, ready=R)
        torch.cuda.synchronize()
        exp = oc.alltoallv(xs, counts, text, R, "bf16", prev)
        for d in range(n):
            assert np.array_equal(to_host(dy[d], "bf16"), exp[d]), (mode, R, d)
    assert comm.get_async_error() == 0
    comm.finalize()


def test_routed_alltoall_tiny_arena_segments():
    """Relay slots that do not fit the arena split the call into segments."""
    n, cnt = 4, 1 << 16
    text = G.alltoall_routed(n, [(1, {(s, d): [(d + 1) % n if (d + 1) % n != s else (d + 2) % n]
                                     for s in range(n) for d in range(n) if s != d})], chunk=16384)
    st = pkg.adapcc.plan_stats(text, cnt, "f32", (1 << n) - 1, False, "staged", -1, 1 << 20)
    assert st["segments"] > 1
    comm = _comm(n, "staged", 2, scratch=1 << 20)
    comm.set_strategy("alltoall", text)
    xs = rank_tensors("f32", n * cnt, n)
    prev = [np.zeros(n * cnt, np.float32)] * n
    dx = [to_dev(x, "f32") for x in xs]
    dy = [to_dev(p, "f32") for p in prev]
    comm.alltoall_lb(dx, dy)
    torch.cuda.synchronize()
    exp = oc.alltoall(xs, text, set(range(n)), "f32", prev)
    for g in range(n):
        assert np.array_equal(to_host(dy[g], "f32"), exp[g])
    assert comm.get_async_error() == 0
    comm.finalize()
