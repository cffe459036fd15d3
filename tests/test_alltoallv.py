"""AlltoAllv (NEXT-4): oracle pins + host plan checks (-m "not gpu") and GPU
parity (-m gpu) on skewed MoE routing."""

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from oracle import collectives as oc
from paper_conf_icdcs_zhaozw24_b200 import generator as G
from synth import moe_counts, rank_tensors


def _inputs(counts, dtype):
    n = len(counts)
    return [rank_tensors(dtype, sum(counts[s]), 1, base=4000 + s)[0] for s in range(n)]


def test_oracle_alltoallv_uniform_equals_alltoall():
    n, cnt = 4, 10
    counts = [[cnt] * n for _ in range(n)]
    xs = rank_tensors("f32", n * cnt, n)
    prev = [np.zeros(n * cnt, np.float32)] * n
    a = oc.alltoallv(xs, counts, G.alltoall_direct(n), set(range(n)), "f32", prev)
    b = oc.alltoall(xs, G.alltoall_direct(n), set(range(n)), "f32", prev)
    assert all(np.array_equal(u, v) for u, v in zip(a, b))


def test_oracle_alltoallv_transpose_involution_and_conservation():
    n = 5
    counts = moe_counts(n, 37, 3)
    xs = _inputs(counts, "i32")
    recv_sizes = [sum(counts[s][d] for s in range(n)) for d in range(n)]
    ys = oc.alltoallv(xs, counts, G.alltoall_direct(n), set(range(n)), "i32",
                      [np.zeros(r, np.int32) for r in recv_sizes])
    tcounts = [[counts[s][d] for s in range(n)] for d in range(n)]   # transpose routes back
    back = oc.alltoallv(ys, tcounts, G.alltoall_direct(n), set(range(n)), "i32",
                        [np.zeros(len(x), np.int32) for x in xs])
    assert all(np.array_equal(a, b) for a, b in zip(back, xs))
    assert sum(map(len, ys)) == sum(map(len, xs))


def test_skewed_routing_is_skewed():
    c = np.array(moe_counts(8, 4096, 1, zipf_a=1.2))
    load = c.sum(0)
    assert load.max() > 2.5 * load.min()


@pytest.mark.gpu
@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_gpu_alltoallv_skewed(mode, engine):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from tests.gpu_util import to_dev, to_host
    n = 8
    counts = moe_counts(n, 512, 4096, zipf_a=1.2)     # C4 shape, skewed routing
    xs = _inputs(counts, "bf16")
    recv_sizes = [sum(counts[s][d] for s in range(n)) for d in range(n)]
    comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=(2 * max(recv_sizes) * 2 + (64 << 20)))
    comm.config("engine", engine)
    text = G.alltoall_direct(n, chunk=1 << 20, lines=2)
    comm.set_strategy("alltoall", text)
    for R in (set(range(n)), {1, 4, 6}):
        prev = [rank_tensors("bf16", r, 1, base=6000 + d)[0] for d, r in enumerate(recv_sizes)]
        dx = [to_dev(x, "bf16") for x in xs]
        dy = [to_dev(p, "bf16") for p in prev]
        comm.alltoallv_lb(dx, dy, counts, ready=R)
        torch.cuda.synchronize()
        exp = oc.alltoallv(xs, counts, text, R, "bf16", prev)
        for d in range(n):
            assert np.array_equal(to_host(dy[d], "bf16"), exp[d]), (mode, R, d)
    assert comm.get_async_error() == 0
    comm.finalize()
