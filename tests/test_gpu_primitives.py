"""GPU parity of the NEXT-4 primitives (Reduce / Broadcast / ReduceScatter) on
the same engine, both transport plans and both kernels, vs the oracle (-m gpu)."""

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests import strategies as S  # noqa: E402
from tests.gpu_util import bits, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu
MODES = ["direct", "staged"]
ENGINES = [0, 1, 3]   # 0: LDG/STG fold kernel, 1: TMA bulk-copy pipeline kernel, 3: flat (flag-free plans; others fall back)


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _comm(n, mode, engine):
    c = pkg.Communicator.loopback(n, scratch_bytes=64 << 20, mode=mode)
    c.config("timeout_ms", 20000)
    c.config("engine", engine)
    return c


def _check(got, exp, ctx):
    for g, (a, b) in enumerate(zip(got, exp)):
        if b is None:
            continue
        assert np.array_equal(bits(a), bits(b)), f"{ctx} rank {g}"


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
def test_reduce(mode, engine, dtype):
    n, count = 6, 70_001
    xs = rank_tensors(dtype, count, n)
    comm = _comm(n, mode, engine)
    user = G.reduce_trees([S.star(n, 4), S.chain([0, 1, 2, 3, 5, 4]), [4, 0, 0, 1, -1, 1]], [2, 1, 1],
                          chunk=8192, noaggs=[(), (), (1,)])
    cases = [(2, None), (4, user)]
    for root, text in cases:
        if text is not None:
            comm.set_strategy("reduce", text)
        ref_text = text or G.reduce_trees([S.star(n, root)])
        for R in (set(range(n)), {0, 3, 5}):
            prev = [rank_tensors(dtype, count, 1, base=900 + g)[0] for g in range(n)]
            dx = [to_dev(x, dtype) if r in R else None for r, x in enumerate(xs)]
            dy = [to_dev(p, dtype) for p in prev]
            comm.reduce_lb(dx, dy, root, ready=R)
            torch.cuda.synchronize()
            exp = oc.reduce(xs, ref_text, R, dtype, y_prev=prev)
            _check([to_host(y, dtype) for y in dy], exp, f"reduce root={root} R={R}")
            # accumulate (phase 2 style) on top of the previous result
            comm.reduce_lb(dx, dy, root, ready=R, accumulate=True)
            torch.cuda.synchronize()
            exp2 = oc.reduce(xs, ref_text, R, dtype, accumulate=True, y_prev=exp)
            _check([to_host(y, dtype) for y in dy], exp2, "reduce accumulate")
    # a user Reduce strategy fixes the root
    with pytest.raises(pkg.AdapccError):
        comm.reduce_lb([to_dev(x, dtype) for x in xs], [to_dev(x, dtype) for x in xs], 1)
    comm.finalize()


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("mode", MODES)
def test_broadcast(mode, engine):
    n, count = 5, 33_333
    xs = rank_tensors("bf16", count, n)
    comm = _comm(n, mode, engine)
    for root, text in ((1, None), (3, G.broadcast_trees(3, [S.star(n, 3), S.chain([0, 1, 2, 4, 3])], [1, 3],
                                                         chunk=4096))):
        if text is not None:
            comm.set_strategy("broadcast", text)
        ref_text = text or G.broadcast_trees(root, [S.star(n, root)])
        for R in (set(range(n)), {0}):
            prev = [rank_tensors("bf16", count, 1, base=700 + g)[0] for g in range(n)]
            dx = [to_dev(x, "bf16") for x in xs]
            dy = [to_dev(p, "bf16") for p in prev]
            comm.broadcast_lb(dx, dy, root, ready=R)
            torch.cuda.synchronize()
            _check([to_host(y, "bf16") for y in dy], oc.broadcast(xs, ref_text, R, "bf16", prev),
                   f"broadcast root={root}")
    comm.finalize()


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("dtype", ["f32", "bf16", "i32"])
def test_reducescatter(mode, engine, dtype):
    n, cnt = 8, 12_289
    xs = rank_tensors(dtype, n * cnt, n)
    comm = _comm(n, mode, engine)
    texts = [G.reducescatter_stars(n, chunk=8192),
             G.reducescatter_trees([(b, S.star(n, b), 1) for b in range(n)] +
                                   [(2, S.chain([0, 1, 3, 4, 5, 6, 7, 2]), 3)], n, chunk=4096)]
    for text in texts:
        comm.set_strategy("reducescatter", text)
        for R in (set(range(n)), {1, 2, 6}):
            dx = [to_dev(x, dtype) if r in R else None for r, x in enumerate(xs)]
            dy = [to_dev(np.zeros(cnt, xs[0].dtype), dtype) for _ in range(n)]
            comm.reducescatter_lb(dx, dy, ready=R)
            torch.cuda.synchronize()
            _check([to_host(y, dtype) for y in dy], oc.reducescatter(xs, text, R, dtype), "reducescatter")
    # in place: recvbuf == sendbuf + rank * recvcount (16-byte aligned blocks)
    cnt = 12_288
    xs = rank_tensors(dtype, n * cnt, n)
    comm.set_strategy("reducescatter", texts[0])
    dx = [to_dev(x, dtype) for x in xs]
    dy = [dx[g][g * cnt:(g + 1) * cnt] for g in range(n)]
    comm.reducescatter_lb(dx, dy)
    torch.cuda.synchronize()
    _check([to_host(y, dtype) for y in dy], oc.reducescatter(xs, texts[0], set(range(n)), dtype),
           "reducescatter in place")
    comm.finalize()
