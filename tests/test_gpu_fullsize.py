"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

AllReduce outputs at the bench point (C2) and the C3 bucket sizes are checked
COMPLETELY: every element of every rank against the oracle's strategy-order
replay of the same inputs, bit-exact.  Larger sweeps use sampled indices the
oracle computes element by element (oracle.allreduce_elements); pure index
maps (AlltoAll) are checked completely.
"""

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import GPT2XL_LAYERS, rank_tensors  # noqa: E402
from tests.gpu_util import bits, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _samples(count, k=4096, seed=11):
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([rng.integers(0, count, size=k), [0, count - 1]]))


def _gather(ts, idx, dtype):
    ti = torch.from_numpy(idx).cuda()
    return [to_host(t.index_select(0, ti), dtype) for t in ts]


def _assert_complete(dy, ys, dtype):
    for g, (y, e) in enumerate(zip(dy, ys)):
        got = bits(to_host(y, dtype))
        bad = int(np.count_nonzero(got != bits(e)))
        assert bad == 0, f"rank {g}: {bad} of {got.size} elements differ from the oracle"


@pytest.mark.parametrize("mode,dtype", [("direct", "f32"), ("staged", "f32"), ("direct", "bf16")])
def test_c2_bench_config_complete(mode, dtype):
    """C2 at the bench point (bench.py's launch configuration): 8 ranks x
    256 MiB, 8 star trees, chunk 256 KiB; every output element checked."""
    n, nbytes = 8, 256 << 20
    es = 4 if dtype == "f32" else 2
    count = nbytes // es
    text = G.allreduce_stars(n, chunk=262144)
    comm = pkg.Communicator.loopback(n, scratch_bytes=(2 * nbytes + (8 << 20)) if mode == "staged"
                                     else 64 << 20, mode=mode)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors(dtype, count, n)
    dx = [to_dev(x, dtype) for x in xs]
    dy = [torch.empty_like(t) for t in dx]
    for y in dy:
        y.view(torch.uint8).fill_(0x5A)
    comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    _assert_complete(dy, oc.allreduce(xs, text, set(range(n)), dtype), dtype)
    comm.finalize()


@pytest.mark.parametrize("mib", [25, 100])
def test_c3_partial_aggregation_complete(mib):
    """C3: 8 ranks, stragglers {3,6} relay in phase 1 (mask-aware weighted stars),
    then join with ACCUMULATE in phase 2; STAGED protocol; every element checked."""
    n = 8
    count = (mib << 20) // 4
    R1, R2 = {0, 1, 2, 4, 5, 7}, {3, 6}
    t1 = G.allreduce_mask_aware_stars(n, R1, chunk=262144)
    t2 = G.allreduce_mask_aware_stars(n, R2, chunk=262144)
    comm = pkg.Communicator.loopback(n, scratch_bytes=2 * (mib << 20) + (16 << 20), mode="staged")
    xs = rank_tensors("f32", count, n)
    dx = [to_dev(x, "f32") for x in xs]
    dy = [torch.empty_like(t) for t in dx]
    comm.set_strategy("allreduce", t1)
    comm.allreduce_lb([x if r in R1 else None for r, x in enumerate(dx)], dy, ready=R1)
    comm.set_strategy("allreduce", t2)
    comm.allreduce_lb([x if r in R2 else None for r, x in enumerate(dx)], dy, ready=R2, accumulate=True)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    p1 = oc.allreduce([x if r in R1 else None for r, x in enumerate(xs)], t1, R1, "f32")
    p2 = oc.allreduce([x if r in R2 else None for r, x in enumerate(xs)], t2, R2, "f32",
                      accumulate=True, y_prev=p1)
    _assert_complete(dy, p2, "f32")
    full = oc.allreduce_exact(xs, set(range(n)), "f32")
    assert np.max(np.abs(p2[0].astype(np.float64) - full)) / np.max(np.abs(full)) < 1e-6
    comm.finalize()


@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_c4_alltoall_full(mode):
    """C4: 8 ranks, [8 dest][512 tokens][4096] bf16 per rank, checked completely."""
    n, cnt = 8, 512 * 4096
    text = G.alltoall_direct(n, chunk=1 << 20)
    comm = pkg.Communicator.loopback(n, scratch_bytes=(2 * n * cnt * 2 + (8 << 20)) if mode == "staged"
                                     else 64 << 20, mode=mode)
    comm.set_strategy("alltoall", text)
    xs = rank_tensors("bf16", n * cnt, n, base=2000)
    dx = [to_dev(x, "bf16") for x in xs]
    dy = [torch.empty_like(t) for t in dx]
    comm.alltoall_lb(dx, dy)
    torch.cuda.synchronize()
    prev = [np.zeros(n * cnt, np.uint16)] * n
    exp = oc.alltoall(xs, text, set(range(n)), "bf16", prev)
    for g in range(n):
        assert np.array_equal(to_host(dy[g], "bf16"), exp[g])
    comm.finalize()


@pytest.mark.parametrize("n", [2, 8])
def test_c5_allgather_gpt2xl_with_swap(n):
    """C5: 192 AllGathers of GPT-2-XL row shards (48 layers x 4 weights), strategy
    swapped at call 96 (star, 256 KiB -> chain, 1 MiB), all enqueued back to back."""
    comm = pkg.Communicator.loopback(n, scratch_bytes=256 << 20, mode="staged")
    t_a, t_b = G.allgather_stars(n, chunk=262144), G.allgather_chains(n, chunk=1 << 20)
    comm.set_strategy("allgather", t_a)
    cache = {}
    calls = []
    for layer in range(48):
        for wi, (_, rows, cols) in enumerate(GPT2XL_LAYERS):
            call = layer * 4 + wi
            if call == 96:
                comm.set_strategy("allgather", t_b)
            key = (wi, layer % 3)
            if key not in cache:
                cnt = rows // n * cols
                xs = rank_tensors("bf16", cnt, n, base=3000 + 10 * wi + layer % 3)
                cache[key] = (xs, [to_dev(x, "bf16") for x in xs])
            xs, dx = cache[key]
            dy = [torch.empty(n * len(xs[0]), dtype=torch.bfloat16, device="cuda") for _ in range(n)]
            comm.allgather_lb(dx, dy)
            calls.append((xs, dy))
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    for call, (xs, dy) in enumerate(calls):   # every element of every call (AllGather = concatenation)
        exp = oc.allgather(xs, t_a if call < 96 else t_b, set(range(n)), "bf16",
                           [np.zeros(n * len(xs[0]), np.uint16)] * n)
        for g in range(n):
            assert np.array_equal(to_host(dy[g], "bf16"), exp[g]), call
    comm.finalize()


def test_c2_max_size_sampled():
    """C2's largest point (2^30 B per rank, P:L289 sweep) at n = 8: 16 GiB of
    inputs + outputs resident, TMA pipeline (auto), sampled parity."""
    n, nbytes = 8, 1 << 30
    count = nbytes // 4
    text = G.allreduce_stars(n, chunk=262144)
    comm = pkg.Communicator.loopback(n, scratch_bytes=64 << 20, mode="direct")
    comm.set_strategy("allreduce", text)
    idx = _samples(count)
    vals, dy = [], []
    dx = []
    for r in range(n):   # one rank at a time keeps host memory at ~1 GiB
        x = rank_tensors("f32", count, 1, base=1000 + r)[0]
        vals.append(x[idx].copy())
        dx.append(to_dev(x, "f32"))
        del x
        dy.append(torch.empty(count, dtype=torch.float32, device="cuda"))
    comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    assert comm.last_engine() == 1
    exp = oc.allreduce_elements(vals, idx, count, text, set(range(n)), "f32")
    for g in _gather(dy, idx, "f32"):
        assert np.array_equal(bits(g), bits(exp))
    comm.finalize()


@pytest.mark.parametrize("engine", [0, 1])
def test_byte_offsets_beyond_2_31(engine):
    """2.25 GiB per rank (int32): byte offsets past 2^31 in every pointer path;
    the ragged tail and the last element are sampled."""
    n = 2
    count = (9 << 28) // 4 + 3
    text = G.allreduce_stars(n, chunk=1 << 20)
    comm = pkg.Communicator.loopback(n, scratch_bytes=64 << 20, mode="direct")
    comm.config("engine", engine)
    comm.set_strategy("allreduce", text)
    idx = np.unique(np.concatenate([_samples(count), np.arange(count - 64, count),
                                    np.arange((1 << 29) - 8, (1 << 29) + 8)]))
    vals, dx = [], []
    for r in range(n):
        x = rank_tensors("i32", count, 1, base=1100 + r)[0]
        vals.append(x[idx].copy())
        dx.append(to_dev(x, "i32"))
        del x
    dy = [torch.empty(count, dtype=torch.int32, device="cuda") for _ in range(n)]
    comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    exp = oc.allreduce_elements(vals, idx, count, text, set(range(n)), "i32")
    for g in _gather(dy, idx, "i32"):
        assert np.array_equal(g, exp)
    comm.finalize()
