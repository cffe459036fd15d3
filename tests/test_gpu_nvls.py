"""NVLS switch reduction (NEXT-2) on the GPU (-m gpu).  The multicast team
needs several NVSwitch-connected GPUs: on a 1-GPU box adapcc_nvls_setup must
refuse cleanly on every rank (and nvls lines must then fail with
UNSUPPORTED instead of hanging); where it succeeds, the switch-reduced
AllReduce matches the oracle's tolerance mode (int32 exactly)."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def test_nvls_line_without_setup_is_refused():
    comm = pkg.Communicator.loopback(4)
    comm.set_strategy("allreduce", G.allreduce_nvls(4))
    xs = [torch.ones(4096, device="cuda") for _ in range(4)]
    with pytest.raises(pkg.AdapccError) as e:
        comm.allreduce_lb(xs, [torch.empty_like(x) for x in xs])
    assert e.value.code == pkg.adapcc.UNSUPPORTED
    comm.finalize()


@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("n", [2, 5, 8])
def test_nvls_plan_on_emulated_switch(mode, n):
    """Loopback emulates the switch (each virtual rank has its own scratch,
    the kernel sums the copies): the whole NVLS plan -- copy in, per-slice
    flags, the switch step, copy out, the ragged tail through a star -- runs
    against the oracle's tolerance mode (int32 exact), with nvls lines mixed
    with star trees, ACCUMULATE, and a partial mask refused."""
    from oracle import bf16 as obf
    from oracle import collectives as oc
    from synth import rank_tensors
    from tests.gpu_util import bits, empty_dev, to_dev, to_host
    comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=64 << 20)
    ok, why = comm.nvls_setup(32 << 20)
    assert ok, why
    text = G.allreduce_nvls(n, chunk=1 << 16, nvls_weight=5, star_weight=1)
    comm.set_strategy("allreduce", text)
    for dtype in ("i32", "f32", "bf16"):
        for count in (1 << 20, (1 << 20) + 3, 777):
            xs = rank_tensors(dtype, count, n)
            dy = [empty_dev(count, dtype) for _ in range(n)]
            comm.allreduce_lb([to_dev(x, dtype) for x in xs], dy)
            torch.cuda.synchronize()
            exp = oc.allreduce(xs, text, set(range(n)), dtype)
            got = [to_host(y, dtype) for y in dy]
            for g in range(1, n):
                assert np.array_equal(bits(got[g]), bits(got[0]))      # every rank the same bytes
            if dtype == "i32":
                assert np.array_equal(got[0], exp[0])
            else:
                f = (lambda a: obf.to_f32(a).astype(np.float64)) if dtype == "bf16" else (lambda a: a.astype(np.float64))
                den = np.sum(np.abs(np.stack([f(x) for x in xs])), axis=0) + 1e-30
                assert np.max(np.abs(f(got[0]) - f(exp[0])) / den) <= oc.nvls_tolerance(dtype, n) * 1.001
    # ACCUMULATE (phase 2 on top of a previous result), int32 exact
    xs = rank_tensors("i32", 100_003, n)
    prev = rank_tensors("i32", 100_003, n, base=1700)
    dy = [to_dev(p, "i32") for p in prev]
    comm.allreduce_lb([to_dev(x, "i32") for x in xs], dy, accumulate=True)
    torch.cuda.synchronize()
    exp = oc.allreduce(xs, text, set(range(n)), "i32", accumulate=True, y_prev=prev)
    assert all(np.array_equal(to_host(y, "i32"), e) for y, e in zip(dy, exp))
    with pytest.raises(pkg.AdapccError) as e:          # the switch sums every copy: whole mask only
        comm.allreduce_lb([to_dev(x, "i32") for x in xs], dy, ready=set(range(1, n)))
    assert e.value.code == pkg.adapcc.UNSUPPORTED
    assert comm.get_async_error() == 0
    comm.finalize()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        from oracle import collectives as oc
        from synth import rank_tensors
        from tests.gpu_util import bits, to_dev, to_host
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 30000)
        ok, why = comm.nvls_setup(64 << 20)
        res = {"ok": ok, "why": why, "checks": []}
        text = G.allreduce_nvls(n, chunk=1 << 18, nvls_weight=3, star_weight=1)
        comm.set_strategy("allreduce", text)
        if not ok:
            x = torch.ones(1 << 16, device="cuda")
            try:
                comm.allreduce(x, torch.empty_like(x))
                res["checks"].append(("refused", False))
            except pkg.AdapccError as e:
                res["checks"].append(("refused", e.code == pkg.adapcc.UNSUPPORTED))
        else:
            for dtype in ("i32", "f32", "bf16"):
                count = (1 << 20) + 5
                xs = rank_tensors(dtype, count, n)
                y = to_dev(np.zeros_like(xs[rank]), dtype)
                comm.allreduce(to_dev(xs[rank], dtype), y)
                torch.cuda.synchronize()
                got = to_host(y, dtype)
                exp = oc.allreduce(xs, text, set(range(n)), dtype)[rank]
                if dtype == "i32":
                    res["checks"].append((dtype, bool(np.array_equal(got, exp))))
                else:
                    from oracle import bf16 as obf
                    f = (lambda a: obf.to_f32(a).astype(np.float64)) if dtype == "bf16" else (lambda a: a.astype(np.float64))
                    den = np.sum(np.abs(np.stack([f(x) for x in xs])), axis=0) + 1e-30
                    err = float(np.max(np.abs(f(got) - f(exp)) / den))
                    res["checks"].append((dtype, err <= 2 * oc.nvls_tolerance(dtype, n)))
        res["err"] = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, res))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, {"exc": traceback.format_exc() + repr(e)}))


def test_nvls_multiprocess():
    import torch.multiprocessing as mp
    n = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, res = q.get(timeout=300)
            out[r] = res
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert "exc" not in out[r], out[r]
        assert out[r]["err"] == 0
        assert all(ok for _, ok in out[r]["checks"]), out[r]
    oks = {out[r]["ok"] for r in range(n)}
    assert len(oks) == 1, out                      # every rank agrees
    if not out[0]["ok"]:
        pytest.skip("no multicast team on this box: " + out[0]["why"])
    assert out[0]["checks"] and all(ok for _, ok in out[0]["checks"])
