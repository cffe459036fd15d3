"""Reduce / Broadcast / ReduceScatter over real CUDA IPC: n processes on ONE GPU
(time-sliced), gloo bootstrap, STAGED protocol (-m gpu)."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


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

        import paper_conf_icdcs_zhaozw24_b200 as pkg
        from oracle import collectives as oc
        from paper_conf_icdcs_zhaozw24_b200 import generator as G
        from synth import rank_tensors
        from tests.gpu_util import bits, to_dev, to_host

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()  # one GPU per rank when the box has them
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        ok = []
        count = 10_007
        for dtype in ("f32", "i32"):
            xs = rank_tensors(dtype, count, n)
            for root in range(n):
                R = set(range(n)) - {(root + 1) % n}
                y = to_dev(np.zeros(count, xs[0].dtype), dtype) if rank == root else None
                comm.reduce(to_dev(xs[rank], dtype), y, root, ready=R)
                torch.cuda.synchronize()
                if rank == root:
                    exp = oc.reduce(xs, G.reduce_trees([G.star_parent(n, root)]), R, dtype)[root]
                    ok.append(np.array_equal(bits(to_host(y, dtype)), bits(exp)))
        xs = rank_tensors("bf16", count, n)
        y = to_dev(np.zeros(count, np.uint16), "bf16")
        comm.broadcast(to_dev(xs[rank], "bf16"), y, root=n - 1)
        torch.cuda.synchronize()
        ok.append(np.array_equal(to_host(y, "bf16"), xs[n - 1]))
        cnt = 4099
        xs = rank_tensors("f32", n * cnt, n)
        text = G.reducescatter_stars(n, chunk=4096)
        comm.set_strategy("reducescatter", text)
        y = to_dev(np.zeros(cnt, np.float32), "f32")
        comm.reducescatter(to_dev(xs[rank], "f32"), y)
        torch.cuda.synchronize()
        exp = oc.reducescatter(xs, text, set(range(n)), "f32")[rank]
        ok.append(np.array_equal(bits(to_host(y, "f32")), bits(exp)))
        err = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, all(ok) and err == 0, f"{ok} err={err}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("n", [2, 3])
def test_ipc_primitives_one_gpu(n):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, n, port, q)) for r in range(n)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=600)
            out[r] = (ok, msg)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert r in out and out[r][0], out.get(r)
