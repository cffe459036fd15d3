"""Multi-process IPC path on ONE GPU (-m gpu).

n processes (one GPU each, or all on cuda:0 on a 1-GPU box) bootstrap over a gloo process group (127.0.0.1),
export/open each other's arenas with CUDA IPC and run the STAGED protocol with
system-scope flags -- the exact code path of the 8-GPU NVSwitch deployment,
time-sliced on one device.  Each process checks its own recvbuf against the
oracle (bit-exact).
"""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, case, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        import paper_conf_icdcs_zhaozw24_b200 as pkg
        from oracle import collectives as oc
        from paper_conf_icdcs_zhaozw24_b200 import generator as G
        from synth import rank_tensors
        from tests.gpu_util import bits, empty_dev, to_dev, to_host

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()  # one GPU per rank when the box has them
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        results = []
        if case == "allreduce":
            for dtype in ("f32", "bf16", "i32"):
                count = 20_011
                xs = rank_tensors(dtype, count, n)
                for text in (G.allreduce_stars(n, chunk=8192), G.allreduce_ring(n, chunk=16384)):
                    comm.set_strategy("allreduce", text)
                    for R in (set(range(n)), {0}, set(range(1, n))):
                        x = to_dev(xs[rank], dtype)
                        y = empty_dev(count, dtype)
                        comm.allreduce(x, y, ready=R)
                        torch.cuda.synchronize()
                        exp = oc.allreduce(xs, text, R, dtype)[rank]
                        results.append(np.array_equal(bits(to_host(y, dtype)), bits(exp)))
            # phase 1 + phase 2 (accumulate), in place
            xs = rank_tensors("i32", 5003, n)
            R1, R2 = set(range(n - 1)), {n - 1}
            comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=4096))
            y = to_dev(xs[rank], "i32")
            comm.allreduce(y, y, ready=R1)
            comm.allreduce(to_dev(xs[rank], "i32"), y, ready=R2, accumulate=True)
            torch.cuda.synchronize()
            exp = oc.allreduce_exact(xs, set(range(n)), "i32")
            results.append(np.array_equal(to_host(y, "i32"), exp))
        elif case == "allgather_alltoall":
            cnt = 7001
            xs = rank_tensors("bf16", cnt, n)
            for text in (G.allgather_stars(n, chunk=4096), G.allgather_chains(n, chunk=2048)):
                comm.set_strategy("allgather", text)
                y = empty_dev(n * cnt, "bf16")
                comm.allgather(to_dev(xs[rank], "bf16"), y)
                torch.cuda.synchronize()
                results.append(np.array_equal(to_host(y, "bf16"), np.concatenate(xs)))
            xs = rank_tensors("f32", n * cnt, n)
            prev = [np.zeros(n * cnt, np.float32)] * n
            for R in (set(range(n)), {1}):
                y = to_dev(prev[rank], "f32")
                comm.alltoall(to_dev(xs[rank], "f32"), y, ready=R)
                torch.cuda.synchronize()
                exp = oc.alltoall(xs, G.alltoall_direct(n), R, "f32", prev)[rank]
                results.append(np.array_equal(bits(to_host(y, "f32")), bits(exp)))
            if n >= 3:   # routed flows (eq. 1): store-and-forward through relay arenas
                routed = G.alltoall_routed(n, [(1, {(0, n - 1): list(range(1, n - 1)), (n - 1, 1): [0]}),
                                               (2, {})], chunk=4096)
                comm.set_strategy("alltoall", routed)
                for R in (set(range(n)), {0}):
                    y = to_dev(prev[rank], "f32")
                    comm.alltoall(to_dev(xs[rank], "f32"), y, ready=R)
                    torch.cuda.synchronize()
                    exp = oc.alltoall(xs, routed, R, "f32", prev)[rank]
                    results.append(np.array_equal(bits(to_host(y, "f32")), bits(exp)))
        err = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, all(results) and err == 0, f"{len(results)} checks, err={err}, {results}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("n", [2, 3])
@pytest.mark.parametrize("case", ["allreduce", "allgather_alltoall"])
def test_ipc_multiprocess_one_gpu(n, case):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, n, port, case, q)) for r in range(n)]
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
        assert r in out, f"rank {r} produced no result"
        assert out[r][0], f"rank {r}: {out[r][1]}"
