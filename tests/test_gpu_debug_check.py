"""Debug-mode call check across processes on ONE GPU (-m gpu).

SURVEY §5 ("race detection and sanitizers"): with `debug_check` on, every
launch first compares a hash of its call with every live peer's for the same
launch (arena headers, before any byte moves), so ranks that disagree on the
collective, the count, the ready mask or the zero-copy registrations fail
with ADAPCC_ERR_MISMATCH at once instead of corrupting data or hanging until
the watchdog.  Matching calls must be unaffected (bit-exact vs the oracle),
across more launches than the header's 4 signature slots, on both kernels
and both transport plans (STAGED and zero-copy DIRECT).
"""

import os
import socket
import sys
import time

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MISMATCH = 8


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, case, engine, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        import paper_conf_icdcs_zhaozw24_b200 as pkg
        from oracle import collectives as oc
        from paper_conf_icdcs_zhaozw24_b200 import generator as G
        from synth import rank_tensors
        from tests.gpu_util import bits, empty_dev, to_dev, to_host

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()  # one GPU per rank when the box has them
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)   # a mismatch must be reported long before this
        comm.config("engine", engine)
        comm.config("debug_check", 1)
        text = G.allreduce_stars(n, chunk=8192)
        comm.set_strategy("allreduce", text)
        count = 12_345
        xs = rank_tensors("f32", count, n)
        msg = ""
        if case == "match":
            ok = []
            big_x = torch.zeros(count + 64, dtype=torch.float32, device="cuda")
            big_y = torch.zeros(count + 64, dtype=torch.float32, device="cuda")
            rx, ry = comm.register(big_x), comm.register(big_y)
            zx, zy = big_x[16:16 + count], big_y[32:32 + count]
            zx.copy_(torch.from_numpy(xs[rank]))
            for it in range(7):          # > 4 launches: every signature slot is reused
                R = set(range(n)) if it % 2 == 0 else set(range(1, n))
                y = empty_dev(count, "f32")
                comm.allreduce(to_dev(xs[rank], "f32"), y, ready=R)
                comm.collective_zc("allreduce", zx, zy, count, ready=R)
                torch.cuda.synchronize()
                exp = bits(oc.allreduce(xs, text, R, "f32")[rank])
                ok.append(np.array_equal(bits(to_host(y, "f32")), exp))
                ok.append(np.array_equal(bits(zy.cpu().numpy()), exp))
            good = all(ok) and comm.get_async_error() == 0
            msg = f"{ok} err={comm.get_async_error()}"
        else:
            big_x = torch.zeros(count + 64, dtype=torch.float32, device="cuda")
            big_y = torch.zeros(count + 64, dtype=torch.float32, device="cuda")
            comm.register(big_x)
            comm.register(big_y)
            t0 = time.perf_counter()
            if case == "count":        # rank 0 reduces 16 more elements than the others
                c = count + (16 if rank == 0 else 0)
                comm.allreduce(torch.zeros(c, device="cuda"), torch.empty(c, device="cuda"))
            elif case == "mask":       # rank 0 believes rank 1 is a straggler
                R = set(range(n)) - ({1} if rank == 0 else set())
                x = torch.zeros(count, device="cuda") if rank in R else None
                comm.allreduce(x, torch.empty(count, device="cuda"), ready=R)
            elif case == "collective":  # rank 0 calls AllGather, the others AllReduce
                if rank == 0:
                    comm.allgather(torch.zeros(count, device="cuda"), torch.empty(n * count, device="cuda"))
                else:
                    comm.allreduce(torch.zeros(count, device="cuda"), torch.empty(count, device="cuda"))
            elif case == "zc_offset":  # same registrations, rank 0 writes at another offset
                off = 64 if rank == 0 else 32
                comm.collective_zc("allreduce", big_x[16:16 + count], big_y[off:off + count], count)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            err = comm.get_async_error()
            good = err == MISMATCH and dt < 30.0
            msg = f"err={err} after {dt:.2f}s"
        dist.barrier()   # no rank unmaps its arena while a peer's kernel may still read it
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, good, msg))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def _spawn(n, case, engine):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, n, port, case, engine, q)) for r in range(n)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=300)
            out[r] = (ok, msg)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    return out


@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("case", ["match", "count", "mask", "collective", "zc_offset"])
def test_debug_check_ipc(case, engine):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    n = 2 if case != "mask" else 3
    out = _spawn(n, case, engine)
    for r in range(n):
        assert r in out, f"rank {r} produced no result"
        assert out[r][0], f"{case}: rank {r}: {out[r][1]}"
