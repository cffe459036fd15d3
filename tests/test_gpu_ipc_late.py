"""Late join on the multi-process STAGED protocol (NEXT-1) over real
CUDA IPC (-m gpu): n processes (one GPU each, or all on cuda:0); the late rank
passes its input to the phase-1 call and pushes its chunks to the roots itself
once it signalled ready.  Checked bit-exactly against the late-join oracle for
the deterministic inclusion sets (signal before phase 1: every chunk joins;
no signal: phase 2 adds everything), and int32 finals equal the full sum."""

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
        from tests.gpu_util import bits, empty_dev, to_dev, to_host

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        late = n - 1
        R = set(range(n)) - {late}
        msgs = []
        for engine, dtype in ((0, "f32"), (1, "f32"), (0, "bf16"), (1, "i32")):
            comm.config("engine", engine)
            count = 300_007
            xs = rank_tensors(dtype, count, n)
            for text in (G.allreduce_stars(n, chunk=65536), G.allreduce_ring(n, chunk=32768)):
                comm.set_strategy("allreduce", text)
                for case in ("all", "none"):
                    x = to_dev(xs[rank], dtype)
                    y = empty_dev(count, dtype)
                    if case == "all" and rank == late:
                        comm.signal_ready(ticket=comm.late_ticket() + 1)   # ready before phase 1
                    dist.barrier()
                    comm.allreduce(x, y, ready=R, late="join")
                    torch.cuda.synchronize()
                    L = {late} if case == "all" else set()
                    e1 = oc.allreduce_late(xs, text, R, dtype, L, phase=1)
                    ok1 = np.array_equal(bits(to_host(y, dtype)), bits(e1[rank]))
                    comm.allreduce(x, y, ready=R, late="complement")
                    torch.cuda.synchronize()
                    e2 = oc.allreduce_late(xs, text, R, dtype, L, phase=2, y_prev=e1)
                    ok2 = np.array_equal(bits(to_host(y, dtype)), bits(e2[rank]))
                    if dtype == "i32":
                        ok2 = ok2 and np.array_equal(to_host(y, "i32"), oc.allreduce_exact(xs, set(range(n)), "i32"))
                    msgs.append((engine, dtype, case, ok1, ok2))
        err = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, err == 0 and all(m[3] and m[4] for m in msgs), f"{msgs} err={err}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("n", [2, 3])
def test_staged_late_join_ipc(n):
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


def _excluded_worker(rank, n, port, q):
    """Late join among the survivors after adapcc_exclude: rank n-1 is
    excluded (it stays alive and idle), rank n-2 is the late rank."""
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
        store = dist.distributed_c10d._get_default_store()
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        dead, late = n - 1, n - 2
        live = set(range(n)) - {dead}
        if rank == dead:
            store.wait(["late-excl/done"])
            q.put((rank, True, "excluded"))
            comm.finalize()
            return
        comm.exclude({dead}, store=store)
        R = live - {late}
        msgs = []
        for engine, dtype in ((0, "f32"), (1, "f32"), (1, "i32")):
            comm.config("engine", engine)
            count = 300_007
            xs = rank_tensors(dtype, count, n)
            for text in (None, G.survivor_stars(n, live, chunk=65536)):
                if text is not None:
                    comm.set_strategy("allreduce", text)
                ref = text or G.survivor_stars(n, live)
                for case in ("all", "none"):
                    x = to_dev(xs[rank], dtype)
                    y = empty_dev(count, dtype)
                    t = comm.late_ticket() + 1
                    if case == "all" and rank == late:
                        comm.signal_ready(ticket=t)
                    torch.cuda.synchronize()
                    # survivors-only barrier through the store
                    store.add(f"late-excl/b/{engine}{dtype}{text is None}{case}", 1)
                    store.wait([f"late-excl/b/{engine}{dtype}{text is None}{case}"])
                    while int(store.add(f"late-excl/b/{engine}{dtype}{text is None}{case}", 0)) < len(live):
                        pass
                    comm.allreduce(x, y, ready=R, late="join")
                    torch.cuda.synchronize()
                    L = {late} if case == "all" else set()
                    e1 = oc.allreduce_late(xs, ref, R, dtype, L, phase=1, members=live)
                    ok1 = np.array_equal(bits(to_host(y, dtype)), bits(e1[rank]))
                    if case == "none" and rank == late:
                        comm.signal_ready(ticket=t)
                    comm.allreduce(x, y, ready=R, late="complement")
                    torch.cuda.synchronize()
                    e2 = oc.allreduce_late(xs, ref, R, dtype, L, phase=2, y_prev=e1, members=live)
                    got = to_host(y, dtype)
                    ok2 = np.array_equal(bits(got), bits(e2[rank]))
                    diag = ""
                    if not ok2 and dtype == "i32":
                        d = got.astype(np.int64) - e2[rank].astype(np.int64)
                        nz = np.nonzero(d)[0]
                        diag = (f"bad={nz.size} first={nz[:3].tolist()} last={nz[-3:].tolist()} "
                                + " ".join(f"x{g}:{int(np.count_nonzero(d[nz] == xs[g][nz]))}/"
                                           f"{int(np.count_nonzero(d[nz] == -xs[g][nz].astype(np.int64)))}"
                                           for g in range(n))
                                + f" e1:{int(np.count_nonzero(d[nz] == e1[rank][nz]))}"
                                + f" e1-e2:{int(np.count_nonzero(e1[rank] != e2[rank]))}")
                    msgs.append((engine, dtype, text is None, case, ok1, ok2, diag))
        err = comm.get_async_error()
        if store.add("late-excl/finished", 1) == len(live):
            store.set("late-excl/done", b"1")
        q.put((rank, err == 0 and all(m[4] and m[5] for m in msgs), f"{msgs} err={err}"))
        comm.finalize()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_staged_late_join_after_exclusion():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    n = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_excluded_worker, args=(r, n, port, q)) for r in range(n)]
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
