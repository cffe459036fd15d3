"""Zero-copy collectives over real CUDA IPC (-m gpu): n processes on ONE GPU
register their tensors; the DIRECT plan then reads peers' inputs and writes
peers' outputs directly (no landing/broadcast slots), bracketed by the
in-kernel entry/exit barriers.  Bit-exact vs the oracle."""

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


def _worker(rank, n, port, engine, q):
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
        comm.config("engine", engine)
        ok = []
        count = 16_384 * n + 4  # blocks of 16 KiB-aligned elements + ragged tail
        big_x = torch.zeros(2 * count + 64, dtype=torch.float32, device="cuda")
        big_y = torch.zeros(2 * count + 64, dtype=torch.float32, device="cuda")
        rx, ry = comm.register(big_x), comm.register(big_y)
        x, y = big_x[16:16 + count], big_y[32:32 + count]     # 64/128-byte offsets into the registrations
        xs = rank_tensors("f32", count, n)
        x.copy_(torch.from_numpy(xs[rank]))
        text = G.allreduce_stars(n, chunk=16384)
        comm.set_strategy("allreduce", text)
        for R in (set(range(n)), set(range(1, n))):
            comm.collective_zc("allreduce", x, y, count, ready=R)
            torch.cuda.synchronize()
            exp = oc.allreduce(xs, text, R, "f32")[rank]
            ok.append(np.array_equal(bits(y.cpu().numpy()), bits(exp)))
        # phase 2 on top (ACCUMULATE): full sum in the end
        comm.collective_zc("allreduce", x, y, count, ready={0}, accumulate=True)
        torch.cuda.synchronize()
        ok.append(np.array_equal(bits(y.cpu().numpy()),
                                 bits(oc.allreduce(xs, text, {0}, "f32", accumulate=True,
                                                   y_prev=oc.allreduce(xs, text, set(range(1, n)), "f32"))[rank])))
        # reduce to root n-1, reducescatter, allgather, alltoall on the same registrations
        comm.collective_zc("reduce", x, y, count, root=n - 1)
        torch.cuda.synchronize()
        if rank == n - 1:
            ok.append(np.array_equal(bits(y.cpu().numpy()),
                                     bits(oc.reduce(xs, G.reduce_trees([G.star_parent(n, n - 1)]),
                                                    set(range(n)), "f32")[n - 1])))
        cnt = count // n
        comm.collective_zc("reducescatter", x, y[:cnt], cnt)
        torch.cuda.synchronize()
        rs = oc.reducescatter([a[:n * cnt] for a in xs], G.reducescatter_stars(n), set(range(n)), "f32")
        ok.append(np.array_equal(bits(y[:cnt].cpu().numpy()), bits(rs[rank])))
        comm.collective_zc("allgather", x[:cnt], y[:n * cnt], cnt)
        torch.cuda.synchronize()
        ok.append(np.array_equal(y[:n * cnt].cpu().numpy(), np.concatenate([a[:cnt] for a in xs])))
        comm.collective_zc("alltoall", x[:n * cnt], y[:n * cnt], cnt)
        torch.cuda.synchronize()
        a2a = oc.alltoall([a[:n * cnt] for a in xs], G.alltoall_direct(n), set(range(n)), "f32",
                          [np.zeros(n * cnt, np.float32)] * n)
        ok.append(np.array_equal(y[:n * cnt].cpu().numpy(), a2a[rank]))
        if n >= 3:   # routed flows (eq. 1): each relay forwards through its own arena
            routed = G.alltoall_routed(n, [(2, {(g, (g + 1) % n): [(g + 2) % n] for g in range(n)}), (1, {})],
                                       chunk=4096)
            comm.set_strategy("alltoall", routed)
            y.zero_()
            comm.collective_zc("alltoall", x[:n * cnt], y[:n * cnt], cnt, ready=set(range(1, n)))
            torch.cuda.synchronize()
            a2a = oc.alltoall([a[:n * cnt] for a in xs], routed, set(range(1, n)), "f32",
                              [np.zeros(n * cnt, np.float32)] * n)
            ok.append(np.array_equal(y[:n * cnt].cpu().numpy(), a2a[rank]))
        err = comm.get_async_error()
        comm.deregister(rx)
        comm.deregister(ry)
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, all(ok) and err == 0, f"{ok} err={err}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("engine", [0, 1, 2, 3])
@pytest.mark.parametrize("n", [2, 3])
def test_zero_copy_one_gpu(n, engine):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, n, port, engine, q)) for r in range(n)]
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


def _big_worker(rank, n, port, mib, q):
    """The N>1 bench path at bench-like size: >= 64 MiB per rank, zero-copy
    DIRECT on the TMA engine (and the STAGED protocol beside it), every
    element of this rank's output against the oracle replay."""
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
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        nbytes = mib << 20
        comm = pkg.Communicator.init(scratch_bytes=2 * nbytes + (64 << 20), device=dev)
        comm.config("timeout_ms", 120000)
        msgs = []
        for dtype in ("f32", "bf16"):
            es = 4 if dtype == "f32" else 2
            count = nbytes // es - 8 * 3 - 5       # ragged: not a multiple of any tile
            text = G.allreduce_stars(n, chunk=262144)
            comm.set_strategy("allreduce", text)
            xs = rank_tensors(dtype, count, n)
            exp = oc.allreduce(xs, text, set(range(n)), dtype)[rank]
            x = to_dev(xs[rank], dtype)
            y = torch.empty_like(x)
            rx, ry = comm.register(x), comm.register(y)
            for engine, path in ((1, "zc"), (0, "zc"), (3, "zc"), (2, "staged")):
                comm.config("engine", engine)
                y.view(torch.uint8).fill_(0x5A)
                if path == "zc":
                    comm.collective_zc("allreduce", x, y, count)
                else:
                    comm.allreduce(x, y)
                torch.cuda.synchronize()
                bad = int(np.count_nonzero(bits(to_host(y, dtype)) != bits(exp)))
                msgs.append(f"{dtype}/{path}/engine{engine}: {bad} bad")
            comm.deregister(rx)
            comm.deregister(ry)
            del x, y
        err = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, err == 0 and all(m.endswith(": 0 bad") for m in msgs), f"{msgs} err={err}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_zero_copy_three_ranks_64mib_complete():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    n, mib = 3, 64
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_big_worker, args=(r, n, port, mib, q)) for r in range(n)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=900)
            out[r] = (ok, msg)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert r in out and out[r][0], out.get(r)
