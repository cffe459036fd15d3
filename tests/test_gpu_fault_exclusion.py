"""NEXT-3 fault tolerance on the GPU (-m gpu): a rank stops participating,
the watchdog latches TIMEOUT, the survivors exclude it (adapcc_exclude,
P:L139-146) and continue on the same communicator; results are bit-exact
against the oracle over the survivors and the excluded rank's buffers are
never touched."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests.gpu_util import bits, empty_dev, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _eq(a, b):
    return np.array_equal(bits(a), bits(b))


@pytest.mark.parametrize("engine", [0, 1])
@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_loopback_timeout_then_exclude(mode, engine):
    n, cnt, dead = 8, 12_345, 5
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=64 << 20, mode=mode)
    comm.config("engine", engine)
    comm.config("timeout_ms", 300)
    xs = rank_tensors("f32", cnt, n)
    # rank 5 stops working: its tasks never run (test hook).  A chain through
    # rank 5 makes every other rank wait for it in both plans.
    comm.set_strategy("allreduce", G.allreduce_ring(n, chunk=8192))
    comm.config("debug_drop_rank", dead)
    dx = [to_dev(x, "f32") for x in xs]
    dy = [empty_dev(cnt, "f32") for _ in range(n)]
    comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == pkg.adapcc.TIMEOUT
    # survivors exclude it; the communicator is usable again
    comm.config("debug_drop_rank", -1)
    comm.exclude({dead})
    assert comm.get_async_error() == 0
    assert comm.members == set(range(n)) - {dead}
    live = comm.members
    sentinel = empty_dev(cnt, "f32", fill_bits=0x3C)
    before = to_host(sentinel, "f32").copy()
    # 1. AllReduce on the survivors' default strategy (one star per live rank)
    dy = [empty_dev(cnt, "f32") if g != dead else sentinel for g in range(n)]
    comm.allreduce_lb([d if g != dead else None for g, d in enumerate(dx)], dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    exp = oc.allreduce(xs, G.survivor_stars(n, live), live, "f32")
    for g in live:
        assert _eq(to_host(dy[g], "f32"), exp[g]), g
    assert _eq(to_host(sentinel, "f32"), before)
    # 2. a partial mask among survivors + phase 2, user strategy with the dead rank as a leaf
    text = G.survivor_stars(n, live, chunk=4096)
    comm.set_strategy("allreduce", text)
    R1 = live - {0, 7}
    dy = [empty_dev(cnt, "f32") if g != dead else sentinel for g in range(n)]
    comm.allreduce_lb(dx, dy, ready=R1)
    comm.allreduce_lb(dx, dy, ready={0, 7}, accumulate=True)
    torch.cuda.synchronize()
    p1 = oc.allreduce(xs, text, R1, "f32")
    exp = oc.allreduce(xs, text, {0, 7}, "f32", accumulate=True, y_prev=p1)
    for g in live:
        assert _eq(to_host(dy[g], "f32"), exp[g]), g
    assert _eq(to_host(sentinel, "f32"), before)
    # 3. strategies that give the dead rank work are refused
    with pytest.raises(pkg.AdapccError):
        comm.set_strategy("allreduce", G.allreduce_ring(n))
    with pytest.raises(pkg.AdapccError):
        comm.allreduce_lb(dx, dy, ready=set(range(n)))
    # 4. AllGather / AlltoAll over survivors: the dead rank's slots stay untouched
    ag_x = rank_tensors("bf16", 3001, n)
    prev = [rank_tensors("bf16", n * 3001, 1, base=900 + g)[0] for g in range(n)]
    dy = [to_dev(p, "bf16") for p in prev]
    comm.allgather_lb([to_dev(x, "bf16") for x in ag_x], dy)
    torch.cuda.synchronize()
    exp = oc.allgather(ag_x, G.allgather_stars(n), live, "bf16", prev)
    for g in range(n):
        assert _eq(to_host(dy[g], "bf16"), exp[g] if g in live else prev[g]), g
    a2a_x = rank_tensors("i32", n * 777, n)
    prev = [rank_tensors("i32", n * 777, 1, base=950 + g)[0] for g in range(n)]
    dy = [to_dev(p, "i32") for p in prev]
    comm.alltoall_lb([to_dev(x, "i32") for x in a2a_x], dy)
    torch.cuda.synchronize()
    exp = oc.alltoall(a2a_x, G.alltoall_direct(n), live, "i32", prev)
    for g in range(n):
        assert _eq(to_host(dy[g], "i32"), exp[g] if g in live else prev[g]), g
    assert comm.get_async_error() == 0
    # 5. a second fault
    comm.exclude({2})
    live2 = live - {2}
    dy = [empty_dev(cnt, "f32") for _ in range(n)]
    comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    exp = oc.allreduce(xs, G.survivor_stars(n, live2), live2, "f32")
    for g in live2:
        assert _eq(to_host(dy[g], "f32"), exp[g]), g
    assert comm.get_async_error() == 0
    comm.finalize()


# ------------------------------------------------------------- multi-process
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, dead, q, release):
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
        comm.config("timeout_ms", 1500)
        if rank == dead:           # the faulty worker: never becomes ready, makes no call
            q.put((rank, True, "faulty"))
            release.wait(600)
            comm.finalize()
            return
        ok = []
        cnt = 20_011
        xs = rank_tensors("f32", cnt, n)
        live = set(range(n)) - {dead}
        # phase 1 among the ready ranks on the default stars: the dead rank roots one -> TIMEOUT
        y = empty_dev(cnt, "f32")
        comm.allreduce(to_dev(xs[rank], "f32"), y, ready=live)
        torch.cuda.synchronize()
        ok.append(comm.get_async_error() == pkg.adapcc.TIMEOUT)
        # T_fault rule + exclusion (coordinator), survivors continue
        from paper_conf_icdcs_zhaozw24_b200 import coordinator as C
        ready_times = {g: (0.0 if g in live else None) for g in range(n)}
        ex = C.exclude_faulty(comm, ready_times, phase1_end=1.0, now=10.0)
        ok.append(ex == {dead} and comm.get_async_error() == 0)
        for it in range(3):
            y = empty_dev(cnt, "f32")
            comm.allreduce(to_dev(xs[rank], "f32"), y)
            torch.cuda.synchronize()
            exp = oc.allreduce(xs, G.survivor_stars(n, live), live, "f32")[rank]
            ok.append(np.array_equal(bits(to_host(y, "f32")), bits(exp)))
        ag = rank_tensors("bf16", 4099, n)
        y = torch.zeros(n * 4099, dtype=torch.bfloat16, device="cuda")
        comm.allgather(to_dev(ag[rank], "bf16"), y)
        torch.cuda.synchronize()
        exp = oc.allgather(ag, G.allgather_stars(n), live, "bf16", [np.zeros(n * 4099, np.uint16)] * n)[rank]
        ok.append(np.array_equal(to_host(y, "bf16"), exp))
        # registration after the exclusion (survivors-only all-gather) + zero-copy call
        bx = torch.from_numpy(xs[rank]).cuda()
        by = torch.zeros(cnt, dtype=torch.float32, device="cuda")
        rx, ry = comm.register(bx), comm.register(by)
        comm.collective_zc("allreduce", bx, by, cnt)
        torch.cuda.synchronize()
        exp = oc.allreduce(xs, G.survivor_stars(n, live), live, "f32")[rank]
        ok.append(np.array_equal(bits(by.cpu().numpy()), bits(exp)))
        ok.append(comm.get_async_error() == 0)
        comm.deregister(rx)
        comm.deregister(ry)
        comm.finalize()
        q.put((rank, all(ok), f"{ok}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("n,dead", [(3, 2), (4, 1)])
def test_ipc_fault_exclusion(n, dead):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    release = ctx.Event()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, n, port, dead, q, release)) for r in range(n)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=600)
            out[r] = (ok, msg)
    finally:
        release.set()
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert out[r][0], f"rank {r}: {out[r][1]}"
