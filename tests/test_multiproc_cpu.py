"""Host side of the N>1 path with world_size 2 over gloo on CPU (-m "not gpu").

Covers: the bootstrap all-gather callback the C ABI calls during adapcc_init
(the paper's IPC-handle AllGather), and that every rank derives the
same global plan and disjoint rank-local task sets from it (plans are built
independently on each rank from identical arguments -- there is no plan
exchange, so this determinism is what keeps epochs and arena layouts aligned).
"""

import ctypes
import os
import socket
import sys

import pytest

torch = pytest.importorskip("torch")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        import paper_conf_icdcs_zhaozw24_b200 as pkg
        from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
        from paper_conf_icdcs_zhaozw24_b200 import generator as G

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        # 1. bootstrap callback, called exactly as libadapcc calls it
        cb = A.make_bootstrap_allgather(None)
        nbytes = 72
        mine = bytes((rank * 31 + i) % 256 for i in range(nbytes))
        send = ctypes.create_string_buffer(mine, nbytes)
        recv = ctypes.create_string_buffer(nbytes * world)
        rc = cb(ctypes.cast(send, ctypes.c_void_p), ctypes.cast(recv, ctypes.c_void_p), nbytes, None)
        ok_ag = rc == 0 and all(
            recv.raw[r * nbytes:(r + 1) * nbytes] == bytes((r * 31 + i) % 256 for i in range(nbytes))
            for r in range(world))
        # 2. plan determinism across ranks, and rank-local partition of the work
        plans = []
        for text, mask, acc in ((G.allreduce_stars(world, chunk=4096), (1 << world) - 1, False),
                                (G.allreduce_ring(world, chunk=2048), 0b01, True),
                                (G.allgather_chains(world, chunk=1024), (1 << world) - 1, False),
                                (G.alltoall_direct(world, chunk=512, lines=2), 0b10, False)):
            whole = pkg.plan_stats(text, 100_003, "f32", mask, acc, mode="staged", rank=-1)
            mine_ = pkg.plan_stats(text, 100_003, "f32", mask, acc, mode="staged", rank=rank)
            plans.append((whole, mine_))
        gathered = [None] * world
        dist.all_gather_object(gathered, plans)
        ok_plan = True
        for i in range(len(plans)):
            wholes = [g[i][0] for g in gathered]
            ok_plan &= all(w == wholes[0] for w in wholes)
            for key in ("tasks", "items", "bytes_read", "bytes_written", "remote_bytes"):
                ok_plan &= sum(g[i][1][key] for g in gathered) == wholes[0][key]
        dist.destroy_process_group()
        q.put((rank, ok_ag and ok_plan, f"ag={ok_ag} plan={ok_plan}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_world2_gloo_bootstrap_and_plan_consistency():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(2):
            r, ok, msg = q.get(timeout=240)
            out[r] = (ok, msg)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(2):
        assert out[r][0], out[r][1]
