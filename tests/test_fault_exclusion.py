"""NEXT-3 fault exclusion, host side (CPU): membership rules of the plan,
byte accounting over survivors, and the survivors-only all-gather used by
adapcc_exclude in multi-process mode (gloo + TCPStore, world size 3)."""

import os
import socket

import pytest

from oracle import strategy as OS
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import generator as G


def _all(n):
    return (1 << n) - 1


@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("dead", [{5}, {0, 3}, {1, 2, 6, 7}])
def test_survivor_plan_touches_no_dead_rank(mode, dead):
    n, cnt = 8, 10_007
    live = set(range(n)) - dead
    text = G.survivor_stars(n, live, chunk=8192)
    mask = sum(1 << g for g in live)
    for g in dead:
        st = A.plan_stats(text, cnt, "f32", mask, mode=mode, rank=g, members=live)
        assert st["tasks"] == 0 and st["bytes_read"] == 0 and st["bytes_written"] == 0
    tot = A.plan_stats(text, cnt, "f32", mask, mode=mode, members=live)
    if mode == "direct":
        # single copy over survivors: every live sendbuf read once, every live recvbuf written once
        assert tot["bytes_read"] == len(live) * cnt * 4
        assert tot["bytes_written"] == len(live) * cnt * 4


def test_dead_rank_must_be_a_leaf():
    n = 6
    live = {0, 1, 2, 4, 5}
    mask = sum(1 << g for g in live)
    ok = G.survivor_stars(n, live)
    A.plan_stats(ok, 4096, "f32", mask, members=live)
    bad_trees = [G.allreduce_stars(n), G.allreduce_ring(n)]   # rank 3 roots a star / relays in a chain
    for t in bad_trees:
        with pytest.raises(A.AdapccError) as e:
            A.plan_stats(t, 4096, "f32", mask, members=live)
        assert e.value.code == A.INVALID_STRATEGY
    with pytest.raises(A.AdapccError) as e:             # a dead rank named ready
        A.plan_stats(ok, 4096, "f32", _all(n), members=live)
    assert e.value.code == A.INVALID_ARGUMENT


def test_dead_rank_rules_for_other_collectives():
    n = 4
    live = {0, 1, 3}
    mask = sum(1 << g for g in live)
    # AllGather: a dead source's tree is skipped; a live source's tree may hold it as leaf only
    A.plan_stats(G.allgather_stars(n), 1000, "bf16", mask, members=live)
    with pytest.raises(A.AdapccError):
        A.plan_stats(G.allgather_chains(n), 1000, "bf16", mask, members=live)
    # AlltoAll: no dead relay
    A.plan_stats(G.alltoall_routed(n, [(1, {(0, 3): [1]})]), 1000, "f32", mask, members=live)
    with pytest.raises(A.AdapccError):
        A.plan_stats(G.alltoall_routed(n, [(1, {(0, 3): [2]})]), 1000, "f32", mask, members=live)
    st = A.plan_stats(G.alltoall_direct(n), 1000, "f32", mask, rank=2, members=live)
    assert st["tasks"] == 0
    # Reduce root must be alive
    with pytest.raises(A.AdapccError):
        A.plan_stats(G.reduce_trees([G.star_parent(n, 2)]), 1000, "f32", mask, members=live)
    # ReduceScatter: the dead rank's block has no destination -> skipped
    st = A.plan_stats(G.reducescatter_stars(n), 1000, "f32", mask, members=live)
    full = A.plan_stats(G.reducescatter_stars(n), 1000, "f32", mask)
    assert st["bytes_written"] == full["bytes_written"] * 3 // 4


def test_survivor_stars_are_valid_strategies():
    for n in (2, 5, 8):
        for live in ({0}, set(range(1, n)), set(range(0, n, 2))):
            st = OS.parse(G.survivor_stars(n, live))
            assert sorted(s.root for s in st.subs) == sorted(live)
            for s in st.subs:
                for g in set(range(n)) - live:
                    assert s.children(g) == []


# --------------------------------------------------- survivors-only all-gather
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ag_worker(rank, n, port, q):
    try:
        import ctypes

        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        live = [0, 2]
        if rank in live:
            cb = A.make_store_allgather(live, rank, tag="t")
            out = []
            for rnd in range(3):
                mine = (ctypes.c_uint64 * 2)(rank * 100 + rnd, 7)
                recv = (ctypes.c_uint64 * 4)()
                rc = cb(ctypes.addressof(mine), ctypes.addressof(recv), 16, None)
                out.append((rc, list(recv)))
            q.put((rank, out))
        else:
            q.put((rank, None))      # the "faulty" rank takes no part
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)))


def test_store_allgather_survivors_only():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    n = 3
    ps = [ctx.Process(target=_ag_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(n))
    for p in ps:
        p.join(timeout=60)
    assert res[1] is None
    for r in (0, 2):
        for rnd, (rc, vals) in enumerate(res[r]):
            assert rc == 0
            assert vals == [0 * 100 + rnd, 7, 2 * 100 + rnd, 7]
