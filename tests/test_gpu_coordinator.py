"""The online coordinator on the GPU (-m gpu, NEXT-1 P:L129-137): real
readiness (ranks signal through the device onto the host-mapped board, two
stragglers after a controlled %globaltimer spin), the coordinator -- not the
test -- decides wait / full / phase 1 and issues LATE_JOIN / LATE_COMPLEMENT;
int32 results equal the full sum exactly, and every recvbuf is identical."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import coordinator as C  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests.gpu_util import empty_dev, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _policy(n, S, buy_s):
    p = C.Coordinator(n, "allreduce", S, 100e9, 5e-6)
    p.buy_cost = lambda k: buy_s        # calibrated buying cost (seconds)
    return p


@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("lag_us,buy_us,expect", [(3000, 50, "phase1"), (0, 100_000, "full")])
def test_coordinator_drives_the_calls(mode, lag_us, buy_us, expect):
    n, count = 8, 2_000_003
    R, late = {0, 1, 2, 4, 5, 7}, [3, 6]
    xs = rank_tensors("i32", count, n)
    comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=64 << 20)
    comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=65536))
    dx = [to_dev(x, "i32") for x in xs]
    dy = [empty_dev(count, "i32") for _ in range(n)]
    cs = torch.cuda.Stream(priority=-1)      # communication: high priority
    side = torch.cuda.Stream()               # the stragglers' "computation"
    coord = C.OnlineCoordinator(comm, lambda: _policy(n, count * 4, buy_us * 1e-6), cycle=2e-6)
    full = oc.allreduce_exact(xs, set(range(n)), "i32")
    for it in range(3):
        t = coord.ticket()
        for r in R:
            comm.signal_ready(r, ticket=t, stream=cs)
        for r in late:
            comm.spin(lag_us * 1000, stream=side)
            comm.signal_ready(r, ticket=t, stream=side)
        res = coord.allreduce(lambda m, lt: comm.allreduce_lb(dx, dy, ready=m, late=lt, stream=cs))
        torch.cuda.synchronize()
        assert comm.get_async_error() == 0
        assert res["action"] == expect, res
        for y in dy:
            assert np.array_equal(to_host(y, "i32"), full), (it, res)
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
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        count = 500_009
        xs = rank_tensors("i32", count, n)
        x, y = to_dev(xs[rank], "i32"), empty_dev(count, "i32")
        late = n - 1
        coord = C.OnlineCoordinator(comm, lambda: _policy(n, count * 4, 100e-6), cycle=5e-6)
        cs = torch.cuda.Stream(priority=-1)
        side = torch.cuda.Stream()
        ok = []
        for it in range(3):
            t = coord.ticket()
            dist.barrier()
            if rank == late:
                comm.spin(20_000_000, stream=side)        # 20 ms straggler
                comm.signal_ready(ticket=t, stream=side)
            else:
                comm.signal_ready(ticket=t, stream=cs)
            res = coord.allreduce(lambda m, lt: comm.allreduce(x, y, ready=m, late=lt, stream=cs))
            torch.cuda.synchronize()
            ok.append((res["action"], np.array_equal(to_host(y, "i32"), oc.allreduce_exact(xs, set(range(n)), "i32"))))
        err = comm.get_async_error()
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, err == 0 and all(a == "phase1" and b for a, b in ok), f"{ok} err={err} shared={coord.board.shared}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_coordinator_multiprocess_shared_board():
    """3 processes: rank 0 decides from the node-shared board and publishes;
    every rank issues the same phase-1 / phase-2 calls (STAGED protocol)."""
    import torch.multiprocessing as mp
    n = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=300)
            out[r] = (ok, msg)
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert r in out and out[r][0], out.get(r)


def test_coordinator_alltoall_two_phases():
    """The coordinator's issue callback is collective-agnostic: AlltoAll
    (P:L135 prices it at N x tensor) runs phase 1 among the ready sources and
    phase 2 for the late ones (their blocks were left untouched, reading
    Q12); the final result is the complete block transpose."""
    from oracle import collectives as oc2
    n, cnt = 8, 4096
    xs = rank_tensors("bf16", n * cnt, n)
    comm = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    comm.set_strategy("alltoall", G.alltoall_direct(n))
    dx = [to_dev(x, "bf16") for x in xs]
    dy = [empty_dev(n * cnt, "bf16") for _ in range(n)]
    side = torch.cuda.Stream()
    all_mask = (1 << n) - 1

    def policy():
        p = C.Coordinator(n, "alltoall", n * cnt * 2, 100e9, 5e-6)
        p.buy_cost = lambda k: 50e-6
        return p

    coord = C.OnlineCoordinator(comm, policy, cycle=2e-6)
    t = coord.ticket()
    for r in range(n):
        if r not in (2, 5):
            comm.signal_ready(r, ticket=t)
    comm.spin(3_000_000, stream=side)
    comm.signal_ready(2, ticket=t, stream=side)
    comm.signal_ready(5, ticket=t, stream=side)

    def issue(mask, late):
        if late is None:
            comm.alltoall_lb(dx, dy)
        elif late == "join":
            comm.alltoall_lb(dx, dy, ready=mask)
        else:   # phase 2: the late sources' blocks
            comm.alltoall_lb(dx, dy, ready=all_mask & ~mask)
    res = coord.allreduce(issue)
    torch.cuda.synchronize()
    assert res["action"] == "phase1" and res["mask"] == all_mask & ~((1 << 2) | (1 << 5)), res
    exp = oc2.alltoall(xs, G.alltoall_direct(n), set(range(n)), "bf16", [np.zeros(n * cnt, np.uint16)] * n)
    for g in range(n):
        assert np.array_equal(to_host(dy[g], "bf16"), exp[g])
    comm.finalize()


@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_coordinator_fault_rule_excludes_silent_rank(mode):
    """NEXT-3 on the hot path: virtual rank 6 never signals.
    The coordinator starts phase 1 without it, and T_fault = 5 x (phase-1 end
    - first ready) after phase 1 marks it faulty. The survivors exclude it and
    keep the phase-1 result (the exact survivors' sum). Later rounds, one of
    them with a straggler among the survivors (late join + phase 2), run on
    the survivors only: rank 6's recvbuf is no longer written."""
    n, count, dead = 8, 1_000_003, 6
    xs = rank_tensors("i32", count, n)
    comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=64 << 20)
    comm.config("timeout_ms", 60000)
    comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=65536))
    dx = [to_dev(x, "i32") for x in xs]
    dy = [empty_dev(count, "i32") for _ in range(n)]
    cs = torch.cuda.Stream(priority=-1)
    side = torch.cuda.Stream()
    coord = C.OnlineCoordinator(comm, lambda: _policy(n, count * 4, 50e-6), cycle=2e-6,
                                fault_factor=5.0, stream=cs, timeout=20.0)
    live = set(range(n)) - {dead}
    survivors_sum = oc.allreduce_exact([xs[g] for g in sorted(live)], set(range(n - 1)), "i32")

    t = coord.ticket()
    for r in live:
        comm.signal_ready(r, ticket=t, stream=cs)
    res = coord.allreduce(lambda m, lt: comm.allreduce_lb(dx, dy, ready=m, late=lt, stream=cs))
    torch.cuda.synchronize()
    assert res["action"] == "phase1" and res["faulty"] == [dead], res
    assert comm.members == live and comm.get_async_error() == 0
    for g in live:
        assert np.array_equal(to_host(dy[g], "i32"), survivors_sum), g
    dy[dead].fill_(-7)
    sentinel = to_host(dy[dead], "i32").copy()
    # a full round, then a straggler (rank 2) among the survivors that signals
    # within T_fault (phase 1 ends ~0.1-0.2 ms after the first ready rank)
    for it, lag_us in enumerate((0, 300)):
        for g in live:
            dy[g].zero_()
        torch.cuda.synchronize()            # (the collectives run on cs)
        t = coord.ticket()
        for r in live - {2}:
            comm.signal_ready(r, ticket=t, stream=cs)
        comm.spin(lag_us * 1000, stream=side)
        comm.signal_ready(2, ticket=t, stream=side)
        res = coord.allreduce(lambda m, lt: comm.allreduce_lb(
            [d if g != dead else None for g, d in enumerate(dx)], dy, ready=m, late=lt, stream=cs))
        torch.cuda.synchronize()
        assert comm.get_async_error() == 0
        assert res["faulty"] == [] and res["action"] == ("full" if lag_us == 0 else "phase1"), (it, res)
        for g in live:
            assert np.array_equal(to_host(dy[g], "i32"), survivors_sum), (it, g)
        assert np.array_equal(to_host(dy[dead], "i32"), sentinel)
    comm.finalize()


def _fault_worker(rank, n, port, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        store = dist.distributed_c10d._get_default_store()
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        count = 300_007
        xs = rank_tensors("i32", count, n)
        x, y = to_dev(xs[rank], "i32"), empty_dev(count, "i32")
        dead = n - 1
        cs = torch.cuda.Stream(priority=-1)
        coord = C.OnlineCoordinator(comm, lambda: _policy(n, count * 4, 100e-6), cycle=5e-6, fault_factor=5.0,
                                    store=store, stream=cs, timeout=60.0)
        t = coord.ticket()
        dist.barrier()
        if rank != dead:                      # the faulty rank never signals
            comm.signal_ready(ticket=t, stream=cs)
        res = coord.allreduce(lambda m, lt: comm.allreduce(x, y, ready=m, late=lt, stream=cs))
        torch.cuda.synchronize()
        live = set(range(n)) - {dead}
        exp = oc.allreduce_exact([xs[g] for g in sorted(live)], set(range(n - 1)), "i32")
        ok = [res["faulty"] == [dead]]
        if os.environ.get("FAULT_TEST_WAIT_DEAD"):   # (diagnostic: the survivors start only once the dead rank's kernel ended)
            if rank == dead:
                store.set("fault-test/dead-idle", b"1")
            else:
                store.wait(["fault-test/dead-idle"])
        if rank == dead:                      # excluded: stays alive (its arena is mapped) until the survivors finish
            store.wait(["fault-test/done"])
        else:
            ok.append(comm.members == live)
            ok.append(np.array_equal(to_host(y, "i32"), exp))
            if os.environ.get("FAULT_TEST_TRACE"):
                comm.config("trace", 1 << 16)
            for _ in range(2):                # the survivors carry on: a full round
                y.zero_()
                torch.cuda.synchronize()      # (the collectives run on cs)
                t = coord.ticket()
                comm.signal_ready(ticket=t, stream=cs)
                res = coord.allreduce(lambda m, lt: comm.allreduce(x, y, ready=m, late=lt, stream=cs))
                torch.cuda.synchronize()
                got = to_host(y, "i32")
                good = np.array_equal(got, exp)
                if not good:   # diagnostics: which elements, and what they hold instead
                    bad = np.nonzero(got != exp)[0]
                    x0, x1 = xs[0], xs[1]
                    kinds = {"x0": int(np.sum(got[bad] == x0[bad])), "x1": int(np.sum(got[bad] == x1[bad])),
                             "zero": int(np.sum(got[bad] == 0)),
                             "sum+x2": int(np.sum(got[bad] == (exp[bad] + xs[2][bad]))),
                             "2x": int(np.sum(got[bad] == 2 * exp[bad]))}
                    good = (False, res, int(bad.size), int(bad[0]), int(bad[-1]), kinds)
                    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
                    if os.environ.get("FAULT_TEST_TRACE"):
                        recs, tot = comm.trace()
                        np.save(os.path.join(ROOT, "gpurun_out", f"fault_trace_r{rank}_{os.getpid()}.npy"), recs)
                    with open(os.path.join(ROOT, "gpurun_out", f"fault_diag_r{rank}.txt"), "a") as f:
                        f.write(repr(good) + "\n")
                ok.append((res["faulty"], good))
                if os.environ.get("FAULT_TEST_TRACE") and good is True:
                    comm.trace()   # (drain: the next round's records start empty)
            if store.add("fault-test/finished", 1) == n - 1:
                store.set("fault-test/done", b"1")
        err = comm.get_async_error()
        good = all(o if isinstance(o, bool) else (o[0] == [] and o[1] is True) for o in ok)
        q.put((rank, err == 0 and good, f"{ok} err={err} res={res}"))
        comm.finalize()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_coordinator_fault_rule_multiprocess():
    """3 processes, rank 2 never signals: the leader applies T_fault after
    phase 1 and publishes the faulty mask on the node-shared board; ranks 0
    and 1 exclude rank 2 through the store (adapcc_exclude) and keep running
    full collectives on the survivors, exact."""
    import torch.multiprocessing as mp
    n = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_fault_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, msg = q.get(timeout=300)
            out[r] = (ok, msg)
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert r in out and out[r][0], out.get(r)
