"""Online coordinator (NEXT-1) host logic on CPU: a fake
communicator exposes a readiness board in host memory; the coordinator must
decide from the board alone (break-even rule), issue phase 1 with the ready
mask, and issue phase 2 only after every late rank signalled -- and a
follower rank must take the leader's decision from the board."""

import ctypes
import threading
import time

import pytest

from paper_conf_icdcs_zhaozw24_b200 import coordinator as C


class FakeComm:
    def __init__(self, n, rank=0, loopback=True, board=None, ticket=4):
        self.nranks, self.rank, self.loopback = n, rank, loopback
        self.board = board if board is not None else (ctypes.c_uint64 * 128)()
        self._ticket = ticket

    def ready_board(self):
        return ctypes.addressof(self.board), True

    def late_ticket(self):
        return self._ticket

    def late_advance(self):
        self._ticket += 1
        return self._ticket


def _policy(n, buy_after):
    """A Coordinator whose buying cost is buy_after seconds."""
    bw = C.comm_volume("allreduce", n, 1.0) / (n * 1.0)   # t(k) ~ (k-1)/k
    c = C.Coordinator(n, "allreduce", 1.0, bw, 1e-4)
    c.buy_cost = lambda k: buy_after
    return c


def test_all_ready_runs_one_full_call():
    comm = FakeComm(4)
    for r in range(4):
        comm.board[r] = 5
    calls = []
    oc = C.OnlineCoordinator(comm, lambda: _policy(4, 1.0), cycle=1e-5)
    res = oc.allreduce(lambda m, late: calls.append((m, late)))
    assert res["action"] == "full" and calls == [(0b1111, None)]
    assert comm.late_ticket() == 5          # the round's ticket is retired


def test_phase1_then_phase2_after_late_ranks_signal():
    n, t = 8, 5
    comm = FakeComm(n)
    for r in range(6):
        comm.board[r] = t          # ranks 0-5 ready; 6, 7 straggle
    comm.board[6] = t - 1          # an old ticket does not count
    calls = []
    signalled = []

    def straggle():
        time.sleep(0.2)
        signalled.append(time.perf_counter())
        comm.board[6] = t
        comm.board[7] = t

    th = threading.Thread(target=straggle)
    oc = C.OnlineCoordinator(comm, lambda: _policy(n, 2e-3), cycle=1e-4)
    th.start()
    res = oc.allreduce(lambda m, late: calls.append((m, late, time.perf_counter())))
    th.join()
    assert res["action"] == "phase1" and res["mask"] == 0b00111111
    assert [c[:2] for c in calls] == [(0b00111111, "join"), (0b00111111, "complement")]
    assert comm.late_ticket() == t     # phase 1 retired the round's ticket (here: the coordinator did)
    assert 1.5e-3 < res["decided_after_s"] < 0.15        # bought after ~the buying cost, before the stragglers
    assert calls[1][2] >= signalled[0]                    # phase 2 only once 6 and 7 signalled


def test_no_one_ready_times_out():
    comm = FakeComm(2)
    oc = C.OnlineCoordinator(comm, lambda: _policy(2, 1.0), cycle=1e-4, timeout=0.02)
    with pytest.raises(TimeoutError):
        oc.allreduce(lambda m, late: None)


def test_follower_takes_the_leaders_decision():
    """Two ranks of one node share the board: rank 0 decides and publishes,
    rank 1 never evaluates the policy but issues the same calls."""
    n, t = 2, 3
    board = (ctypes.c_uint64 * 128)()
    board[0] = t
    leader = C.OnlineCoordinator(FakeComm(n, 0, False, board, t - 1), lambda: _policy(n, 1e-3), cycle=1e-4)
    follower = C.OnlineCoordinator(FakeComm(n, 1, False, board, t - 1),
                                   lambda: pytest.fail("a follower must not decide"), cycle=1e-4)
    out = {}

    def run(name, oc):
        calls = []
        out[name] = (oc.allreduce(lambda m, late: calls.append((m, late))), calls)

    tf = threading.Thread(target=run, args=("f", follower))
    tf.start()
    time.sleep(0.01)
    threading.Timer(0.03, lambda: board.__setitem__(1, t)).start()
    run("l", leader)
    tf.join()
    assert out["l"][1] == out["f"][1] == [(0b01, "join"), (0b01, "complement")]
    assert out["f"][0]["action"] == "phase1"


class ExcludingComm(FakeComm):
    def __init__(self, *a, **k):
        super().__init__(*a, **k)
        self.members = set(range(self.nranks))
        self.excluded = []

    def exclude(self, dead, store=None):
        self.excluded.append(set(dead))
        self.members -= set(dead)


def test_fault_rule_excludes_a_rank_that_never_signals():
    """phase 1 ends, the late rank stays silent for more than
    T_fault = factor x (phase-1 end - first ready): it is excluded, phase 2
    is not issued; the next round prices and masks the survivors only."""
    n, t = 4, 5
    comm = ExcludingComm(n)
    for r in range(3):
        comm.board[r] = t               # rank 3 never signals
    calls = []

    def issue(m, late):
        calls.append((m, late))
        time.sleep(0.01)                # "phase 1" runs 10 ms after the first ready rank
    oc = C.OnlineCoordinator(comm, lambda: _policy(n, 1e-3), cycle=1e-4, fault_factor=2.0, timeout=5.0)
    t0 = time.perf_counter()
    res = oc.allreduce(issue)
    took = time.perf_counter() - t0
    assert calls == [(0b0111, "join")] and res["faulty"] == [3] and res["phase2_after_s"] is None
    assert comm.excluded == [{3}] and comm.members == {0, 1, 2}
    assert 0.02 < took < 1.0            # ~ phase 1 (>= 10 ms) + 2 x that, not the timeout
    # next round: all survivors ready -> one "full" call over the survivors' mask
    for r in range(3):
        comm.board[r] = t + 1
    calls.clear()
    res = oc.allreduce(lambda m, late: calls.append((m, late)))
    assert res["action"] == "full" and calls == [(0b0111, None)]


def test_late_rank_within_t_fault_is_not_excluded():
    n, t = 4, 5
    comm = ExcludingComm(n)
    for r in range(3):
        comm.board[r] = t
    calls = []

    def issue(m, late):
        calls.append((m, late))
        if late == "join":
            time.sleep(0.02)
            threading.Timer(0.01, lambda: comm.board.__setitem__(3, t)).start()   # ready 10 ms after phase 1
    oc = C.OnlineCoordinator(comm, lambda: _policy(n, 1e-3), cycle=1e-4, fault_factor=5.0, timeout=5.0)
    res = oc.allreduce(issue)
    assert res["faulty"] == [] and comm.excluded == []
    assert calls == [(0b0111, "join"), (0b0111, "complement")]


def test_follower_takes_the_leaders_fault_decision():
    n, t = 3, 3
    board = (ctypes.c_uint64 * 128)()
    board[0] = board[1] = t            # rank 2 never signals
    lc = ExcludingComm(n, 0, False, board, t - 1)
    fc = ExcludingComm(n, 1, False, board, t - 1)
    leader = C.OnlineCoordinator(lc, lambda: _policy(n, 1e-3), cycle=1e-4, fault_factor=1.0, timeout=5.0)
    follower = C.OnlineCoordinator(fc, lambda: pytest.fail("a follower must not decide"), cycle=1e-4,
                                   timeout=5.0)
    out = {}

    def run(name, oc):
        calls = []
        out[name] = (oc.allreduce(lambda m, late: calls.append((m, late))), calls)

    tf = threading.Thread(target=run, args=("f", follower))
    tf.start()
    run("l", leader)
    tf.join()
    assert out["l"][1] == out["f"][1] == [(0b011, "join")]
    assert out["l"][0]["faulty"] == out["f"][0]["faulty"] == [2]
    assert lc.excluded == fc.excluded == [{2}]
