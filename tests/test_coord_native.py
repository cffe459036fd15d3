"""Native coordinator loops (adapcc_coord_decide / adapcc_coord_await,
NEXT-1 / NEXT-3) on CPU: host-only C functions over a board in host memory.
Checked against the Python policy (Coordinator.step, the break-even rule of
P:L133-137) and the T_fault rule (faulty_workers)."""

import ctypes
import threading
import time

import pytest

from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import coordinator as C


def _board():
    b = (ctypes.c_uint64 * 128)()
    return b, ctypes.addressof(b)


def test_everyone_ready_is_full_at_once():
    b, addr = _board()
    for r in range(4):
        b[r] = 7
    full, ready, t_first, t_dec = A.coord_decide(addr, 4, {0, 1, 2, 3}, 7, [1.0] * 5, 1e-4, 1.0)
    assert full and ready == {0, 1, 2, 3} and 0 <= t_dec - t_first < 0.01


def test_old_tickets_do_not_count_and_members_limit_the_set():
    b, addr = _board()
    b[0], b[1], b[2] = 7, 6, 9          # rank 1 signalled an older collective only
    full, ready, _, _ = A.coord_decide(addr, 3, {0, 2}, 7, [1.0] * 4, 1e-4, 1.0)
    assert full and ready == {0, 2}     # rank 1 is excluded: {0, 2} is everyone


@pytest.mark.parametrize("buy_cycles", [0.5, 3, 20])
def test_break_even_matches_the_python_policy(buy_cycles):
    """A fixed ready set: the native loop buys after the same number of
    cycles as Coordinator.step (waited + cycle > buy_cost(k))."""
    cycle = 2e-4
    n, k = 8, 6
    pol = C.Coordinator(n, "allreduce", 1.0, 1.0, cycle)
    pol.buy_cost = lambda kk: buy_cycles * cycle
    steps = 0
    while pol.step(steps * cycle, set(range(k))).action == "wait":
        steps += 1
    b, addr = _board()
    for r in range(k):
        b[r] = 3
    t0 = time.perf_counter()
    full, ready, _, t_dec = A.coord_decide(addr, n, set(range(n)), 3, [buy_cycles * cycle] * (n + 1), cycle, 5.0)
    assert not full and ready == set(range(k))
    waited = t_dec - t0
    assert steps * cycle - 1e-4 <= waited < steps * cycle + 0.02, (steps, waited)


def test_decide_times_out_when_nobody_is_ready():
    b, addr = _board()
    with pytest.raises(TimeoutError):
        A.coord_decide(addr, 2, {0, 1}, 1, [0.0] * 3, 1e-4, 0.01)


def test_decide_rejects_bad_members():
    b, addr = _board()
    with pytest.raises(A.AdapccError):
        A.coord_decide(addr, 2, {0, 5}, 1, [0.0] * 3, 1e-4, 0.01)


def test_await_returns_once_the_late_ranks_signal():
    b, addr = _board()
    threading.Timer(0.02, lambda: (b.__setitem__(3, 4), b.__setitem__(6, 4))).start()
    t0 = time.perf_counter()
    dead = A.coord_await(addr, 8, {3, 6}, 4, None, None, None, 5.0)
    assert dead == set() and 0.015 < time.perf_counter() - t0 < 1.0


def test_await_applies_t_fault():
    """P:L139 with phase 1 already ended at the call (no event): first ready
    30 ms ago, factor 2 -> faulty after 2 x 30 ms; the same verdict as
    faulty_workers on the same times."""
    b, addr = _board()
    b[6] = 4                                     # 6 signalled, 3 never does
    t_first = time.perf_counter() - 0.03
    t0 = time.perf_counter()
    dead = A.coord_await(addr, 8, {3, 6}, 4, None, t_first, 2.0, 5.0)
    took = time.perf_counter() - t0
    assert dead == {3}
    assert 0.055 < took < 0.5, took
    assert C.faulty_workers({0: t_first, 3: None, 6: t_first}, t0, t0 + took, factor=2.0) == {3}


def test_await_times_out_without_fault_rule():
    b, addr = _board()
    with pytest.raises(TimeoutError):
        A.coord_await(addr, 4, {1}, 4, None, time.perf_counter(), None, 0.02)
