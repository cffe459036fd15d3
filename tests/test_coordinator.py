"""Relay coordinator pins (-m "not gpu"): S of P:L135 in closed form, the
break-even (ski-rental) decision rule of P:L133-137 on hand-built traces, its
competitive ratio <= 2 against the offline optimum on random traces, and the
T_fault = 5x rule of P:L139."""

import math

import numpy as np
import pytest

from paper_conf_icdcs_zhaozw24_b200 import coordinator as C


def test_comm_volume_closed_forms():
    # AllReduce 2(N-1) x tensor, AlltoAll N x tensor, Broadcast tensor
    assert C.comm_volume("allreduce", 8, 10) == 140
    assert C.comm_volume("alltoall", 8, 10) == 80
    assert C.comm_volume("broadcast", 8, 10) == 10
    assert C.comm_volume("allreduce", 1, 10) == 0


def test_all_ready_at_once_runs_full_collective():
    c = C.Coordinator(8, "allreduce", 1 << 20, 100e9, 1e-6)
    d = c.step(0.0, range(8))
    assert d.action == "full"


def test_break_even_time_hand_derived():
    # 6 of 8 ready from t=0, two never ready: the coordinator waits while
    # waited + cycle <= buy_cost and buys in the first cycle that would exceed it
    n, S, bw, cyc = 8, 64 << 20, 100e9, 10e-6
    c = C.Coordinator(n, "allreduce", S, bw, cyc)
    # buy cost by hand: phase 1 with 6 workers + phase 2 with the 2 late + 1
    p1 = 2 * 5 * S / (6 * bw)
    p2 = 2 * 2 * S / (3 * bw)
    assert math.isclose(c.buy_cost(6), p1 + p2)
    k = 0
    while True:
        d = c.step(k * cyc, set(range(6)))
        if d.action != "wait":
            break
        k += 1
    assert d.action == "phase1" and d.relays == {6, 7}
    assert k == math.floor((p1 + p2) / cyc)   # k cycles waited, the (k+1)-th would exceed


def test_nothing_ready_never_buys():
    c = C.Coordinator(4, "allreduce", 1 << 20, 1e9, 1e-3)
    for k in range(1000):
        assert c.step(k * 1e-3, set()).action == "wait"


@pytest.mark.parametrize("coll", ["allreduce", "alltoall"])
def test_competitive_ratio_at_most_two(coll):
    rng = np.random.default_rng(0)
    n, S, bw, cyc = 8, 32 << 20, 100e9, 5e-6
    worst = 0.0
    for _ in range(300):
        base = rng.exponential(50e-6, size=n)
        if rng.random() < 0.5:   # a straggler or two
            base[rng.integers(0, n, size=rng.integers(1, 3))] += rng.exponential(2e-3)
        arrivals = list(base - base.min())
        c = C.Coordinator(n, coll, S, bw, cyc)
        _, finish = c.run(arrivals)
        opt = C.offline_optimum(arrivals, n, coll, S, bw, cyc)
        worst = max(worst, finish / opt)
        assert finish <= 2 * opt + 2 * cyc
    assert worst >= 1.0


def test_fault_rule_five_times_since_fastest_ready():
    ready = {0: 0.0, 1: 1.0, 2: None}
    # phase 1 ended at t=2 -> T_fault = 5 x (2 - 0) = 10
    assert C.faulty_workers(ready, 2.0, now=11.9) == set()
    assert C.faulty_workers(ready, 2.0, now=12.0) == {2}
