"""Routed AlltoAll (SURVEY §8(a) a9 "direct or along a route"; eq. 1,
P:L209-211): oracle pins, loader cross-check, plan byte accounting (CPU)."""

import itertools
import os
import random

import pytest

from oracle import loads as OL
from oracle import strategy as OS
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import generator as G

GOLD = os.path.join(os.path.dirname(__file__), "golden", "a2a_routes.txt")


def _text(n, route, lines=1):
    return (f"adapcc-strategy 1\nnranks {n}\ncollective alltoall\n" +
            "".join(f"a2a weight=1 chunk=4096 route={route}\n" for _ in range(lines)))


def _random_routes(rng, n, k):
    routes = {}
    pairs = [(s, d) for s in range(n) for d in range(n) if s != d]
    for s, d in rng.sample(pairs, min(k, len(pairs))):
        others = [g for g in range(n) if g not in (s, d)]
        if not others:
            continue
        routes[(s, d)] = rng.sample(others, rng.randint(1, min(3, len(others))))
    return routes


# ------------------------------------------------------------------ oracle pins
def test_golden_link_loads():
    """Hand-worked loads (tests/golden/a2a_routes.txt, P:L169/L171/L209-211)."""
    cases = 0
    for line in open(GOLD):
        line = line.split("#", 1)[0].strip()
        if not line:
            continue
        head, tail = line.split("|")
        n, ready, route = head.split()
        n = int(n)
        R = {int(g) for g in ready.split(",")}
        exp = {}
        for tok in tail.split():
            i, j, v = map(int, tok.split(","))
            exp[(i, j)] = v
        N = OL.alltoall_link_loads(_text(n, route), R)[0]
        got = {(i, j): N.get((i, j), 0) for i in range(n) for j in range(n) if i != j}
        assert got == exp
        cases += 1
    assert cases == 2


def test_direct_loads_closed_form():
    """Without routes every flow is its own edge: N_ij = 1 iff i is ready."""
    for n in (2, 3, 5, 8):
        for R in ({0}, set(range(n)), set(range(0, n, 2))):
            N = OL.alltoall_link_loads(G.alltoall_direct(n), R)[0]
            exp = {(i, j): 1 for i in R for j in range(n) if j != i}
            assert N == exp


def test_flow_conservation_eq1():
    """Eq. 1: out - in = 1 at Src_f, -1 at Dst_f, 0 elsewhere, for every flow."""
    rng = random.Random(5)
    for n in (3, 4, 6, 8):
        st = OS.parse(_text(n, ";".join(f"{s}:{d}:{','.join(map(str, h))}"
                                        for (s, d), h in _random_routes(rng, n, 2 * n).items())))
        sub = st.subs[0]
        for s, d in itertools.permutations(range(n), 2):
            E = OL.flow_edges(sub, s, d)
            assert len(set(E)) == len(E)
            for i in range(n):
                bal = sum(1 for (a, _) in E if a == i) - sum(1 for (_, b) in E if b == i)
                assert bal == (1 if i == s else -1 if i == d else 0)


def test_total_bytes_is_hops_times_blocks():
    """Sum over edges = sum over flows of (relays + 1) x the flow's bytes."""
    rng = random.Random(7)
    n, cnt = 6, 1001
    routes = _random_routes(rng, n, 10)
    text = G.alltoall_routed(n, [(3, routes), (1, {})], chunk=4096)
    R = {0, 1, 3, 4}
    EB = OL.alltoall_edge_bytes(text, cnt, "f32", R)
    b = OS.partition(cnt, 4, [3 * n, 1 * n])
    exp = 0
    for s in R:
        for d in range(n):
            if d != s:
                exp += (b[1] - b[0]) * 4 * (len(routes.get((s, d), [])) + 1) + (b[2] - b[1]) * 4
    assert sum(EB.values()) == exp


BAD = ["0:0:1", "0:1:", "0:1:1", "0:1:0", "0:1:2,2", "0:9:1", "-1:1:2", "0:1:2;0:1:3", "0:1", "0:1:2:3",
       "x:1:2", "0:1:+2", ""]


@pytest.mark.parametrize("route", BAD)
def test_bad_routes_rejected_by_both(route):
    text = _text(4, route)
    with pytest.raises(OS.StrategyError):
        OS.parse(text)
    with pytest.raises(A.AdapccError):
        A.strategy_check(text)


def test_route_key_only_on_a2a():
    t = "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0 route=0:1:0\n"
    with pytest.raises(OS.StrategyError):
        OS.parse(t)
    with pytest.raises(A.AdapccError):
        A.strategy_check(t)


# ------------------------------------------------------------ loader cross-check
def test_loader_routes_match_oracle():
    rng = random.Random(11)
    for trial in range(30):
        n = rng.randint(3, 9)
        lines = [(rng.randint(1, 4), _random_routes(rng, n, rng.randint(0, 2 * n))) for _ in range(rng.randint(1, 3))]
        text = G.alltoall_routed(n, lines, chunk=16 * rng.randint(1, 64))
        st = OS.parse(text)
        for m, sub in enumerate(st.subs):
            for s, d in itertools.permutations(range(n), 2):
                assert A.strategy_route(text, m, s, d) == list(sub.routes.get((s, d), ())), (text, m, s, d)


@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_plan_egress_matches_oracle_link_bytes(mode):
    """Per rank, the plan's cross-rank bytes = the oracle's bytes on that
    rank's outgoing edges (every hop is one push, P:L171 + P:L209-211)."""
    rng = random.Random(13 if mode == "direct" else 17)
    for trial in range(12):
        n = rng.randint(3, 8)
        lines = [(rng.randint(1, 3), _random_routes(rng, n, rng.randint(0, 3 * n))) for _ in range(rng.randint(1, 3))]
        text = G.alltoall_routed(n, lines, chunk=16 * rng.randint(4, 256))
        cnt = rng.randint(1, 5000)
        dtype = rng.choice(["f32", "bf16"])
        R = {g for g in range(n) if rng.random() < 0.7} or {0}
        mask = sum(1 << g for g in R)
        EB = OL.alltoall_edge_bytes(text, cnt, dtype, R)
        for r in range(n):
            st = A.plan_stats(text, cnt, dtype, mask, 0, mode, r, 64 << 20)
            egress = sum(v for (i, _), v in EB.items() if i == r)
            assert st["remote_bytes"] == egress, (text, cnt, R, r)


def test_detour_generator_avoids_slow_edges():
    n = 8
    slow = [(0, 1), (1, 0), (2, 5), (7, 3)]
    text = G.alltoall_detour(n, slow, chunk=1 << 16)
    N = OL.alltoall_link_loads(text)[0]
    for e in slow:
        assert N.get(e, 0) == 0
    assert max(N.values()) <= 2
