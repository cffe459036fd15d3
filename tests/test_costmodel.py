"""NEXT-2 cost model and profiler pins (-m "not gpu"): the alpha-beta closed form
of P:L113, least squares on exact synthetic probes, the Fig. 5(b) probe
schedule, the link-load model of Fig. 8(b), eq. 5 on a
single edge by hand, and chunk choice behaving as the pipelining trade-off."""

import math

import pytest

from paper_conf_icdcs_zhaozw24_b200 import costmodel as CM
from paper_conf_icdcs_zhaozw24_b200 import generator as G


def test_alpha_beta_closed_form():
    alpha, beta, n, s = 3e-6, 1 / 700e9, 8, 1 << 20
    t_many = n * (alpha + beta * s)
    t_once = alpha + beta * n * s
    a, b = CM.solve_alpha_beta(t_many, t_once, n, s)
    assert math.isclose(a, alpha, rel_tol=1e-9) and math.isclose(b, beta, rel_tol=1e-9)


def test_least_squares_recovers_exact_model():
    alpha, beta = 5e-6, 1 / 400e9
    calls = iter(range(10 ** 6))

    def copy(nbytes):
        next(calls)
        return alpha + beta * nbytes

    a, b, samples = CM.probe_link(copy, sizes=(4096, 1 << 20), repeats=(1, 4, 16))
    assert math.isclose(a, alpha, rel_tol=1e-6) and math.isclose(b, beta, rel_tol=1e-6)
    assert len(samples) == 12


def test_probe_rounds_are_permutations():
    for n in (2, 3, 4, 8):
        rounds = CM.probe_rounds(n)
        assert len(rounds) == n - 1
        seen = set()
        for r in rounds:
            assert sorted(a for a, _ in r) == list(range(n))       # one outgoing flow per port
            assert sorted(b for _, b in r) == list(range(n))       # one incoming flow per port
            assert all(a != b for a, b in r)
            seen |= set(r)
        assert len(seen) == n * (n - 1)                            # every ordered pair once


def test_link_loads_fig8b():
    parent = [1, 2, -1, 1]                      # 0->1, 3->1, 1->2
    assert CM.link_loads(parent)[(1, 2)] == 1
    assert CM.link_loads(parent, noagg={1})[(1, 2)] == 3


def test_single_edge_eq5_by_hand():
    alpha, beta = CM.uniform_links(2, 2e-6, 1e-9)
    S, C = 10_000_000, 1_000_000
    T, h, bottle = CM.tree_time([-1, 0], S, C, alpha, beta)
    t = 2e-6 + 1e-9 * C
    assert math.isclose(h, t) and math.isclose(bottle, t)
    assert math.isclose(T, t + math.ceil(S / C) * t)


def test_chunk_tradeoff_latency_vs_pipelining():
    n = 8
    alpha, beta = CM.uniform_links(n, 3e-6, 1 / 700e9)
    S = 256 << 20
    best, scored = CM.best_chunk(lambda c: G.allreduce_stars(n, chunk=c), S, alpha, beta)
    times = dict((c, t) for t, c in scored)
    # tiny chunks pay alpha per chunk, huge chunks lose pipelining: the optimum is interior
    assert times[best] <= min(times.values()) + 1e-15
    assert best not in (1 << 14,)
    # a deeper tree (chain) is never faster than the star on a uniform switch
    chain = G.allreduce_trees([G.chain_parent(list(range(n)))], chunk=best)
    assert CM.allreduce_time(chain, S, alpha, beta) >= CM.allreduce_time(G.allreduce_stars(n, chunk=best), S,
                                                                          alpha, beta)


# ------------------------------------------------------------- AlltoAll (routes)
def test_alltoall_loads_match_oracle():
    """Product cost model's N_ij (via the C loader) = the oracle's (own parser)."""
    import random

    from oracle import loads as OL
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    rng = random.Random(21)
    for _ in range(20):
        n = rng.randint(3, 8)
        lines = []
        for _ in range(rng.randint(1, 3)):
            routes = {}
            for s in range(n):
                for d in range(n):
                    if s != d and rng.random() < 0.3:
                        others = [g for g in range(n) if g not in (s, d)]
                        routes[(s, d)] = rng.sample(others, rng.randint(1, min(2, len(others))))
            lines.append((rng.randint(1, 3), routes))
        text = G.alltoall_routed(n, lines)
        R = {g for g in range(n) if rng.random() < 0.7} or {0}
        exp = {}
        for N in OL.alltoall_link_loads(text, R):
            for e, v in N.items():
                exp[e] = exp.get(e, 0) + v
        assert CM.alltoall_link_loads(text, R) == exp


def test_alltoall_time_closed_form_direct():
    """Direct flows on a uniform switch: every edge carries one flow, so
    T = t + ceil(S/C) t with t = alpha + beta C (eqs. 2, 5, 6)."""
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    n, C, S = 8, 1 << 20, 16 << 20
    a, b = 2e-6, 1 / 700e9
    A_, B_ = CM.uniform_links(n, a, b)
    t = a + b * C
    assert CM.alltoall_time(G.alltoall_direct(n, chunk=C), S, A_, B_) == pytest.approx(t + (S // C) * t)


def test_alltoall_detour_around_a_slow_link_pays_off():
    """A 10x slower link (heterogeneous links, the paper's motivation):
    routing its flows through a relay beats the direct path in the model."""
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    n, C, S = 4, 1 << 20, 64 << 20
    A_, B_ = CM.uniform_links(n, 2e-6, 1 / 700e9)
    B_[0][1] = B_[1][0] = 10 / 700e9
    direct = CM.alltoall_time(G.alltoall_direct(n, chunk=C), S, A_, B_)
    detour = CM.alltoall_time(G.alltoall_detour(n, [(0, 1), (1, 0)], chunk=C), S, A_, B_)
    assert detour < 0.5 * direct
