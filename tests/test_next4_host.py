"""NEXT-4 primitives (Reduce / Broadcast / ReduceScatter): C++ loader and plan
vs the oracle on the host (-m "not gpu")."""

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from oracle import strategy as ost
from paper_conf_icdcs_zhaozw24_b200 import generator as G
from tests import strategies as S

TEXTS = [
    G.reduce_trees([S.star(5, 2), S.chain([0, 1, 3, 4, 2]), [2, 2, -1, 1, 3]], [1, 2, 3], 64, [(), (), (1,)]),
    G.broadcast_trees(3, [S.star(6, 3), S.chain([0, 1, 2, 4, 5, 3])], [2, 1], 128),
    G.reducescatter_stars(8),
    G.reducescatter_trees([(0, S.star(3, 0), 1), (1, S.chain([0, 2, 1]), 2), (2, S.star(3, 2), 1),
                           (1, S.star(3, 1), 5)], 3, 48),
]


@pytest.mark.parametrize("text", TEXTS)
def test_loader_matches_oracle(text):
    st = ost.parse(text)
    n, coll, nsubs = pkg.strategy_check(text)
    assert (n, nsubs) == (st.nranks, len(st.subs))
    assert coll == {"reduce": 3, "broadcast": 4, "reducescatter": 5}[st.collective]
    for m, sub in enumerate(st.subs):
        w, c, par, src = pkg.strategy_sub(text, m)
        assert (w, c, par, src) == (sub.weight, sub.chunk, sub.parent, sub.src)


def test_reducescatter_partition_per_block():
    text = TEXTS[3]
    st = ost.parse(text)
    for b in range(3):
        ws = [s.weight for s in st.subs if s.src == b]
        assert pkg.strategy_partition(text, 4099, "f32", src=b) == ost.partition(4099, 4, ws)


def test_plan_traffic_reduce_and_reducescatter():
    n, count = 8, 1 << 20
    full = (1 << n) - 1
    # Reduce DIRECT, one star at root 0: read every input once, write the root's output once
    st = pkg.plan_stats(G.reduce_trees([S.star(n, 0)]), count, "f32", full, mode="direct")
    assert st["bytes_read"] == n * count * 4 and st["bytes_written"] == count * 4
    # ReduceScatter DIRECT: read every input once, write n blocks of count/n
    st = pkg.plan_stats(G.reducescatter_stars(n), count // n, "f32", full, mode="direct")
    assert st["bytes_read"] == n * count * 4 and st["bytes_written"] == count * 4
    # ReduceScatter STAGED per rank: pushes (n-1)/n S remote, no broadcast back
    st = pkg.plan_stats(G.reducescatter_stars(n), count // n, "f32", full, mode="staged", rank=3)
    assert st["remote_bytes"] == (n - 1) * count * 4 // n
