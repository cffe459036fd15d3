"""relay=store (relays as real store-and-forward hops) on CPU: both
loaders accept it, the oracle's results do not depend on it (bytes arrive
unchanged either way), and the plan compiler gives every pure relay a
forwarding task (DIRECT: a slot + flag at the relay; STAGED: a landing slot
at the relay and a push to its consumer) while keeping tuples unchanged."""

import itertools

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from oracle import collectives as oc
from oracle import strategy as ost
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import generator as G
from synth import rank_tensors

CHAIN = [-1, 0, 1, 2]          # 3 -> 2 -> 1 -> 0
BINARY = [-1, 0, 0, 1, 1, 2, 2]


@pytest.mark.parametrize("parent", [CHAIN, BINARY])
def test_oracle_result_independent_of_relay_mode(parent):
    n = len(parent)
    xs = rank_tensors("f32", 3001, n)
    for k in range(1, n + 1):
        for R in itertools.combinations(range(n), k):
            a = oc.allreduce(xs, G.allreduce_trees([parent], chunk=4096), set(R), "f32")
            b = oc.allreduce(xs, G.allreduce_trees([parent], chunk=4096, relay="store"), set(R), "f32")
            assert all(np.array_equal(x.view(np.uint32), y.view(np.uint32)) for x, y in zip(a, b))


def test_loaders_agree():
    text = G.allreduce_trees([CHAIN, [1, -1, 1, 2]], chunk=4096, relay="store")
    st = ost.parse(text)
    assert all(s.relay == "store" for s in st.subs)
    assert pkg.strategy_check(text)[2] == len(st.subs)
    # the behaviour tuples do not change
    for mask in range(1, 16):
        assert pkg.adapcc.strategy_tuples(text, 0, mask) == \
            pkg.adapcc.strategy_tuples(G.allreduce_trees([CHAIN], chunk=4096), 0, mask)


@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_chain_of_relays_forwards(mode):
    """Mask {0, 3} on 3 -> 2 -> 1 -> 0: ranks 2 and 1 are pure relays.
    bypass: rank 3's chunk goes straight to the root; store: 2 and 1 each
    own a forwarding task that waits for the previous hop (a chain of flags)."""
    mask = 0b1001
    by = A.plan_items(G.allreduce_trees([CHAIN], chunk=65536), 1 << 18, "f32", mask, 32, mode=mode)[1]
    st = A.plan_items(G.allreduce_trees([CHAIN], chunk=65536, relay="store"), 1 << 18, "f32", mask, 32,
                      mode=mode)[1]
    fwd = [t for t in st if int(t["owner"]) in (1, 2) and t["nsrc"] == 1 and t["npost"] == 1 and t["ndst"] == 1]
    assert sorted(int(t["owner"]) for t in fwd) == [1, 2]
    assert [int(t["nwait"]) for t in sorted(fwd, key=lambda t: -int(t["owner"]))] == [
        0 if mode == "direct" else 1, 1]            # 2 reads x3 (DIRECT) or its landing slot (STAGED)
    assert not any(int(t["owner"]) in (1, 2) and t["npost"] == 1 and t["ndst"] == 1 and t["nsrc"] == 1 and
                   int(t["nwait"]) <= 1 and int(t["level"]) > 0 for t in by if mode == "direct")
    assert max(int(t["level"]) for t in st) > max(int(t["level"]) for t in by)
