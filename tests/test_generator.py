"""Strategy generator: valid text (oracle parser) and the link-load model (-m "not gpu").

Pins: SURVEY §8(d) d-4 table, computed from the paper's link-load model
 on a uniform switch -- full AllReduce 1.75 S per GPU at n = 8;
phase 1 (6 ready) 1.714 S with relays as roots, 2.00 S as leaves; phase 2
(2 ready) 1.158 S with relays as roots, 4.00 S as leaves.
"""

import pytest

from oracle import strategy as ost
from paper_conf_icdcs_zhaozw24_b200 import generator as G


@pytest.mark.parametrize("text", [
    G.allreduce_stars(8), G.allreduce_stars(8, roots=[0, 1]), G.allreduce_double_binary(8),
    G.allreduce_ring(8), G.allgather_stars(4), G.allgather_chains(4), G.alltoall_direct(8, lines=4),
    G.allreduce_mask_aware_stars(8, {0, 1, 2, 4, 5, 7}),
])
def test_generated_text_parses(text):
    st = ost.parse(text)
    assert st.nranks in (4, 8)


def test_double_binary_trees_are_trees_and_differ():
    st = ost.parse(G.allreduce_double_binary(8))
    assert st.subs[0].parent != st.subs[1].parent


@pytest.mark.parametrize("ready,roots,expect", [
    (set(range(8)), True, 1.75),
    ({0, 1, 2, 4, 5, 7}, True, 1.714),
    ({0, 1, 2, 4, 5, 7}, False, 2.00),
    ({3, 6}, True, 1.158),
    ({3, 6}, False, 4.00),
])
def test_mask_aware_weights_reproduce_load_table(ready, roots, expect):
    _, w, t = G.mask_aware_star_weights(8, ready, relays_as_roots=roots)
    assert abs(sum(w) - 1) < 1e-9
    assert abs(t - expect) < 2e-3


def test_full_mask_load_is_2_n_minus_1_over_n():
    for n in (2, 4, 8):
        eg, ig, t = G.star_loads(n, set(range(n)), [1.0 / n] * n)
        assert abs(t - 2 * (n - 1) / n) < 1e-12
