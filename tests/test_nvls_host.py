"""NVLS switch edges (NEXT-2) on CPU: the C++ loader and the oracle agree on
nvls lines, the plan compiler emits the copy-in / switch-reduce / copy-out
tasks with the right flags (host-only adapcc_plan_items, planned as if NVLS
scratch existed), partial masks and excluded ranks are refused."""

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from oracle import strategy as ost
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import generator as G


@pytest.mark.parametrize("n,star_w", [(2, 0), (4, 1), (8, 3)])
def test_loader_matches_oracle(n, star_w):
    text = G.allreduce_nvls(n, chunk=65536, nvls_weight=2, star_weight=star_w)
    st = ost.parse(text)
    nn, coll, nsubs = pkg.strategy_check(text)
    assert (nn, coll, nsubs) == (n, 0, len(st.subs))
    for m, sub in enumerate(st.subs):
        w, c, par, _ = pkg.strategy_sub(text, m)
        assert (w, c) == (sub.weight, sub.chunk)
        assert (sub.kind == "nvls") == (par == [-2] * n)
    for count in (1000, 1003):
        assert pkg.strategy_partition(text, count, "f32") == ost.partition(count, 4, [s.weight for s in st.subs])


@pytest.mark.parametrize("n", [2, 4, 8])
@pytest.mark.parametrize("count", [1 << 20, (1 << 20) + 3])
def test_nvls_plan_tasks(n, count):
    text = G.allreduce_nvls(n, chunk=1 << 18)
    items, tasks = A.plan_items(text, count, "f32", (1 << n) - 1, 64, mode="staged")
    # per slice k: n copy-ins (1 post to k), 1 switch reduce (n waits, n posts), n copy-outs (1 wait)
    reduce_t = [t for t in tasks if t["nwait"] == n and t["npost"] == n]
    assert len(reduce_t) == n and sorted(int(t["owner"]) for t in reduce_t) == list(range(n))
    cin = [t for t in tasks if t["nwait"] == 0 and t["npost"] == 1 and t["nsrc"] == 1]
    cout = [t for t in tasks if t["nwait"] == 1 and t["npost"] == 0 and t["nsrc"] == 1]
    assert len(cin) >= n * n and len(cout) >= n * n
    # the switch-reduced slices tile the 16-byte-aligned range; the tail (if any) goes to a star at rank 0
    spans = sorted((int(t["lo"]), int(t["hi"])) for t in reduce_t)
    assert spans[0][0] == 0 and all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
    assert spans[-1][1] == count // 4 * 4
    assert all((hi - lo) % 4 == 0 for lo, hi in spans)
    for it in items:                          # every item lies inside its task's range
        t = tasks[it["task"]]
        a = int(t["lo"]) + int(it["chunk"]) * int(t["chunk_elems"]) + int(it["off"])
        assert int(t["lo"]) <= a and a + int(it["len"]) <= int(t["hi"])


def test_nvls_needs_the_whole_mask():
    text = G.allreduce_nvls(4)
    with pytest.raises(A.AdapccError) as e:
        A.plan_items(text, 1 << 16, "f32", 0b0111, 64, mode="staged")
    assert e.value.code == A.UNSUPPORTED
    with pytest.raises(A.AdapccError) as e:
        A.plan_items(text, 1 << 16, "f32", 0b1111, 64, mode="staged", late="join")
    assert e.value.code == A.UNSUPPORTED


def test_excluded_rank_invalidates_nvls():
    text = G.allreduce_nvls(4)
    with pytest.raises(A.AdapccError) as e:
        A.plan_stats(text, 1 << 16, "f32", 0b0111, members={0, 1, 2})
    assert e.value.code == A.INVALID_STRATEGY
