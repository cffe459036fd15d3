"""Pins for the CPU oracle (-m "not gpu").

Each test checks the oracle against something other than itself: values the
paper prints (tests/golden/, cited there), hand-derived IEEE results, closed
forms, invariants, brute force over every small tree/mask, or an independent
library (ml_dtypes).  See DESIGN.md §4 for the pin table.
"""

import itertools
import os

import numpy as np
import pytest

from oracle import bf16 as obf
from oracle import collectives as oc
from oracle import strategy as ost
from oracle import tuples as otu
from synth import rank_tensors
from tests import strategies as S


def _read_golden(golden_dir, name):
    rows = []
    with open(os.path.join(golden_dir, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def _ints(s):
    return [] if s == "-" else [int(t) for t in s.split(",")]


# --------------------------------------------------------------------------- bf16
def test_bf16_rne_matches_ml_dtypes():
    ml = pytest.importorskip("ml_dtypes")
    rng = np.random.default_rng(0)
    pats = rng.integers(0, 1 << 32, size=1 << 18, dtype=np.uint64).astype(np.uint32)
    # every tie / near-tie low half with both parities of the kept LSB
    hi = rng.integers(0, 1 << 16, size=4096, dtype=np.uint64).astype(np.uint32) << 16
    lows = np.array([0x0000, 0x7FFF, 0x8000, 0x8001, 0xFFFF], dtype=np.uint32)
    pats = np.concatenate([pats, (hi[:, None] | lows[None, :]).ravel(),
                           np.array([0x7F7FFFFF, 0xFF7FFFFF, 0x00000001, 0x807FFFFF,
                                     0x7F800000, 0x00000000, 0x80000000], dtype=np.uint32)])
    x = pats.view(np.float32)
    x = x[~np.isnan(x)]
    ours = obf.from_f32_rne(x)
    ref = x.astype(ml.bfloat16).view(np.uint16)
    assert np.array_equal(ours, ref)


def test_bf16_widen_is_exact_for_every_pattern():
    b = np.arange(1 << 16, dtype=np.uint32).astype(np.uint16)
    f = obf.to_f32(b)
    ok = ~np.isnan(f)
    assert np.array_equal(obf.from_f32_rne(f[ok]), b[ok])


# ------------------------------------------------------------------- strategy text
def test_partition_closed_form_examples():
    # hand-derived from reading Q9: u=16/esize, U=floor(count/u), b_m=floor(U*sum_{j<m}w/W)*u
    assert ost.partition(10, 4, [1, 1, 1]) == [0, 0, 4, 10]
    assert ost.partition(1 << 20, 4, [1] * 8) == [k * 131072 for k in range(8)] + [1 << 20]
    assert ost.partition(100, 2, [3, 1]) == [0, 72, 100]
    assert ost.partition(3, 4, [5]) == [0, 3]


@pytest.mark.parametrize("esize", [2, 4])
def test_partition_invariants(esize):
    rng = np.random.default_rng(1)
    for _ in range(300):
        m = int(rng.integers(1, 9))
        w = [int(v) for v in rng.integers(0, 50, size=m)]
        if sum(w) == 0:
            w[0] = 1
        count = int(rng.integers(0, 5000))
        b = ost.partition(count, esize, w)
        u = 16 // esize
        assert b[0] == 0 and b[-1] == count
        assert all(b[i] <= b[i + 1] for i in range(m))
        assert all(x % u == 0 for x in b[:-1])
        # each share is within one unit of its exact proportional share (of the aligned body)
        U = count // u
        tot = 0
        for i in range(m):
            exact = U * tot / sum(w) * u
            assert abs(b[i] - exact) < u
            tot += w[i]


def test_chunks_cover_partition():
    assert ost.chunks(0, 10, 16, 4) == [(0, 4), (4, 8), (8, 10)]
    assert ost.chunks(5, 5, 16, 4) == []


def test_ring_expansion_closed_form():
    st = ost.parse(S.allreduce_ring(4, chunk=64, weight=3))
    # reading Q13, hand-derived for order 0,1,2,3
    assert [s.parent for s in st.subs] == [[-1, 2, 3, 0], [1, -1, 3, 0],
                                         [1, 2, -1, 0], [1, 2, 3, -1]]
    assert [s.weight for s in st.subs] == [3, 3, 3, 3]


def test_ring_weight_equals_w_over_n_against_trees():
    # ring weight=4 plus a tree weight=1 at n=4: chains get 4/4 = 1 each, i.e. equal to the tree
    txt = S.allreduce_ring(4, chunk=64, weight=4) + S.tree_line(S.star(4, 0), 1, 64)
    st = ost.parse(txt)
    assert [s.weight for s in st.subs] == [4, 4, 4, 4, 4]


BAD = [
    "",
    "adapcc-strategy 2\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 0\ncollective allreduce\ntree weight=1 chunk=16 parent=-1\n",
    "adapcc-strategy 1\nnranks 65\ncollective allreduce\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\n",
    "adapcc-strategy 1\nnranks 2\ncollective gather\ntree weight=1 chunk=16 parent=-1,0\n",
    # reduce trees must share one root; broadcast lines one src; rtree root == dst;
    # every reducescatter block needs a positive-weight line
    "adapcc-strategy 1\nnranks 2\ncollective reduce\ntree weight=1 chunk=16 parent=-1,0\n"
    "tree weight=1 chunk=16 parent=1,-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective reduce\nring weight=1 chunk=16 order=0,1\n",
    "adapcc-strategy 1\nnranks 2\ncollective broadcast\nbcast src=0 weight=1 chunk=16 parent=-1,0\n"
    "bcast src=1 weight=1 chunk=16 parent=1,-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective reducescatter\nrtree dst=0 weight=1 chunk=16 parent=1,-1\n"
    "rtree dst=1 weight=1 chunk=16 parent=1,-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective reducescatter\nrtree dst=0 weight=1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective reducescatter\nrtree dst=0 weight=1 chunk=16 parent=-1,0\n"
    "rtree dst=1 weight=0 chunk=16 parent=1,-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=8 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=24 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=0 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=-1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,-1\n",
    "adapcc-strategy 1\nnranks 3\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,2,1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,5\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0 noagg=0\n",
    "adapcc-strategy 1\nnranks 3\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0,0 noagg=1,1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0 bogus=1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\nring weight=1 chunk=16 order=0,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\nbcast src=0 weight=1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allgather\nbcast src=0 weight=1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allgather\nbcast src=0 weight=1 chunk=16 parent=1,-1\n"
    "bcast src=1 weight=1 chunk=16 parent=1,-1\n",
    "adapcc-strategy 1\nnranks 2\ncollective alltoall\na2a weight=1\n",
    "adapcc-strategy 1\nnranks 2\nnranks 2\ncollective alltoall\na2a weight=1 chunk=16\n",
    "adapcc-strategy 1\nnranks 2\ncollective alltoall\na2a weight=1x chunk=16\n",
    # relay=store|bypass on tree lines only
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\ntree weight=1 chunk=16 parent=-1,0 relay=copy\n",
    "adapcc-strategy 1\nnranks 2\ncollective reduce\ntree weight=1 chunk=16 parent=-1,0 relay=stored\n",
    "adapcc-strategy 1\nnranks 2\ncollective allgather\nbcast src=0 weight=1 chunk=16 parent=-1,0 relay=store\n"
    "bcast src=1 weight=1 chunk=16 parent=1,-1\n",
    # nvls (NEXT-2 switch reduction): allreduce only, weight and chunk only
    "adapcc-strategy 1\nnranks 2\ncollective allgather\nnvls weight=1 chunk=16\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\nnvls weight=1 chunk=16 parent=-1,0\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\nnvls weight=1\n",
    "adapcc-strategy 1\nnranks 2\ncollective allreduce\nnvls weight=0 chunk=16\n",
]


@pytest.mark.parametrize("text", BAD)
def test_parser_rejects_malformed(text):
    with pytest.raises(ost.StrategyError):
        ost.parse(text)


def test_parser_accepts_comments_and_blank_lines():
    txt = "# hi\n\nadapcc-strategy 1   # v1\nnranks 2\n collective allreduce\n" \
          "tree weight=1 chunk=16 parent=-1,0  # root 0\n"
    st = ost.parse(txt)
    assert st.nranks == 2 and st.subs[0].parent == [-1, 0]


# --------------------------------------------------------------------- tuples (Fig. 7)
def test_fig7_tuples(golden_dir):
    for parent, ready, rank, tup in _read_golden(golden_dir, "fig7_tuples.txt"):
        t, _ = otu.behavior(_ints(parent), set(_ints(ready)))
        assert tuple(int(v) for v in t[int(rank)]) == tuple(_ints(tup)), (parent, ready, rank)


def test_fig8b_flow_counts(golden_dir):
    for parent, ready, noagg, nflows in _read_golden(golden_dir, "fig8b_loads.txt"):
        _, fl = otu.behavior(_ints(parent), set(_ints(ready)), frozenset(_ints(noagg)))
        assert len(fl[1]) == int(nflows)


def test_fig8b_sum_is_correct_either_way():
    xs = rank_tensors("i32", 33, 4)
    for noagg in ("", " noagg=1"):
        txt = S.header(4, "allreduce") + f"tree weight=1 chunk=16 parent=1,2,-1,1{noagg}\n"
        ys = oc.allreduce(xs, txt, {0, 1, 2, 3}, "i32")
        ref = oc.allreduce_exact(xs, {0, 1, 2, 3}, "i32")
        for y in ys:
            assert np.array_equal(y, ref)


def test_broadcast_tuples_reverse_the_tree():
    bt = otu.broadcast_tuples([-1, 0, 1, 1])
    assert bt == {0: (False, False, True), 1: (True, False, True),
                  2: (True, False, False), 3: (True, False, False)}


# ----------------------------------------------------------------------- Fig. 6
def test_fig6_relay_value4(golden_dir):
    for n, r1, v1, r2, v2 in _read_golden(golden_dir, "fig6_relay.txt"):
        n = int(n)
        ones = [np.ones(40, dtype=np.float32) for _ in range(n)]
        for parent in S.all_rooted_trees(n) if n <= 4 else [S.star(n, m) for m in range(n)]:
            txt = S.allreduce_trees([parent], chunk=16)
            ys = oc.allreduce(ones, txt, set(_ints(r1)), "f32")
            assert all(np.all(y == float(v1)) for y in ys)
            if r2 != "-":
                ys = oc.allreduce(ones, txt, set(_ints(r2)), "f32", accumulate=True, y_prev=ys)
                assert all(np.all(y == float(v2)) for y in ys)


# ---------------------------------------------------------------- reduction order
def test_fold_order_golden(golden_dir):
    for dtype, parent, xs_hex, exp in _read_golden(golden_dir, "fold_order.txt"):
        parent = _ints(parent)
        n = len(parent)
        np_t = np.uint32 if dtype == "f32" else np.uint16
        xs = [np.array([int(h, 16)], dtype=np_t) for h in xs_hex.split(",")]
        if dtype == "f32":
            xs = [x.view(np.float32) for x in xs]
        ys = oc.allreduce(xs, S.allreduce_trees([parent], chunk=16), set(range(n)), dtype)
        for y in ys:
            assert int(y.view(np_t)[0]) == int(exp, 16), (dtype, parent)


# ------------------------------------------------- brute force over every small tree
@pytest.mark.parametrize("n", [2, 3, 4])
def test_every_tree_every_mask_int32_and_intval_exact(n):
    count = 23  # ragged: not a multiple of the 16-byte unit
    xi = rank_tensors("i32", count, n)
    xf = rank_tensors("f32", count, n, dist="intval")
    nonroot_subsets = lambda p: [set(c) for k in range(n) for c in  # noqa: E731
                                 itertools.combinations([g for g in range(n) if p[g] != -1], k)]
    for parent in S.all_rooted_trees(n):
        for noagg in nonroot_subsets(parent):
            txt = S.allreduce_trees([parent], chunk=16, noaggs=[sorted(noagg)])
            for mask in range(1 << n):
                R = {r for r in range(n) if mask >> r & 1}
                yi = oc.allreduce(xi, txt, R, "i32")
                ri = oc.allreduce_exact(xi, R, "i32", count)
                yf = oc.allreduce(xf, txt, R, "f32")
                rf = oc.allreduce_exact(xf, R, "f32", count)
                for g in range(n):
                    assert np.array_equal(yi[g], ri), (parent, noagg, mask)
                    assert np.array_equal(yf[g].astype(np.float64), rf), (parent, noagg, mask)


def _kernel_depth(parent, R, noagg):
    t, _ = otu.behavior(parent, R, noagg)
    n = len(parent)
    best = 0
    for g in range(n):
        d, x = 0, g
        while x != -1:
            d += t[x][2]
            x = parent[x]
        best = max(best, d)
    return best


@pytest.mark.parametrize("n", [3, 4, 5])
def test_every_tree_fp_error_within_textbook_bound(n):
    """fp32: |y - sum| <= gamma_{k-1} * sum|x| ; bf16: d roundings of 2^-8 on top."""
    count = 64
    xf = rank_tensors("f32", count, n)
    xb = rank_tensors("bf16", count, n)
    trees = S.all_rooted_trees(n) if n <= 4 else [S.star(n, 0), S.chain(list(range(n)))]
    for parent in trees:
        txt = S.allreduce_trees([parent], chunk=16)
        for mask in range(1, 1 << n):
            R = {r for r in range(n) if mask >> r & 1}
            k = len(R)
            gam = (k - 1) * 2.0 ** -24 / (1 - (k - 1) * 2.0 ** -24)
            absf = np.sum(np.stack([np.abs(xf[r].astype(np.float64)) for r in R]), 0)
            yf = oc.allreduce(xf, txt, R, "f32")[0].astype(np.float64)
            assert np.all(np.abs(yf - oc.allreduce_exact(xf, R, "f32")) <= gam * absf + 1e-300)
            d = _kernel_depth(parent, R, frozenset())
            absb = np.sum(np.stack([np.abs(obf.to_f32(xb[r]).astype(np.float64)) for r in R]), 0)
            yb = obf.to_f32(oc.allreduce(xb, txt, R, "bf16")[0]).astype(np.float64)
            bound = ((1 + 2.0 ** -8) ** d * (1 + 2.0 ** -24) ** k - 1) * absb
            assert np.all(np.abs(yb - oc.allreduce_exact(xb, R, "bf16")) <= bound)
            # north_star tolerance for the star (d <= 1) case: 1e-2 relative (normwise)
            if d <= 1:
                err = np.max(np.abs(yb - oc.allreduce_exact(xb, R, "bf16"))) / max(np.max(absb), 1e-30)
                assert err <= 1e-2


def test_multitree_weights_and_ring_int32_exact():
    n = 8
    count = 1000 + 3
    xs = rank_tensors("i32", count, n)
    rng = np.random.default_rng(5)
    trees = [S.star(n, m) for m in range(n)] + [S.chain(list(rng.permutation(n)))]
    txts = [S.allreduce_trees(trees, weights=[int(w) for w in rng.integers(0, 5, len(trees))] + [0] * 0,
                              chunk=64),
            S.allreduce_ring(n, chunk=32, weight=2),
            S.allreduce_ring(n, chunk=32) + S.tree_line(S.star(n, 3), 5, 48, noagg=(1, 2))]
    for txt in txts:
        if sum(s.weight for s in ost.parse(txt).subs) == 0:
            continue
        for mask in (0xFF, 0xB7, 0x48, 0x01, 0x80):
            R = {r for r in range(n) if mask >> r & 1}
            ys = oc.allreduce(xs, txt, R, "i32")
            ref = oc.allreduce_exact(xs, R, "i32")
            for y in ys:
                assert np.array_equal(y, ref)


def test_broadcast_identity_all_ranks_bitwise_equal():
    n = 6
    xs = rank_tensors("f32", 517, n)
    txt = S.allreduce_trees([S.chain([5, 3, 1, 0, 2, 4]), S.star(n, 2)], weights=[3, 2], chunk=32)
    for mask in (0x3F, 0x15, 0x20):
        R = {r for r in range(n) if mask >> r & 1}
        ys = oc.allreduce(xs, txt, R, "f32")
        for y in ys[1:]:
            assert np.array_equal(y.view(np.uint32), ys[0].view(np.uint32))


def test_nonready_tensor_never_read():
    n = 4
    xs = rank_tensors("f32", 50, n)
    R = {0, 2}
    xs_none = [x if r in R else None for r, x in enumerate(xs)]
    txt = S.allreduce_stars(n, chunk=16)
    a = oc.allreduce(xs, txt, R, "f32")
    b = oc.allreduce(xs_none, txt, R, "f32")
    for u, v in zip(a, b):
        assert np.array_equal(u, v)


@pytest.mark.parametrize("dtype", ["i32", "f32"])
def test_phase1_plus_phase2_equals_full(dtype):
    n = 8
    xs = rank_tensors(dtype, 777, n, dist="int" if dtype == "i32" else "intval")
    R1 = {0, 1, 2, 4, 5, 7}
    R2 = {3, 6}
    txt = S.allreduce_stars(n, chunk=64)
    y1 = oc.allreduce(xs, txt, R1, dtype)
    y2 = oc.allreduce(xs, S.allreduce_ring(n, chunk=48), R2, dtype, accumulate=True, y_prev=y1)
    full = oc.allreduce_exact(xs, set(range(n)), dtype)
    for y in y2:
        assert np.array_equal(y.astype(full.dtype), full)


def test_empty_mask_zero_or_untouched():
    n = 3
    xs = rank_tensors("f32", 21, n)
    txt = S.allreduce_stars(n, chunk=16)
    ys = oc.allreduce(xs, txt, set(), "f32")
    assert all(np.array_equal(y.view(np.uint32), np.zeros(21, np.uint32)) for y in ys)
    prev = [-x for x in xs]   # includes -0.0? no zeros in N(0,1) draws; check untouched
    ys = oc.allreduce(xs, txt, set(), "f32", accumulate=True, y_prev=prev)
    assert all(np.array_equal(a.view(np.uint32), b.view(np.uint32)) for a, b in zip(ys, prev))


def test_accumulate_rounds_once_bf16():
    # prev = 1.0, result = 2^-8 -> 1 + 2^-8 is a tie in bf16 -> even -> 1.0 (0x3f80)
    n = 2
    xs = [np.array([0x3b80], np.uint16), np.array([0x0000], np.uint16)]
    prev = [np.array([0x3f80], np.uint16)] * 2
    ys = oc.allreduce(xs, S.allreduce_stars(n, chunk=16), {0}, "bf16", accumulate=True, y_prev=prev)
    assert [int(y[0]) for y in ys] == [0x3f80, 0x3f80]


# --------------------------------------------------------------- AllGather / AlltoAll
def test_allgather_is_concatenation_and_mask_leaves_slots():
    n, cnt = 5, 13
    xs = rank_tensors("bf16", cnt, n)
    prev = [np.full(n * cnt, 0x1234, np.uint16) for _ in range(n)]
    full = oc.allgather(xs, S.allgather_stars(n, chunk=16), set(range(n)), "bf16", prev)
    cat = np.concatenate(xs)
    assert all(np.array_equal(y, cat) for y in full)
    part = oc.allgather(xs, S.allgather_chains(n, chunk=32), {1, 3}, "bf16", prev)
    for y in part:
        for s in range(n):
            exp = xs[s] if s in (1, 3) else prev[0][s * cnt:(s + 1) * cnt]
            assert np.array_equal(y[s * cnt:(s + 1) * cnt], exp)


def test_alltoall_is_block_transpose_and_involution():
    n, cnt = 4, 9
    xs = rank_tensors("f32", n * cnt, n)
    prev = [np.zeros(n * cnt, np.float32) for _ in range(n)]
    txt = S.alltoall_direct(n, chunk=16, lines=2)
    ys = oc.alltoall(xs, txt, set(range(n)), "f32", prev)
    blocks = np.stack([x.reshape(n, cnt) for x in xs])           # [s][d][cnt]
    for d in range(n):
        assert np.array_equal(ys[d].reshape(n, cnt), blocks[:, d, :])
    back = oc.alltoall(ys, txt, set(range(n)), "f32", prev)
    assert all(np.array_equal(a, b) for a, b in zip(back, xs))
    part = oc.alltoall(xs, txt, {2}, "f32", prev)
    for d in range(n):
        for s in range(n):
            blk = part[d][s * cnt:(s + 1) * cnt]
            assert np.array_equal(blk, xs[2][d * cnt:(d + 1) * cnt] if s == 2 else prev[d][:cnt])


def test_allreduce_elements_equals_full_replay_at_samples():
    n, count = 5, 4099
    xs = rank_tensors("bf16", count, n)
    txt = S.allreduce_trees([S.chain([4, 2, 0, 1, 3]), S.star(n, 1), [1, 2, -1, 1, 2]],
                            weights=[3, 1, 2], chunk=64, noaggs=[(), (), (0,)])
    idx = np.array([0, 1, 7, 8, 1000, 2047, 2048, 3000, 4090, 4098])
    for R in ({0, 1, 2, 3, 4}, {0, 3}, set()):
        full = oc.allreduce(xs, txt, R, "bf16")[0]
        got = oc.allreduce_elements([x[idx] for x in xs], idx, count, txt, R, "bf16")
        assert np.array_equal(full[idx], got)


# ------------------------------------------------------- NEXT-4: Reduce / Broadcast / RS
def test_reduce_equals_allreduce_at_root_and_leaves_others():
    n, count = 5, 301
    xs = rank_tensors("f32", count, n)
    trees = [S.chain([4, 3, 2, 1, 0]), S.star(n, 0), [-1, 0, 1, 1, 2]]
    red = S.header(n, "reduce") + "".join(S.tree_line(p, w, 32) for p, w in zip(trees, [2, 1, 3]))
    allr = S.allreduce_trees(trees, [2, 1, 3], chunk=32)
    prev = [np.full(count, 7.0, np.float32) for _ in range(n)]
    for R in ({0, 1, 2, 3, 4}, {1, 3}, set()):
        ys = oc.reduce(xs, red, R, "f32", y_prev=prev)
        ref = oc.allreduce(xs, allr, R, "f32")[0]
        assert np.array_equal(ys[0].view(np.uint32), ref.view(np.uint32))   # same trees, same order
        assert all(np.array_equal(ys[g], prev[g]) for g in range(1, n))


def test_reduce_int32_brute_force_and_accumulate():
    n, count = 4, 77
    xs = rank_tensors("i32", count, n)
    red = S.header(n, "reduce") + S.tree_line(S.chain([1, 2, 3, 0]), 1, 16) + S.tree_line(S.star(n, 0), 2, 16)
    y1 = oc.reduce(xs, red, {0, 1}, "i32", y_prev=[np.zeros(count, np.int32)] * n)
    y2 = oc.reduce(xs, red, {2, 3}, "i32", accumulate=True, y_prev=y1)
    assert np.array_equal(y2[0], oc.allreduce_exact(xs, set(range(n)), "i32"))


def test_broadcast_copies_root_or_untouched():
    n, count = 4, 33
    xs = rank_tensors("bf16", count, n)
    txt = S.header(n, "broadcast") + "".join(
        f"bcast src=2 weight={w} chunk=16 parent={','.join(map(str, p))}\n"
        for w, p in [(1, S.star(n, 2)), (2, S.chain([0, 1, 3, 2]))])
    prev = [np.full(count, 0x1234, np.uint16) for _ in range(n)]
    assert all(np.array_equal(y, xs[2]) for y in oc.broadcast(xs, txt, {0, 2}, "bf16", prev))
    assert all(np.array_equal(y, p) for y, p in zip(oc.broadcast(xs, txt, {0, 1}, "bf16", prev), prev))


def test_reducescatter_is_block_of_allreduce():
    n, cnt = 4, 50
    xs = rank_tensors("i32", n * cnt, n)
    txt = S.header(n, "reducescatter") + "".join(
        f"rtree dst={b} weight=1 chunk=16 parent={','.join(map(str, S.star(n, b)))}\n" for b in range(n)) \
        + "rtree dst=1 weight=3 chunk=32 parent=1,-1,1,2 noagg=2\n"
    for R in (set(range(n)), {0, 3}):
        ys = oc.reducescatter(xs, txt, R, "i32")
        full = oc.allreduce_exact(xs, R, "i32", n * cnt)
        for b in range(n):
            assert np.array_equal(ys[b], full[b * cnt:(b + 1) * cnt])
    # fp32 order: one star per block rooted at b equals the allreduce star replay of that block
    xf = rank_tensors("f32", n * cnt, n)
    rs = S.header(n, "reducescatter") + "".join(
        f"rtree dst={b} weight=1 chunk=16 parent={','.join(map(str, S.star(n, b)))}\n" for b in range(n))
    ys = oc.reducescatter(xf, rs, set(range(n)), "f32")
    for b in range(n):
        blk = [x[b * cnt:(b + 1) * cnt] for x in xf]
        ref = oc.allreduce(blk, S.allreduce_trees([S.star(n, b)], chunk=16), set(range(n)), "f32")[0]
        assert np.array_equal(ys[b].view(np.uint32), ref.view(np.uint32))


# ------------------------------------------------------------ nvls (NEXT-2)
NVLS = ("adapcc-strategy 1\nnranks {n}\ncollective allreduce\nnvls weight=3 chunk=4096\n"
        "tree weight=1 chunk=4096 parent={star}\n")


def _nvls_text(n):
    return NVLS.format(n=n, star=",".join(["-1"] + ["0"] * (n - 1)))


@pytest.mark.parametrize("n", [2, 3, 5])
def test_nvls_int32_is_the_brute_force_sum(n):
    """An nvls partition is the switch's sum over the ready ranks: int32 adds
    commute exactly, so it equals brute force mod 2^32 for every mask."""
    xs = rank_tensors("i32", 4099, n)
    text = _nvls_text(n)
    for k in range(1, n + 1):
        for R in itertools.combinations(range(n), k):
            got = oc.allreduce(xs, text, set(R), "i32")
            exp = oc.allreduce_exact(xs, set(R), "i32")
            assert all(np.array_equal(g, exp) for g in got)


def test_nvls_float_within_switch_bound_and_integer_exact():
    """fp32 / bf16: within the any-order bound of nvls_tolerance against the
    fp64 definition; integer-valued fp32 (partial sums < 2^24) is exact."""
    n = 8
    text = _nvls_text(n)
    st = ost.parse(text)
    lo, hi = ost.partition(20_000, 4, [s.weight for s in st.subs])[:2]
    for dtype in ("f32", "bf16"):
        xs = rank_tensors(dtype, 20_000, n)
        got = oc.allreduce(xs, text, set(range(n)), dtype)[0]
        ex = oc.allreduce_exact(xs, set(range(n)), dtype)
        vals = [(obf.to_f32(x) if dtype == "bf16" else x).astype(np.float64) for x in xs]
        den = np.sum(np.abs(np.stack(vals)), axis=0)
        g = (obf.to_f32(got) if dtype == "bf16" else got).astype(np.float64)
        err = np.abs(g[lo:hi] - ex[lo:hi]) / den[lo:hi]
        assert err.max() <= oc.nvls_tolerance(dtype, n)
        assert oc.nvls_tolerance(dtype, n) < (1e-6 if dtype == "f32" else 1e-2)
    xi = rank_tensors("f32", 20_000, n, dist="intval")
    got = oc.allreduce(xi, text, set(range(n)), "f32")[0]
    assert np.array_equal(got[lo:hi].astype(np.float64), oc.allreduce_exact(xi, set(range(n)), "f32")[lo:hi])
