"""Pins for the late-join oracle (NEXT-1) (-m "not gpu")."""

import itertools

import numpy as np

from oracle import collectives as oc
from synth import rank_tensors
from tests import strategies as S


def _subsets(xs):
    return [set(c) for k in range(len(xs) + 1) for c in itertools.combinations(xs, k)]


def test_phase1_plus_phase2_is_full_sum_for_every_inclusion_int32():
    n, count = 6, 301
    xs = rank_tensors("i32", count, n)
    R = {0, 1, 3, 4}
    for text in (S.allreduce_stars(n, chunk=64), S.allreduce_ring(n, chunk=32),
                 S.allreduce_trees([[1, -1, 1, 2, 2, 0]], chunk=16, noaggs=[(3,)])):
        for L in _subsets([2, 5]):
            y1 = oc.allreduce_late(xs, text, R, "i32", L, phase=1)
            y2 = oc.allreduce_late(xs, text, R, "i32", L, phase=2, y_prev=y1)
            full = oc.allreduce_exact(xs, set(range(n)), "i32")
            assert all(np.array_equal(y, full) for y in y2)
            part = oc.allreduce_exact(xs, R | L, "i32")
            assert all(np.array_equal(y, part) for y in y1)


def test_empty_inclusion_equals_plain_partial_allreduce():
    n, count = 5, 257
    xs = rank_tensors("bf16", count, n)
    text = S.allreduce_trees([S.chain([4, 3, 2, 1, 0]), S.star(n, 2)], [1, 2], chunk=64)
    R = {0, 1, 4}
    a = oc.allreduce_late(xs, text, R, "bf16", set(), phase=1)
    b = oc.allreduce(xs, text, R, "bf16")
    assert all(np.array_equal(u, v) for u, v in zip(a, b))


def test_late_inputs_fold_after_regular_terms_hand_derived():
    # star root 0; ready {0, 1}; rank 2 late and included.  fp32 values chosen so
    # that the order matters (tests/golden/fold_order.txt convention):
    # regular terms [x0, x1] then late x2: (1 + 2^-24) + 2^-23 = 1 + 2^-23
    xs = [np.array([1.0], np.float32), np.array([2 ** -24], np.float32),
          np.array([2 ** -23], np.float32)]
    y = oc.allreduce_late(xs, S.allreduce_trees([S.star(3, 0)], chunk=16), {0, 1}, "f32", {2})
    assert int(y[0].view(np.uint32)[0]) == 0x3F800001


def test_non_kernel_root_with_late_input_is_rounded_once_bf16():
    # root 0 not ready, single flow from 1; late rank 2 joins: fold([x1, x2]) in fp32, one RNE
    xs = [np.array([0x3f80], np.uint16), np.array([0x3f80], np.uint16), np.array([0x3b80], np.uint16)]
    y = oc.allreduce_late(xs, S.allreduce_trees([S.star(3, 0)], chunk=16), {1}, "bf16", {2})
    # 1 + 2^-8 is a tie in bf16 -> even -> 1.0
    assert int(y[0][0]) == 0x3f80


def test_excluded_ranks_are_never_late_int32():
    """members (after a fault exclusion): phase 1 + phase 2 is
    the exact sum over the members only, for every inclusion set, and the
    excluded rank's input (poisoned here) never enters."""
    n, count = 6, 211
    xs = rank_tensors("i32", count, n)
    dead = 4
    xs[dead] = np.full(count, 1 << 20, np.int32)
    members = set(range(n)) - {dead}
    R = {0, 3, 5}
    for text in (S.allreduce_stars(n, chunk=64), S.allreduce_trees([S.star(n, 0)], chunk=32)):
        for L in _subsets([1, 2]):
            y1 = oc.allreduce_late(xs, text, R, "i32", L, phase=1, members=members)
            y2 = oc.allreduce_late(xs, text, R, "i32", L, phase=2, y_prev=y1, members=members)
            want = sum(xs[g].astype(np.int64) for g in members).astype(np.int32)
            assert all(np.array_equal(y, want) for y in y2)
            if L == set():
                y2n = oc.allreduce_late(xs, text, R, "i32", L, phase=2, y_prev=y1)
                assert not np.array_equal(y2n[0], want)     # without members the dead rank would be added
