"""C++ strategy loader / tuple derivation / partition / planner vs the oracle (-m "not gpu").

The two sides are independent implementations of DESIGN.md §2-§3 (they share
no code); these tests call libadapcc.so's host-only entry points, which need
no GPU.
"""

import itertools
import os
import re

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from oracle import strategy as ost
from oracle import tuples as otu
from tests import strategies as S
from tests.test_oracle_pins import BAD

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "adapcc.h")).read()
    declared = set(re.findall(r"ADAPCC_API\s+[\w\s\*]+?\b(adapcc_\w+)\s*\(", hdr))
    assert len(declared) >= 19
    lib = A._load()
    for name in sorted(declared):
        assert hasattr(lib, name), name
    # and nothing else leaks out of the library
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", A.lib_path()], capture_output=True,
                         text=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    assert {s for s in exported if s.startswith("adapcc_")} == declared


@pytest.mark.parametrize("text", BAD)
def test_loader_rejects_what_the_oracle_rejects(text):
    with pytest.raises(A.AdapccError) as e:
        pkg.strategy_check(text)
    assert e.value.code == A.INVALID_STRATEGY


GOOD = [
    S.allreduce_stars(8),
    S.allreduce_ring(5, chunk=48, weight=7),
    S.allreduce_ring(4, chunk=64) + S.tree_line(S.star(4, 2), 3, 32, noagg=(0, 1)),
    S.allreduce_trees([S.chain([3, 1, 0, 2]), [1, 2, -1, 1]], [2, 5], 1024, [(), (1,)]),
    S.allgather_stars(6, chunk=32),
    S.allgather_chains(3),
    S.alltoall_direct(8, lines=3),
    "# c\nadapcc-strategy 1\nnranks 1\ncollective allreduce\ntree weight=1 chunk=16 parent=-1\n",
]


@pytest.mark.parametrize("text", GOOD)
def test_loader_matches_oracle_subs(text):
    st = ost.parse(text)
    n, coll, nsubs = pkg.strategy_check(text)
    assert n == st.nranks and nsubs == len(st.subs)
    assert coll == {"allreduce": 0, "allgather": 1, "alltoall": 2}[st.collective]
    for m, sub in enumerate(st.subs):
        w, c, par, src = pkg.strategy_sub(text, m)
        assert (w, c, src) == (sub.weight, sub.chunk, sub.src)
        if sub.parent is not None:
            assert par == sub.parent


def test_tuples_match_oracle_every_small_tree_mask_noagg():
    for n in (2, 3, 4):
        for parent in S.all_rooted_trees(n):
            nonroot = [g for g in range(n) if parent[g] != -1]
            for k in range(len(nonroot) + 1):
                for na in itertools.combinations(nonroot, k):
                    text = S.allreduce_trees([parent], chunk=16, noaggs=[na])
                    for mask in range(1 << n):
                        R = {r for r in range(n) if mask >> r & 1}
                        tup, fl = otu.behavior(parent, R, frozenset(na))
                        ctup, cfl = pkg.strategy_tuples(text, 0, mask)
                        assert ctup == [tup[g] for g in range(n)], (parent, na, mask)
                        assert cfl == [len(fl[g]) for g in range(n)], (parent, na, mask)


def test_tuples_match_oracle_random_large():
    rng = np.random.default_rng(3)
    for _ in range(200):
        n = int(rng.integers(5, 65))
        parent = [-1] + [int(rng.integers(0, g)) for g in range(1, n)]
        perm = rng.permutation(n)
        p2 = [None] * n
        for g in range(n):
            p2[perm[g]] = -1 if parent[g] == -1 else int(perm[parent[g]])
        na = [g for g in range(n) if p2[g] != -1 and rng.random() < 0.2]
        mask = int(rng.integers(0, 1 << 62)) & ((1 << n) - 1)
        text = S.allreduce_trees([p2], chunk=16, noaggs=[na])
        tup, fl = otu.behavior(p2, {r for r in range(n) if mask >> r & 1}, frozenset(na))
        ctup, cfl = pkg.strategy_tuples(text, 0, mask)
        assert ctup == [tup[g] for g in range(n)]
        assert cfl == [len(fl[g]) for g in range(n)]


def test_partition_matches_oracle():
    rng = np.random.default_rng(4)
    for _ in range(300):
        m = int(rng.integers(1, 9))
        n = 4
        w = [int(v) for v in rng.integers(0, 1 << 20, size=m)]
        w[0] += 1
        text = S.allreduce_trees([S.star(n, i % n) for i in range(m)], w, 64)
        for dtype, es in (("f32", 4), ("bf16", 2), ("i32", 4)):
            count = int(rng.integers(0, 1 << 34))
            assert pkg.strategy_partition(text, count, dtype) == ost.partition(
                count, es, [s.weight for s in ost.parse(text).subs])


def test_allgather_partition_per_source():
    text = S.header(3, "allgather") + "".join(
        f"bcast src={s} weight={w} chunk=32 parent={','.join(map(str, S.star(3, s)))}\n"
        for s, w in [(0, 1), (1, 2), (0, 3), (2, 1), (1, 1)])
    st = ost.parse(text)
    for s in range(3):
        ws = [sub.weight for sub in st.subs if sub.src == s]
        assert pkg.strategy_partition(text, 1001, "bf16", src=s) == ost.partition(1001, 2, ws)


def test_plan_stats_direct_star_moves_minimal_bytes():
    n, count = 8, 1 << 20
    st = pkg.plan_stats(S.allreduce_stars(n), count, "f32", (1 << n) - 1, mode="direct")
    # every input read once, every output written once: 2 n S
    assert st["bytes_read"] == n * count * 4
    assert st["bytes_written"] == n * count * 4
    assert st["levels"] == 1


def test_plan_stats_staged_star_traffic_model():
    n, count = 8, 1 << 20
    S_ = count * 4
    full = (1 << n) - 1
    per_rank = [pkg.plan_stats(S.allreduce_stars(n), count, "f32", full, mode="staged", rank=r)
                for r in range(n)]
    for st in per_rank:
        # remote bytes issued by one rank: pushes (its NVLink egress) + pulls (its
        # ingress), each (n-1)/n * S; with the peers' symmetric traffic every GPU
        # moves 2(n-1)/n * S per direction -- the AllReduce bound (SURVEY d-3)
        assert st["remote_bytes"] == 2 * (n - 1) * S_ // n
        assert st["levels"] == 3


def test_plan_segments_when_arena_small():
    n, count = 4, 1 << 20
    st = pkg.plan_stats(S.allreduce_stars(n), count, "f32", 0xF, mode="staged", rank=-1,
                        scratch_bytes=1 << 20)
    assert st["segments"] > 1
    assert st["arena_bytes"] <= ((1 << 20) - 4096) // 2
