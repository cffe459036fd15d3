"""Host logic of the plan compiler's work items (CPU, no GPU): the pieces the
engine executes tile every task chunk exactly, flagged chunks stay whole,
pieces are 16-byte aligned, mid-size flag-free calls give every CTA at most m
items (the balanced-piece rule, DESIGN.md §6 "Pieces"), and the claim order is
topological (an item never precedes a lower-level item of the same chunk,
DESIGN.md §6 "Work items and deadlock freedom").  Read through the C ABI's
host-only adapcc_plan_items."""
import math

import numpy as np
import pytest

import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import generator as G

ALIGN = 512  # elements (plan.cpp: keeps every piece 16-byte aligned for every dtype)


def _check_tiling(items, tasks):
    cover = {}
    for it in items:
        cover.setdefault((int(it["task"]), int(it["chunk"])), []).append((int(it["off"]), int(it["len"])))
    for t_idx, t in enumerate(tasks):
        for c in range(int(t["nchunks"])):
            c0 = int(t["lo"]) + c * int(t["chunk_elems"])
            clen = min(int(t["hi"]), c0 + int(t["chunk_elems"])) - c0
            pieces = sorted(cover.pop((t_idx, c), []))
            assert pieces, (t_idx, c)
            pos = 0
            for off, ln in pieces:
                assert off == pos and ln > 0
                assert off % ALIGN == 0
                pos += ln
            assert pos == clen, (t_idx, c, pos, clen)
            if t["npost"]:
                assert len(pieces) == 1  # a posted flag means "the whole chunk is written"
    assert not cover  # no item outside a task chunk


def _check_order(items, tasks):
    """Every item of level L on chunk c comes after every item of level < L on
    chunk c (waits target posts of lower levels on the same chunk index)."""
    last_pos = {}
    for pos, it in enumerate(items):
        t = tasks[int(it["task"])]
        last_pos[(int(it["chunk"]), int(t["level"]))] = pos
    for pos, it in enumerate(items):
        t = tasks[int(it["task"])]
        if t["nwait"] == 0:
            continue
        for lv in range(int(t["level"])):
            if (int(it["chunk"]), lv) in last_pos:
                assert last_pos[(int(it["chunk"]), lv)] < pos


STRATS = {
    "stars8": lambda: G.allreduce_stars(8),
    "dbinary8": lambda: G.allreduce_double_binary(8),
    "ring4": lambda: G.allreduce_ring(4),
    "chain_noagg": lambda: G.allreduce_trees([[1, 2, 3, -1]], chunk=65536, noaggs=[[1]]),
    "a2a8": lambda: G.alltoall_direct(8),
    "ag8": lambda: G.allgather_stars(8),
}


@pytest.mark.parametrize("name", sorted(STRATS))
@pytest.mark.parametrize("mode", ["direct", "staged"])
@pytest.mark.parametrize("count", [1, 4099, (1 << 20) + 12, 3 << 22])
@pytest.mark.parametrize("tma,grid", [(False, 296), (True, 148), (False, 7)])
@pytest.mark.parametrize("partial", [False, True])
def test_items_tile_tasks_in_topological_order(name, mode, count, tma, grid, partial):
    text = STRATS[name]()
    n = pkg.strategy_check(text)[0]
    mask = (1 << n) - 1
    if partial:  # ranks 1 and 3 relay
        mask &= ~0b1010
    items, tasks = pkg.plan_items(text, count, "f32", mask, grid, tma=tma, mode=mode, scratch_bytes=1 << 30)
    _check_tiling(items, tasks)
    _check_order(items, tasks)


@pytest.mark.parametrize("per_rank_mib", [1, 2, 4, 8, 16, 64])
@pytest.mark.parametrize("tma,grid", [(False, 296), (True, 148)])
def test_balanced_pieces_items_per_cta(per_rank_mib, tma, grid):
    """Flag-free star AllReduce: at most m items per CTA, m = ceil(traffic / (grid x 512 KiB)) (before
    the taper, which only applies from m >= 3)."""
    count = per_rank_mib << 18  # fp32 elements
    items, tasks = pkg.plan_items(G.allreduce_stars(8), count, "f32", 255, grid, tma=tma, taper=1)
    traffic = sum(int(t["hi"] - t["lo"]) * 4 * (int(t["nsrc"]) + int(t["ndst"])) for t in tasks)
    m = max(1, math.ceil(traffic / (grid * 512 * 1024)))
    assert len(items) <= m * grid
    _check_tiling(items, tasks)


def test_measured_mid_size_case():
    """8 virtual ranks x 4 MiB fp32 on 296 LDG CTAs -> 256 items of 4096 elements
    (16 KiB per stream), not 304 ragged ones."""
    items, _ = pkg.plan_items(G.allreduce_stars(8), 1 << 20, "f32", 255, 296)
    assert len(items) == 256
    assert set(int(x) for x in items["len"]) == {4096}


def test_auto_taper_only_from_three_items_per_cta():
    text = G.allreduce_stars(8)
    # 8 MiB per rank on the TMA grid: m = 2 -> automatic taper off (no extra items)
    auto, _ = pkg.plan_items(text, 2 << 20, "f32", 255, 148, tma=True, taper=0)
    off, _ = pkg.plan_items(text, 2 << 20, "f32", 255, 148, tma=True, taper=1)
    assert len(auto) == len(off)
    # 64 MiB per rank: m >= 3 -> the last ~2 x grid items are halved
    auto, tasks = pkg.plan_items(text, 16 << 20, "f32", 255, 148, tma=True, taper=0)
    off, _ = pkg.plan_items(text, 16 << 20, "f32", 255, 148, tma=True, taper=1)
    assert len(off) < len(auto) <= len(off) + 2 * 148
    _check_tiling(auto, tasks)


def test_plan_items_rejects_bad_arguments():
    text = G.allreduce_stars(4)
    with pytest.raises(pkg.AdapccError):
        pkg.plan_items(text, 1024, "f32", 15, 0)           # grid < 1
    with pytest.raises(pkg.AdapccError):
        pkg.plan_items(text, 1024, "f32", 15, 8, segment=5)  # no such segment
    with pytest.raises(pkg.AdapccError):
        pkg.plan_items(text, 1024, "f32", 1 << 5, 8)       # mask names rank 5 of 4


@pytest.mark.parametrize("name", ["stars8", "dbinary8", "ring4"])
@pytest.mark.parametrize("rank", [-1, 0, 3])
def test_staged_late_join_plan(name, rank):
    """STAGED late join (NEXT-1): per tree, every non-ready rank owns
    one conditional push task (no waits, one post per chunk) whose range is the
    tree's; the root task waits for them in addition to its regular sources;
    items still tile every chunk and keep a topological claim order."""
    text = STRATS[name]()
    n, _, nsubs = pkg.strategy_check(text)
    late = {3, n - 2}
    mask = sum(1 << g for g in range(n) if g not in late)
    count = 100_003
    items, tasks = pkg.adapcc.plan_items(text, count, "f32", mask, 64, mode="staged", rank=rank, late="join")
    if rank == -1:
        _check_tiling(items, tasks)
    _check_order(items, tasks)
    _, plain = pkg.adapcc.plan_items(text, count, "f32", mask, 64, mode="staged", rank=rank)
    # every tree range gets exactly one push per late rank that is not its root
    ranges = {}
    for t in plain:
        ranges.setdefault((int(t["lo"]), int(t["hi"])), []).append(t)
    extra = len(tasks) - len(plain)
    if rank == -1:
        roots = []
        for m in range(nsubs):
            _, _, parent, _ = pkg.strategy_sub(text, m)
            roots.append(parent.index(-1))
        assert extra == sum(len(late - {r}) for r in roots)
        pushes = [t for t in tasks if int(t["owner"]) in late and int(t["nwait"]) == 0 and int(t["npost"]) == 1
                  and int(t["nsrc"]) == 1]
        assert len(pushes) >= extra
    else:   # (tasks are listed for every rank; items only for `rank`)
        mine = {int(it["task"]) for it in items}
        assert all(int(tasks[i]["owner"]) == rank for i in mine)
        assert any(int(tasks[i]["owner"]) in late and int(tasks[i]["nsrc"]) == 1 and int(tasks[i]["nwait"]) == 0
                   for i in range(len(tasks)))
