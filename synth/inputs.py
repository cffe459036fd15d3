"""Seeded input generators (no method arithmetic; see synth/__init__.py).

Distributions:
  'normal'  fp32 N(0,1)                                seed = base + rank
  'intval'  fp32 holding integers U[-2^20, 2^20)       (every partial sum of
            <= 8 such values is exact in fp32: |sum| < 2^23 < 2^24)
  'int'     int32 U[-2^20, 2^20)                       (reading Q15)
  bf16      the top 16 bits of an fp32 N(0,1) draw (truncation: a bit
            operation that only defines the input distribution).
No NaN, Inf or subnormal values are produced (reading Q16).
"""

import numpy as np

# Workload shapes (BASELINE.json configs)
GPT2XL_LAYERS = [  # (name, rows, cols) of one GPT-2-XL block's weights, d=1600
    ("attn.c_attn", 1600, 4800),
    ("attn.c_proj", 1600, 1600),
    ("mlp.c_fc", 1600, 6400),
    ("mlp.c_proj", 6400, 1600),
]

CONFIGS = {
    # C1: AllReduce fp32 1M elements, 2 ranks, single tree, chunk 256 KB
    "C1": dict(coll="allreduce", n=2, dtype="f32", count=1 << 20, chunk=262144),
    # C2: AllReduce fp32/bf16 size sweep, 8 ranks, multi-tree; bench point 256 MiB
    #     (the paper's "float data of 256 MB")
    "C2": dict(coll="allreduce", n=8, dtype="f32", count=(256 << 20) // 4, chunk=1 << 20),
    # C3: partial AllReduce 8 ranks, stragglers {3,6}, 25/50/100 MiB buckets
    "C3": dict(coll="allreduce", n=8, dtype="f32", sizes_mib=(25, 50, 100),
               stragglers=(3, 6)),
    # C4: AlltoAll MoE dispatch, 8 ranks, [8][512 tokens][4096] bf16 per rank
    "C4": dict(coll="alltoall", n=8, dtype="bf16", count_per_peer=512 * 4096),
    # C5: AllGather of GPT-2-XL shards at 2/4/8 ranks, 48 layers x 4 weights
    "C5": dict(coll="allgather", ns=(2, 4, 8), dtype="bf16", layers=48),
}


def _rng(seed):
    return np.random.Generator(np.random.PCG64(seed))


def bf16_bits_from_normal(count, seed):
    """bf16 bit patterns: top half of fp32 N(0,1) draws (never NaN/Inf)."""
    x = _rng(seed).standard_normal(count, dtype=np.float32)
    return (x.view(np.uint32) >> np.uint32(16)).astype(np.uint16)


def rank_tensor(dtype, count, rank, dist="normal", base=1000):
    """One rank's send tensor.  dtype in {'f32','bf16','i32'}."""
    seed = base + rank
    if dtype == "i32" or dist == "int":
        v = _rng(seed + 100).integers(-(1 << 20), 1 << 20, size=count, dtype=np.int64)
        return v.astype(np.int32)
    if dtype == "bf16":
        return bf16_bits_from_normal(count, seed)
    if dist == "intval":
        v = _rng(seed + 200).integers(-(1 << 20), 1 << 20, size=count, dtype=np.int64)
        return v.astype(np.float32)
    if dist == "normal":
        return _rng(seed).standard_normal(count, dtype=np.float32)
    raise ValueError(dist)


def rank_tensors(dtype, count, n, dist="normal", base=1000):
    return [rank_tensor(dtype, count, r, dist, base) for r in range(n)]


def ready_set_from_mask(mask, n):
    return {r for r in range(n) if (mask >> r) & 1}


def mask_from_set(ready):
    m = 0
    for r in ready:
        m |= 1 << r
    return m


def moe_counts(n, tokens_per_rank, hidden, zipf_a=1.2, seed=2100):
    """Skewed top-1 MoE routing (NEXT-4, P:L309 MoE workload): every rank routes
    `tokens_per_rank` tokens to n experts (one per rank) with Zipf(a) expert
    popularity (a global random popularity order); returns counts[s][d] in
    ELEMENTS (tokens x hidden).  a = 0 gives uniform routing."""
    rng = _rng(seed)
    order = rng.permutation(n)
    p = 1.0 / (np.arange(1, n + 1) ** zipf_a)
    p = p / p.sum()
    probs = np.empty(n)
    probs[order] = p
    counts = []
    for s in range(n):
        tok = rng.multinomial(tokens_per_rank, probs)
        counts.append([int(t) * hidden for t in tok])
    return counts
