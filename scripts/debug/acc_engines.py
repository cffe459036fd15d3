"""ACCUMULATE AllReduce (phase 2 of partial aggregation: ready = {3, 6}, recv += sum)
on the LDG vs the TMA kernel at 8 virtual ranks, graph-timed, per size."""
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

n, R2 = 8, {3, 6}
comms = {}
for e in (0, 1):
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.config("engine", e)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    comms[e] = c
for lg in range(16, 26):
    count = (1 << lg) // 4
    xs = [torch.randn(count, device="cuda") for _ in range(n)]
    ys = [torch.randn(count, device="cuda") for _ in range(n)]
    row = {"bytes_per_rank": 1 << lg}
    for e, c in comms.items():
        fn = lambda: c.allreduce_lb([x if r in R2 else None for r, x in enumerate(xs)], ys, ready=R2, accumulate=True)  # noqa
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(20):
                fn()
        t = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            t.append(a.elapsed_time(b) / 20 * 1e3)
        row[f"engine{e}_us"] = round(statistics.median(t), 2)
    print(json.dumps(row), flush=True)
