"""ACCUMULATE (phase 2, ready {3,6} of 8) at small sizes: LDG vs TMA (bulk reduce-add), graph-timed."""
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
for kib in (64, 256, 1024, 2048, 4096, 8192):
    count = kib * 256
    xs = [torch.randn(count, device="cuda") if r in R2 else None for r in range(n)]
    ys = [torch.randn(count, device="cuda") for _ in range(n)]
    row = {"kib_per_rank": kib}
    for e, c in comms.items():
        fn = lambda: c.allreduce_lb(xs, ys, ready=R2, accumulate=True)  # noqa: E731
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(50):
                fn()
        t = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            t.append(a.elapsed_time(b) / 50 * 1e3)
        row[f"engine{e}_us"] = round(statistics.median(t), 2)
        del g
    print(json.dumps(row), flush=True)
