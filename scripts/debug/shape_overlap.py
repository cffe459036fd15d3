"""TMA ring shapes for back-to-back DIRECT AllReduce (8 virtual ranks, fp32, graph-timed):
shape 1 (1 CTA/SM x 3 x 64 KiB, 166 regs) vs shape 2 (3 x 32 KiB, 96 regs) at grid 296 (2/SM)
and at grid 148 (1/SM: the next launch's CTAs can be resident while this one drains)."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

n = 8
variants = {"s1": (1, 0), "s2g296": (2, 0), "s2g148": (2, 148)}
comms = {}
for name, (shape, ctas) in variants.items():
    os.environ["ADAPCC_TMA_SHAPE"] = str(shape)
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.config("engine", 1)
    if ctas:
        c.config("max_ctas", ctas)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    comms[name] = c
peak = 6534.1
for mib in (4, 8, 16, 64, 256):
    count = (mib << 20) // 4
    xs = [torch.randn(count, device="cuda") for _ in range(n)]
    ys = [torch.empty_like(x) for x in xs]
    row = {"mib": mib}
    for name, c in comms.items():
        fn = lambda: c.allreduce_lb(xs, ys)  # noqa: E731
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        iters = 20 if mib < 64 else 5
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(iters):
                fn()
        t = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            t.append(a.elapsed_time(b) / iters * 1e3)
        us = statistics.median(t)
        row[name] = {"us": round(us, 2), "hbm_frac": round(2 * n * count * 4 / (us * 1e-6) / 1e9 / peak, 4)}
        del g
    print(json.dumps(row), flush=True)
