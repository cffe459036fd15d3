"""ACCUMULATE (phase 2, ready {3,6} of 8) at 16 / 25 MiB per rank: piece size x
taper x grid sweep, graph-timed, fraction of the HBM roofline on 18 S."""
import itertools
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if __import__("os").path.exists("MEASURED_PEAKS.json") else 6534.1
n, R2 = 8, {3, 6}
for mib in (16, 25):
    count = (mib << 20) // 4
    xs = [torch.randn(count, device="cuda") if r in R2 else None for r in range(n)]
    ys = [torch.randn(count, device="cuda") for _ in range(n)]
    for piece, taper, ctas in itertools.product((0, 128, 256, 1024), (0, 1, 4), (0, 296)):
        c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
        c.config("piece_kib", piece)
        c.config("taper", taper)
        c.config("max_ctas", ctas)
        c.set_strategy("allreduce", G.allreduce_stars(n))
        fn = lambda: c.allreduce_lb(xs, ys, ready=R2, accumulate=True)  # noqa: E731
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
        us = statistics.median(t)
        print(json.dumps({"mib": mib, "piece_kib": piece, "taper": taper, "max_ctas": ctas, "us": round(us, 2),
                          "frac": round(18 * count * 4 / (us * 1e-6) / 1e9 / peak, 4)}), flush=True)
        del g
        c.finalize()
