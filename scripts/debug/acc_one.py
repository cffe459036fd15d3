"""A few ACCUMULATE AllReduce calls (phase 2: ready {3, 6}, 8 virtual ranks) for ncu.

    python scripts/debug/acc_one.py [MiB per rank, default 16] [acc_red 0|1, default 1]"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

mib = float(sys.argv[1]) if len(sys.argv) > 1 else 16
n, R2, count = 8, {3, 6}, int(mib * (1 << 20)) // 4
c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
c.config("acc_red", int(sys.argv[2]) if len(sys.argv) > 2 else 1)
c.set_strategy("allreduce", G.allreduce_stars(n))
xs = [torch.randn(count, device="cuda") for _ in range(n)]
ys = [torch.randn(count, device="cuda") for _ in range(n)]
for _ in range(4):
    c.allreduce_lb([x if r in R2 else None for r, x in enumerate(xs)], ys, ready=R2, accumulate=True)
torch.cuda.synchronize()
print("engine", c.last_engine())
