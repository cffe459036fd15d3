"""LDG vs TMA engine crossover for AllReduce / AllGather / AlltoAll (8 virtual ranks, DIRECT), graph-timed."""
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

n = 8


def gtime(fn, iters=30):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(iters):
            fn()
    t = []
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        t.append(a.elapsed_time(b) / iters * 1e3)
    return round(statistics.median(t), 2)


for mode in ("direct", "staged"):
    comms = {}
    for e in (0, 1):
        c = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=512 << 20)
        c.config("engine", e)
        comms[e] = c
    for mib in (1, 2, 4, 8, 16):
        count = (mib << 20) // 4
        xs = [torch.randn(count, device="cuda") for _ in range(n)]
        ys = [torch.empty_like(x) for x in xs]
        row = {"mode": mode, "mib_per_rank": mib}
        for e, c in comms.items():
            row[f"allreduce_e{e}"] = gtime(lambda: c.allreduce_lb(xs, ys))
            yg = [torch.empty(n * (count // n), device="cuda") for _ in range(n)]
            row[f"allgather_e{e}"] = gtime(lambda: c.allgather_lb([x[:count // n] for x in xs], yg))
            row[f"alltoall_e{e}"] = gtime(lambda: c.alltoall_lb(xs, ys))
        print(json.dumps(row), flush=True)
