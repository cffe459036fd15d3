"""Small-call floor: graph-timed back-to-back launches of (a) a 1-element torch
add (the device's kernel-to-kernel floor) and (b) a 1 KiB-per-rank AllReduce
of the engine at n = 1, 2, 8 virtual ranks, both kernels."""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

REPS = 200


def graph_us(fn):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(REPS):
                fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = 1e9
    for _ in range(5):
        g.replay()
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / REPS * 1e3)
    return round(best, 3)


out = {}
x = torch.zeros(1, device="cuda")
out["torch_add_1elem"] = graph_us(lambda: x.add_(1))
for n in (1, 2, 8):
    for eng in (0, 1):
        comm = pkg.Communicator.loopback(n, mode="direct")
        comm.config("engine", eng)
        comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=262144))
        xs = [torch.randn(256, device="cuda") for _ in range(n)]
        ys = [torch.empty_like(t) for t in xs]
        out[f"allreduce_1KiB_n{n}_engine{eng}"] = graph_us(lambda: comm.allreduce_lb(xs, ys))
        assert comm.get_async_error() == 0
        comm.finalize()
print(json.dumps(out))
