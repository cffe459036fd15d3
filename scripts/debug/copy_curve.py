"""Practical HBM roofline vs size: graph-timed device-to-device copies
(torch copy_ kernel and cudaMemcpyAsync D2D) whose read + write traffic equals
the engine's algorithmic traffic at each AllReduce size (8 virtual ranks:
2 x 8 x S bytes).  Same buffers every replay (like scripts/sweep_sizes.py)."""
import json
import statistics
import sys

import torch

REPS = 5


def graph_us(fn, iters):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(iters):
            fn()
    g.replay()
    torch.cuda.synchronize()
    t = []
    for _ in range(REPS):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        t.append(a.elapsed_time(b) / iters * 1e3)
    return round(statistics.median(t), 3)


out = []
for lg in range(16, 29):
    per_rank = 1 << lg
    copy_bytes = 8 * per_rank  # read 8S + write 8S = the DIRECT AllReduce traffic at n = 8
    src = torch.empty(copy_bytes // 4, device="cuda")
    dst = torch.empty_like(src)
    iters = int(min(400, max(10, 2e4 / (copy_bytes / 6.5e9 * 1e6 + 3))))
    us_k = graph_us(lambda: dst.copy_(src), iters)
    row = {"bytes_per_rank": per_rank, "traffic": 2 * copy_bytes, "copy_kernel_us": us_k,
           "copy_kernel_gbs": round(2 * copy_bytes / us_k / 1e3, 1)}
    print(json.dumps(row), flush=True)
    out.append(row)
    del src, dst
    torch.cuda.empty_cache()
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1)
