"""ACCUMULATE (ready {3,6} of 8, 16 MiB per rank) eager vs graph, grid capped or not:
    python scripts/debug/acc_cap_eager.py <max_ctas or 0>"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

cap = int(sys.argv[1]) if len(sys.argv) > 1 else 0
n, R2, count = 8, {3, 6}, (16 << 20) // 4
c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
if cap:
    c.config("max_ctas", cap)
c.set_strategy("allreduce", G.allreduce_stars(n))
xs = [torch.randn(count, device="cuda") if r in R2 else None for r in range(n)]
ys = [torch.randn(count, device="cuda") for _ in range(n)]
fn = lambda: c.allreduce_lb(xs, ys, ready=R2, accumulate=True)  # noqa: E731
for _ in range(5):
    fn()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(100):
    fn()
b.record()
torch.cuda.synchronize()
eager = a.elapsed_time(b) / 100 * 1e3
s = torch.cuda.Stream()
s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(100):
            fn()
torch.cuda.synchronize()
g.replay()
torch.cuda.synchronize()
a.record()
g.replay()
b.record()
torch.cuda.synchronize()
print(f"cap={cap} eager_us={eager:.2f} graph_us={a.elapsed_time(b) / 100 * 1e3:.2f}")
