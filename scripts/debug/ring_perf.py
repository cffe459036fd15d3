import sys, torch
sys.path.insert(0, '.')
import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import generator as G
n = 8
nbytes = 256 << 20
count = nbytes // 4
xs = [torch.randn(count, device="cuda") for _ in range(n)]
ys = [torch.empty_like(x) for x in xs]
def t(comm, iters=10):
    for _ in range(3): comm.allreduce_lb(xs, ys)
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(iters): comm.allreduce_lb(xs, ys)
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / iters
for name, fn in [("ring", lambda c: G.allreduce_ring(n, chunk=c)), ("dbin", lambda c: G.allreduce_double_binary(n, chunk=c)), ("star", lambda c: G.allreduce_stars(n, chunk=c))]:
    for chunk in (256 << 10, 1 << 20, 4 << 20):
        for eng in (0, 1):
            comm = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=1 << 30)
            comm.config("engine", eng)
            text = fn(chunk)
            comm.set_strategy("allreduce", text)
            st = pkg.adapcc.plan_stats(text, count, "f32", (1 << n) - 1, False, "direct", -1, 1 << 30)
            ms = t(comm)
            tr = st["bytes_read"] + st["bytes_written"]
            print(f"{name} chunk {chunk>>10}K eng {eng}: {ms:.3f} ms busbw {nbytes/ms/1e6*1.75:.0f} traffic {tr/2**30:.2f} GiB -> {tr/ms/1e6:.0f} GB/s, levels {st['levels']} segs {st['segments']}")
            comm.finalize()
