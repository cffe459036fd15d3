import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import generator as G
n = 2
count = int(sys.argv[1]) if len(sys.argv) > 1 else (9 << 28) // 4 + 3
eng = int(sys.argv[2]) if len(sys.argv) > 2 else 1
torch.manual_seed(0)
xs = [torch.randint(-(1 << 20), 1 << 20, (count,), dtype=torch.int32, device="cuda") for _ in range(n)]
ref = xs[0] + xs[1]
comm = pkg.Communicator.loopback(n, scratch_bytes=64 << 20, mode="direct")
comm.config("engine", eng)
comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=1 << 20))
ys = [torch.full((count,), 7, dtype=torch.int32, device="cuda") for _ in range(n)]
comm.allreduce_lb(xs, ys)
torch.cuda.synchronize()
print("err", comm.get_async_error(), "engine", comm.last_engine())
for g in range(n):
    bad = (ys[g] != ref).nonzero().flatten()
    print("rank", g, "bad", bad.numel())
    if bad.numel():
        b = bad.cpu().numpy()
        print(" first", b[:10], "last", b[-5:], "min", b.min(), "max", b.max())
        i = int(b[0])
        print(" got", int(ys[g][i]), "x0", int(xs[0][i]), "x1", int(xs[1][i]), "ref", int(ref[i]))
        # contiguous runs
        runs = np.split(b, np.where(np.diff(b) != 1)[0] + 1)
        print(" runs", len(runs), [(int(r[0]), len(r)) for r in runs[:8]])
