"""One G1 k-input Reduce (1 GiB per input) for ncu: warm-up calls, then one call."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

k = int(sys.argv[1]) if len(sys.argv) > 1 else 2
eng = int(sys.argv[2]) if len(sys.argv) > 2 else 1
count = (1 << 30) // 4
xs = [torch.randn(count, device="cuda") for _ in range(k)]
y = torch.empty(count, device="cuda")
comm = pkg.Communicator.loopback(k, mode="direct", scratch_bytes=64 << 20)
comm.config("engine", eng)
comm.set_strategy("reduce", G.reduce_trees([G.star_parent(k, 0)], chunk=1 << 20))
for _ in range(4):
    comm.reduce_lb(xs, [y] + [None] * (k - 1), root=0)
torch.add(xs[0], xs[1], out=y)
torch.cuda.synchronize()
