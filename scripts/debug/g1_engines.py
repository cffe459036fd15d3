"""G1 local reduction (k virtual 1 GiB inputs -> one output) per engine and k:
HBM fraction of (k+1) S / t against the measured copy peak."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650.0
nbytes = int(sys.argv[1]) << 20 if len(sys.argv) > 1 else 1 << 30
ks = [int(v) for v in sys.argv[2].split(",")] if len(sys.argv) > 2 else [2, 3, 4, 8]
count = nbytes // 4
xs = [torch.randn(count, device="cuda") for _ in range(max(ks))]
y = torch.empty(count, device="cuda")
out = []
for k in ks:
    for eng in (0, 1):
        comm = pkg.Communicator.loopback(k, mode="direct", scratch_bytes=64 << 20)
        comm.config("engine", eng)
        comm.set_strategy("reduce", G.reduce_trees([G.star_parent(k, 0)], chunk=1 << 20))
        dy = [y] + [None] * (k - 1)
        for _ in range(3):
            comm.reduce_lb(xs[:k], dy, root=0)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(10):
            comm.reduce_lb(xs[:k], dy, root=0)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 10
        out.append({"k": k, "engine": eng, "ms": round(ms, 4),
                    "hbm_frac": round((k + 1) * nbytes / ms / 1e6 / peak, 4)})
        print(json.dumps(out[-1]), flush=True)
        comm.finalize()
