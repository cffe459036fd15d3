"""G1 k=2 (two 1 GiB inputs -> one output, TMA engine): do the buffers' relative
offsets matter (DRAM channel/bank conflicts between same-offset streams)?
Buffers are carved out of one allocation at offsets i * (S + pad)."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650.0
S = 1 << 30
count = S // 4
k = 2
for pad in (0, 4096, 65536, 3 << 20, 7 * 4096 * 37):
    big = torch.empty((k + 1) * (count + pad // 4), device="cuda")
    bufs = [big[i * (count + pad // 4): i * (count + pad // 4) + count] for i in range(k + 1)]
    for b in bufs[:k]:
        b.normal_()
    comm = pkg.Communicator.loopback(k, mode="direct", scratch_bytes=64 << 20)
    comm.config("engine", 1)
    comm.set_strategy("reduce", G.reduce_trees([G.star_parent(k, 0)], chunk=1 << 20))
    dy = [bufs[k]] + [None] * (k - 1)
    for _ in range(3):
        comm.reduce_lb(bufs[:k], dy, root=0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(10):
        comm.reduce_lb(bufs[:k], dy, root=0)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / 10
    # torch reference kernels on the same buffers: y = x0 + x1 and a plain copy
    a.record()
    for _ in range(10):
        torch.add(bufs[0], bufs[1], out=bufs[k])
    b.record()
    torch.cuda.synchronize()
    ms_t = a.elapsed_time(b) / 10
    print(json.dumps({"pad": pad, "ms": round(ms, 4), "hbm_frac": round(3 * S / ms / 1e6 / peak, 4),
                      "torch_add_ms": round(ms_t, 4), "torch_add_frac": round(3 * S / ms_t / 1e6 / peak, 4)}),
          flush=True)
    comm.finalize()
    del big, bufs
    torch.cuda.empty_cache()
