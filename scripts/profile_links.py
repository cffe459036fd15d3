"""NEXT-2 link profile on the box: graph-captured alpha-beta probes
through adapcc_link_probe, both engines, plus the cost model's chunk choice.

  python scripts/profile_links.py --out gpurun_out/links_r02.json          # 1 GPU (loopback)
  python bench.py-style multi-GPU: torchrun --nproc-per-node N scripts/profile_links.py --out ...
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import costmodel as CM  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--vranks", type=int, default=8)
    a = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1:
        import torch.distributed as dist
        local = int(os.environ.get("LOCAL_RANK", "0"))
        torch.cuda.set_device(local)
        dist.init_process_group("gloo")
        comm = pkg.Communicator.init(scratch_bytes=256 << 20, device=local)
    else:
        comm = pkg.Communicator.loopback(a.vranks, scratch_bytes=256 << 20)
    res = {"where": "loopback (one GPU: every link is the HBM copy path)" if world == 1 else f"{world} GPUs"}
    for engine in ("sm", "ce"):
        p = CM.profile_links(comm, sizes=(1 << 14, 1 << 16, 1 << 20, 1 << 22), repeats=(1, 4, 16), engine=engine)
        p.pop("samples")
        n = p["n"]
        best, scored = CM.chunk_from_profile(p, 256 << 20)
        best25, scored25 = CM.chunk_from_profile(p, 25 << 20)
        p["chunk_model"] = {"strategy": f"{n} star trees", "S256MiB": {"best_chunk": best,
                            "predicted_us": {str(c): round(t * 1e6, 2) for t, c in scored}},
                            "S25MiB": {"best_chunk": best25, "predicted_us": {str(c): round(t * 1e6, 2) for t, c in scored25}}}
        p["per_gpu_bw_GBps"] = CM.per_gpu_bandwidth(p)
        w, _, load = G.mask_aware_star_weights(n, set(range(n)) - {3, 6} if n == 8 else set(range(n - 1)),
                                               bw=p["per_gpu_bw_GBps"])
        p["mask_aware_weights_from_profile"] = {"weights": w, "max_load_over_S": load}
        res[engine] = p
        print(json.dumps({engine: {"alpha_us_0_1": p["alpha_us"][0][1], "GBps_0_1": p["beta_GBps"][0][1],
                                   "fanout": p["fanout"], "best_chunk_256MiB": best}}), flush=True)
    comm.config("default_chunk", res["sm"]["chunk_model"]["S256MiB"]["best_chunk"])
    if a.out and (world == 1 or int(os.environ.get("RANK", "0")) == 0):
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)
    comm.finalize()


if __name__ == "__main__":
    main()
