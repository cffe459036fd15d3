"""relay=store vs bypass A/B on one B200, 8 virtual ranks, graph-timed:
AllReduce with relays in the middle of deep trees (chains / double binary),
masks with 2 and 4 non-ready ranks, both transport plans.

    python scripts/bench_relay.py --out gpurun_out/relay_ab_r02.json
"""
import argparse
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402


def graph_us(fn, iters=20, reps=5):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(iters):
            fn()
    t = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        t.append(a.elapsed_time(b) / iters * 1e3)
    return statistics.median(t)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--sizes", default="4,64")
    a = ap.parse_args()
    n = 8
    order = [0, 1, 2, 3, 4, 5, 6, 7]
    strategies = {"chains8": lambda r: G.allreduce_trees([G.chain_parent(order[m:] + order[:m]) for m in range(n)],
                                                         chunk=262144, relay=r),
                  "double_binary": lambda r: G.allreduce_trees([G.binary_tree_parent(order),
                                                                G.binary_tree_parent(order[::-1])], chunk=262144,
                                                               relay=r)}
    rows = []
    for mode in ("staged", "direct"):
        for name, mk in strategies.items():
            for mib in [int(s) for s in a.sizes.split(",")]:
                count = (mib << 20) // 4
                xs = [torch.randn(count, device="cuda") for _ in range(n)]
                ys = [torch.empty_like(x) for x in xs]
                for mask_name, R in (("2 relays", {0, 1, 2, 3, 5, 6}), ("4 relays", {0, 2, 4, 6})):
                    row = {"mode": mode, "strategy": name, "mib_per_rank": mib, "mask": mask_name}
                    for relay in ("bypass", "store"):
                        text = mk(relay)
                        comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=(4 * (mib << 20) + (64 << 20))
                                                         if mode == "staged" else 64 << 20)
                        comm.set_strategy("allreduce", text)
                        row[relay + "_us"] = round(graph_us(lambda: comm.allreduce_lb(
                            [x if r in R else None for r, x in enumerate(xs)], ys, ready=R)), 2)
                        assert comm.get_async_error() == 0
                        comm.finalize()
                    row["store_over_bypass"] = round(row["store_us"] / row["bypass_us"], 3)
                    rows.append(row)
                    print(json.dumps(row), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"what": "relay=store vs bypass, 8 virtual ranks, graph-timed", "rows": rows}, f, indent=1)


if __name__ == "__main__":
    main()
