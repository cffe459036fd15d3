"""Phase-2 ACCUMULATE AllReduce (partial aggregation): ready = {3, 6}
of 8 virtual ranks, recv += sum, 8 star trees, DIRECT loopback, graph-timed.

Traffic per call = 18 S (2 sources read, 8 recv read + written); roofline =
that traffic / time against MEASURED_PEAKS.json hbm_gbs.  Variants: bulk
reduce-add into recv (acc_red=1) vs shared-memory read-modify-write
(acc_red=0), TMA ring shape 1 x 3 x 64 KiB (shape 1) vs 2 x 3 x 32 KiB (2).

    python scripts/bench_accumulate.py [--sizes 16,25,64,100,256] [--out file.json]
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


def peak():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:  # noqa: BLE001
        return 6650.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="16,25,64,100,256")
    ap.add_argument("--variants", default="red:0,red:1,red:2,rmw:2")
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    n, R2 = 8, {3, 6}
    pk = peak()
    comms = {}
    for v in a.variants.split(","):
        kind, shape = v.split(":")
        os.environ["ADAPCC_TMA_SHAPE"] = shape
        c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
        # (the base kind decides acc_red: "red" and its modified forms red+t4, red@96, rednopdl, ...)
        c.config("acc_red", 1 if kind.startswith("red") else 0)
        if kind == "ldg":
            c.config("engine", 0)
        while "+" in kind:             # red+t4+p128: taper 4, piece_kib 128
            kind, opt = kind.rsplit("+", 1)
            c.config({"t": "taper", "p": "piece_kib"}[opt[0]], int(opt[1:]))
        if "@" in kind:                # red@96: grid capped at 96 CTAs
            kind, cap = kind.split("@")
            c.config("max_ctas", int(cap))
        if kind.endswith("nopdl"):
            c.config("pdl", 0)
            kind = kind[:-5]
        if kind.startswith("flat"):   # flat kernel, optional CTAs per SM: flat6 = 6 per SM
            c.config("engine", 3)
            if kind[4:]:
                c.config("flat_ctas", int(kind[4:]))
        c.set_strategy("allreduce", G.allreduce_stars(n))
        comms[v] = c
    os.environ.pop("ADAPCC_TMA_SHAPE", None)
    rows = []
    for mib in [float(s) for s in a.sizes.split(",")]:
        count = int(mib * (1 << 20)) // 4
        xs = [torch.randn(count, device="cuda") if r in R2 else None for r in range(n)]
        ys = [torch.randn(count, device="cuda") for _ in range(n)]
        row = {"mib_per_rank": mib, "traffic_bytes": 18 * count * 4}
        for v, c in comms.items():
            fn = lambda: c.allreduce_lb(xs, ys, ready=R2, accumulate=True)  # noqa: E731
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            iters = max(5, min(200, int(2e-2 / (18 * count * 4 / (pk * 1e9)))))
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(iters):
                    fn()
            t = []
            for _ in range(a.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                g.replay()
                e1.record()
                torch.cuda.synchronize()
                t.append(e0.elapsed_time(e1) / iters * 1e3)
            us = statistics.median(t)
            row[v] = {"us": round(us, 2), "frac": round(18 * count * 4 / (us * 1e-6) / 1e9 / pk, 4),
                      "engine": c.last_engine()}
            assert c.get_async_error() == 0
            del g
        rows.append(row)
        print(json.dumps(row), flush=True)
    out = {"what": __doc__.strip().splitlines()[0], "peak_gbs": pk, "rows": rows,
           "variants": {"red": "bulk reduce-add (cp.reduce.async.bulk .add) of the folded tile into recv",
                        "rmw": "recv tiles TMA-loaded into the stage, added in shared memory, bulk-stored",
                        "shape 0": "auto", "shape 1": "1 CTA/SM x 3 x 64 KiB", "shape 2": "2 CTAs/SM x 3 x 32 KiB"}}
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
