"""Interleaved A/B of engine configs on one GPU (graph-timed, median of reps).

    python scripts/debug/ab_configs.py --coll allreduce --sizes 20,21,22,23 \
        --configs 'sched=0;sched=1;piece_kib=512' [--reps 5] [--out f.json]

Each config is a ';'-separated list of key=value[,key=value] adapcc_config
settings applied to its own loopback communicator (8 virtual ranks, fp32)."""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--coll", default="allreduce")
    ap.add_argument("--sizes", default="20,21,22,23")
    ap.add_argument("--configs", required=True)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--mode", default="direct")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G

    n = a.ranks
    cfgs = []
    for c in a.configs.split(";"):
        kv = dict(x.split("=") for x in c.split(",") if x)
        cfgs.append((c, {k: int(v) for k, v in kv.items()}))
    comms = []
    for name, kv in cfgs:
        cm = pkg.Communicator.loopback(n, scratch_bytes=1 << 30, mode=a.mode)
        for k, v in kv.items():
            cm.config(k, v)
        text = {"allreduce": G.allreduce_stars(n), "allgather": G.allgather_stars(n),
                "alltoall": G.alltoall_direct(n)}[a.coll]
        cm.set_strategy(a.coll, text)
        comms.append(cm)
    out = []
    for lg in [int(s) for s in a.sizes.split(",")]:
        count = (1 << lg) // 4
        if a.coll == "allgather":
            xs = [torch.randn(count // n, device="cuda") for _ in range(n)]
            ys = [torch.empty(count // n * n, device="cuda") for _ in range(n)]
        else:
            xs = [torch.randn(count, device="cuda") for _ in range(n)]
            ys = [torch.empty_like(x) for x in xs]
        graphs = []
        for cm in comms:
            fn = getattr(cm, a.coll + "_lb")
            for _ in range(3):
                fn(xs, ys)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); fn(xs, ys); e1.record(); torch.cuda.synchronize()
            iters = int(min(500, max(5, 10.0 / max(e0.elapsed_time(e1), 1e-3))))
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(iters):
                    fn(xs, ys)
            graphs.append((g, iters))
        times = [[] for _ in cfgs]
        for _ in range(a.reps):
            for i, (g, iters) in enumerate(graphs):
                g.replay()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
                times[i].append(e0.elapsed_time(e1) / iters * 1e3)
        row = {"bytes_per_rank": 1 << lg}
        for (name, _), t in zip(cfgs, times):
            row[name or "default"] = round(statistics.median(t), 3)
        print(json.dumps(row), flush=True)
        out.append(row)
        del graphs, xs, ys
        torch.cuda.empty_cache()
    for cm in comms:
        assert cm.get_async_error() == 0
    if a.out:
        json.dump({"coll": a.coll, "ranks": n, "mode": a.mode, "rows": out}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
