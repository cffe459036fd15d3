"""Work-piece sizing sweep (one B200, loopback virtual ranks, CUDA-graph timed).

    python scripts/sweep_taper.py [--ranks 8] [--dtype f32] [--mode direct] [--coll allreduce]
                                  [--tapers 1,2,4,8] [--pieces 0,128] [--out gpurun_out/taper.json]

For each message size (bytes per rank), every (piece_kib, taper) setting is timed
as a CUDA graph of back-to-back calls, settings interleaved and repeated 3 times
(median), so that the comparison is not skewed by clock drift.  Reports us per
call and the HBM fraction of the DIRECT plan's algorithmic bytes (2 n S).
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--dtype", default="f32", choices=["f32", "bf16"])
    ap.add_argument("--mode", default="direct", choices=["direct", "staged"])
    ap.add_argument("--coll", default="allreduce", choices=["allreduce", "alltoall"])
    ap.add_argument("--engine", type=int, default=2)
    ap.add_argument("--tapers", default="1,2,4,8")
    ap.add_argument("--pieces", default="0")
    ap.add_argument("--blobs", default="1", help="first_blob settings (LDG kernel first-item blobs)")
    ap.add_argument("--min-log2", type=int, default=20)
    ap.add_argument("--max-log2", type=int, default=28)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "taper.json"))
    a = ap.parse_args()

    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G

    n = a.ranks
    es = 4 if a.dtype == "f32" else 2
    tdt = torch.float32 if a.dtype == "f32" else torch.bfloat16
    pk = os.path.join(ROOT, "MEASURED_PEAKS.json")
    peak = json.load(open(pk))["hbm_gbs"] if os.path.exists(pk) else 6650.0
    maxb = 1 << a.max_log2
    scratch = 64 << 20 if a.mode == "direct" else 2 * maxb + (64 << 20)
    comm = pkg.Communicator.loopback(n, scratch_bytes=scratch, mode=a.mode)
    comm.config("engine", a.engine)
    if a.coll == "allreduce":
        comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=256 << 10))
    else:
        comm.set_strategy("alltoall", G.alltoall_direct(n, chunk=256 << 10))
    settings = [(int(p), int(t), int(b)) for p in a.pieces.split(",") for t in a.tapers.split(",")
                for b in a.blobs.split(",")]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    res = []
    for lg in range(a.min_log2, a.max_log2 + 1):
        nbytes = 1 << lg
        count = nbytes // es
        xs = [torch.randn(count, device="cuda").to(tdt) for _ in range(n)]
        ys = [torch.empty_like(x) for x in xs]
        fn = comm.allreduce_lb if a.coll == "allreduce" else comm.alltoall_lb
        graphs = {}
        for (pc, tp, bl) in settings:
            comm.config("piece_kib", pc)
            comm.config("taper", tp)
            comm.config("first_blob", bl)
            for _ in range(3):
                fn(xs, ys)
            torch.cuda.synchronize()
            e0.record()
            fn(xs, ys)
            e1.record()
            torch.cuda.synchronize()
            iters = int(min(500, max(5, 10.0 / max(e0.elapsed_time(e1), 1e-3))))
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(iters):
                    fn(xs, ys)
            graphs[(pc, tp, bl)] = (g, iters)
        times = {s: [] for s in settings}
        for _ in range(3):
            for s in settings:
                g, iters = graphs[s]
                g.replay()
                torch.cuda.synchronize()
                e0.record()
                g.replay()
                e1.record()
                torch.cuda.synchronize()
                times[s].append(e0.elapsed_time(e1) / iters)
        for s in settings:
            ms = statistics.median(times[s])
            res.append({"bytes_per_rank": nbytes, "piece_kib": s[0], "taper": s[1], "first_blob": s[2],
                        "us": round(ms * 1e3, 3),
                        "hbm_frac": round(2 * n * nbytes / (ms * 1e-3) / 1e9 / peak, 4)})
            print(json.dumps(res[-1]), flush=True)
        del graphs, xs, ys
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
    assert comm.get_async_error() == 0
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump({"ranks": n, "dtype": a.dtype, "mode": a.mode, "coll": a.coll, "engine": a.engine,
               "note": "graph-timed, same buffers every call, median of 3 interleaved repetitions",
               "points": res}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
