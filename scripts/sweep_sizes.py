"""Message-size sweep of the engine on one B200 (loopback virtual ranks).

    python scripts/sweep_sizes.py [--ranks 8] [--dtype f32] [--mode direct] [--out gpurun_out/sizes.json]

For each size (bytes per rank, 1 KiB .. 1 GiB) times back-to-back calls with CUDA
events (>= 20 ms per point, 5 <= iters <= 2000) and reports time per call,
algbw, busbw = algbw * 2(n-1)/n, and the HBM roofline fraction of the DIRECT
plan (2 n S algorithmic bytes per call).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--dtype", default="f32", choices=["f32", "bf16"])
    ap.add_argument("--mode", default="direct", choices=["direct", "staged"])
    ap.add_argument("--coll", default="allreduce", choices=["allreduce", "allgather", "alltoall", "reducescatter", "reduce", "broadcast"])
    ap.add_argument("--chunk-kib", type=int, default=256)
    ap.add_argument("--min-log2", type=int, default=10)
    ap.add_argument("--max-log2", type=int, default=30)
    ap.add_argument("--graph", action="store_true", help="time a CUDA graph of back-to-back calls")
    ap.add_argument("--engine", type=int, default=-1, help="0 LDG, 1 TMA, 2 auto (default: library default)")
    ap.add_argument("--piece-kib", type=int, default=-1, help="work-piece traffic target (0 = automatic)")
    ap.add_argument("--sched", type=int, default=-1, help="LDG kernel: 0 dynamic claims, 1 static, 2 auto")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sizes.json"))
    a = ap.parse_args()

    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G

    n = a.ranks
    es = 4 if a.dtype == "f32" else 2
    tdt = torch.float32 if a.dtype == "f32" else torch.bfloat16
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    maxb = 1 << a.max_log2
    scratch = 64 << 20 if a.mode == "direct" else 2 * maxb + (64 << 20)
    comm = pkg.Communicator.loopback(n, scratch_bytes=scratch, mode=a.mode)
    if a.engine >= 0:
        comm.config("engine", a.engine)
    if a.sched >= 0:
        comm.config("sched", a.sched)
    if a.piece_kib >= 0:
        comm.config("piece_kib", a.piece_kib)
    chunk = a.chunk_kib * 1024
    if a.coll == "allreduce":
        comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=chunk))
    elif a.coll == "allgather":
        comm.set_strategy("allgather", G.allgather_stars(n, chunk=chunk))
    elif a.coll == "alltoall":
        comm.set_strategy("alltoall", G.alltoall_direct(n, chunk=chunk))
    elif a.coll == "reducescatter":
        comm.set_strategy("reducescatter", G.reducescatter_stars(n, chunk=chunk))
    # reduce / broadcast: the library's default star rooted at the call's root (rank 0)
    res = []
    for lg in range(a.min_log2, a.max_log2 + 1):
        nbytes = 1 << lg
        count = nbytes // es
        if a.coll == "allreduce":
            xs = [torch.randn(count, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty_like(x) for x in xs]
            call = lambda: comm.allreduce_lb(xs, ys)  # noqa: E731
            factor, alg_bytes = 2.0 * (n - 1) / n, 2 * n * nbytes
        elif a.coll == "allgather":
            xs = [torch.randn(count // n or 1, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty(n * xs[0].numel(), device="cuda", dtype=tdt) for _ in range(n)]
            call = lambda: comm.allgather_lb(xs, ys)  # noqa: E731
            # DIRECT: every shard read once, written to all n outputs
            factor, alg_bytes = (n - 1.0) / n, n * n * xs[0].numel() * es + n * xs[0].numel() * es
        elif a.coll == "alltoall":
            xs = [torch.randn(count, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty_like(x) for x in xs]
            call = lambda: comm.alltoall_lb(xs, ys)  # noqa: E731
            factor, alg_bytes = (n - 1.0) / n, 2 * n * nbytes
        elif a.coll == "reducescatter":  # bytes_per_rank = input per rank (n blocks), nccl-tests convention
            xs = [torch.randn(count // n * n or n, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty(xs[0].numel() // n, device="cuda", dtype=tdt) for _ in range(n)]
            call = lambda: comm.reducescatter_lb(xs, ys)  # noqa: E731
            # DIRECT: every input read once, every output block written once
            factor, alg_bytes = (n - 1.0) / n, (n + 1) * xs[0].numel() * es
        elif a.coll == "reduce":
            xs = [torch.randn(count, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty_like(x) for x in xs]
            call = lambda: comm.reduce_lb(xs, ys, 0)  # noqa: E731
            factor, alg_bytes = 1.0, (n + 1) * nbytes
        else:
            xs = [torch.randn(count, device="cuda").to(tdt) for _ in range(n)]
            ys = [torch.empty_like(x) for x in xs]
            call = lambda: comm.broadcast_lb(xs, ys, 0)  # noqa: E731
            factor, alg_bytes = 1.0, (n + 1) * nbytes
        for _ in range(5):
            call()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        call()
        e1.record()
        torch.cuda.synchronize()
        one = max(e0.elapsed_time(e1), 1e-3)
        iters = int(min(2000, max(5, 20.0 / one)))
        if a.graph:   # device time only: no host launch gaps between calls
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(iters):
                    call()
            g.replay()
            torch.cuda.synchronize()
            e0.record()
            g.replay()
            e1.record()
        else:
            e0.record()
            for _ in range(iters):
                call()
            e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / iters
        algbw = nbytes / (ms * 1e-3) / 1e9
        res.append({"bytes_per_rank": nbytes, "us": round(ms * 1e3, 3), "algbw": round(algbw, 3),
                    "busbw": round(algbw * factor, 3),
                    "hbm_frac": round(alg_bytes / (ms * 1e-3) / 1e9 / peak, 4), "iters": iters})
        print(json.dumps(res[-1]), flush=True)
        del xs, ys
        torch.cuda.empty_cache()
    assert comm.get_async_error() == 0
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump({"ranks": n, "dtype": a.dtype, "mode": a.mode, "coll": a.coll, "chunk": chunk,
               "graph": a.graph, "engine": a.engine, "piece_kib": a.piece_kib, "sched": a.sched, "note": "same buffers every call: sizes whose 2nS fit in L2 run from L2",
               "points": res}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
