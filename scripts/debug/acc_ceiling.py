"""Phase-2 ACCUMULATE ceiling: plain kernels (acc_ceiling.cu) vs the engine at
16-100 MiB per rank, graph-timed back to back like scripts/bench_accumulate.py.

    python scripts/debug/acc_ceiling.py [--sizes 16,25,64,100]
"""
import argparse
import ctypes
import json
import os
import statistics
import subprocess
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))


def lib():
    so = os.path.join(HERE, "acc_ceiling.so")
    if not os.path.exists(so):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                               "-Xcompiler", "-fPIC", "-o", so, os.path.join(HERE, "acc_ceiling.cu")])
    L = ctypes.CDLL(so)
    L.acc_launch.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                             ctypes.POINTER(ctypes.c_void_p), ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                             ctypes.c_void_p]
    return L


def gtime(fn, traffic, pk, reps=7):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    iters = max(5, min(200, int(2e-2 / (traffic / (pk * 1e9)))))
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(iters):
            fn()
    t = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        t.append(e0.elapsed_time(e1) / iters * 1e3)
    return statistics.median(t)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="16,25,64,100")
    ap.add_argument("--ar-sizes", default="8,16,32,64")
    a = ap.parse_args()
    pk = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]) \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6534.1
    L = lib()
    n, R2 = 8, {3, 6}
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    for mib in [float(s) for s in a.sizes.split(",")]:
        count = int(mib * (1 << 20)) // 4
        traffic = 18 * count * 4
        xs = [torch.randn(count, device="cuda") if r in R2 else None for r in range(n)]
        ys = [torch.randn(count, device="cuda") for _ in range(n)]
        dst = (ctypes.c_void_p * 8)(*[y.data_ptr() for y in ys])
        row = {"mib_per_rank": mib}
        row["engine"] = gtime(lambda: c.allreduce_lb(xs, ys, ready=R2, accumulate=True), traffic, pk)
        for kind, kn, unrolls, grids in ((0, "ldst", (1, 4), ((2, 256), (4, 256), (16, 256))),
                                         (2, "batch", (1, 2), ((1, 256), (2, 256), (4, 256), (8, 256)))):
            for unroll in unrolls:
                for grid_mult, block in grids:
                    fn = lambda: L.acc_launch(kind, unroll, xs[3].data_ptr(), xs[6].data_ptr(), dst,  # noqa: E731
                                              count // 4, 148 * grid_mult, block,
                                              torch.cuda.current_stream().cuda_stream)
                    row[f"{kn}_u{unroll}_g{grid_mult}x{block}"] = gtime(fn, traffic, pk)
        cp_src = torch.empty(traffic // 8, dtype=torch.float32, device="cuda")
        cp_dst = torch.empty_like(cp_src)
        row["torch_copy_same_bytes"] = gtime(lambda: cp_dst.copy_(cp_src), traffic, pk)
        out = {"mib_per_rank": mib, "traffic": traffic}
        for k, us in row.items():
            if k != "mib_per_rank":
                out[k] = {"us": round(us, 2), "frac": round(traffic / (us * 1e-6) / 1e9 / pk, 4)}
        print(json.dumps(out), flush=True)
        del xs, ys, cp_src, cp_dst
        torch.cuda.empty_cache()
    L.ar_launch.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_void_p),
                            ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
    for mib in [float(s) for s in a.ar_sizes.split(",")]:
        count = int(mib * (1 << 20)) // 4
        traffic = 2 * n * count * 4
        xs = [torch.randn(count, device="cuda") for r in range(n)]
        ys = [torch.randn(count, device="cuda") for _ in range(n)]
        src = (ctypes.c_void_p * 8)(*[x.data_ptr() for x in xs])
        dst = (ctypes.c_void_p * 8)(*[y.data_ptr() for y in ys])
        row = {"engine": gtime(lambda: c.allreduce_lb(xs, ys), traffic, pk)}
        for unroll in (1, 2):
            for grid_mult in (1, 2, 4, 8):
                fn = lambda: L.ar_launch(unroll, src, dst, count // 4, 148 * grid_mult, 256,  # noqa: E731
                                         torch.cuda.current_stream().cuda_stream)
                row[f"ar_u{unroll}_g{grid_mult}x256"] = gtime(fn, traffic, pk)
        out = {"allreduce_mib_per_rank": mib, "traffic": traffic}
        for k, us in row.items():
            out[k] = {"us": round(us, 2), "frac": round(traffic / (us * 1e-6) / 1e9 / pk, 4)}
        print(json.dumps(out), flush=True)
        del xs, ys
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
