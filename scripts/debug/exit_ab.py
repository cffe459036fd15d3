"""A/B of compile-time engine variants (-D defines) on the loopback DIRECT path,
interleaved subprocesses, graph-timed: ACCUMULATE (phase 2, ready {3, 6} of 8,
18 S of traffic) and plain AllReduce (16 S), fraction of the HBM copy peak.

    python scripts/debug/exit_ab.py --build         # here: compile the variants in-tree
    python scripts/debug/exit_ab.py [--rounds 3]    # GPU box
"""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
VARIANTS = {"base": (), "exit_read": ("ADAPCC_EXIT_READ=1",)}   # exit_read: r02 A/B, define since removed
PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]


def lib(v):
    return os.path.join(ROOT, "paper_conf_icdcs_zhaozw24_b200", f"libadapcc_ab_{v}.so")


def run_one():
    import torch
    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    n, R2 = 8, {3, 6}
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    out = {}
    for what, mib in (("acc", 16), ("acc", 25), ("acc", 64), ("ar", 16), ("ar", 64)):
        count = (mib << 20) // 4
        xs = [torch.randn(count, device="cuda") for _ in range(n)]
        ys = [torch.randn(count, device="cuda") for _ in range(n)]
        if what == "acc":
            fn = lambda: c.allreduce_lb([x if r in R2 else None for r, x in enumerate(xs)], ys, ready=R2,  # noqa
                                        accumulate=True)
            traffic = 18 * (mib << 20)
        else:
            fn = lambda: c.allreduce_lb(xs, ys)  # noqa
            traffic = 16 * (mib << 20)
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        reps = 10
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(reps):
                fn()
        t = []
        for _ in range(7):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            t.append(a.elapsed_time(b) / reps * 1e3)
        us = statistics.median(t)
        out[f"{what}{mib}"] = {"us": round(us, 2), "frac": round(traffic / us / 1e3 / PEAK, 4)}
        del xs, ys, g
    assert c.get_async_error() == 0
    print(json.dumps(out))


def main():
    if "--one" in sys.argv:
        return run_one()
    if "--build" in sys.argv:
        from paper_conf_icdcs_zhaozw24_b200 import _build
        for v, d in VARIANTS.items():
            _build.build(out=lib(v), defines=d)
        return
    rounds = int(sys.argv[sys.argv.index("--rounds") + 1]) if "--rounds" in sys.argv else 3
    res = {v: [] for v in VARIANTS}
    for _ in range(rounds):
        for v in VARIANTS:
            p = subprocess.run([sys.executable, __file__, "--one"], env=dict(os.environ, ADAPCC_LIB=lib(v)),
                               capture_output=True, text=True, timeout=300)
            line = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
            r = json.loads(line[-1]) if line else {"error": p.stderr[-400:]}
            res[v].append(r)
            print(v, json.dumps(r), flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "exit_ab.json"), "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
