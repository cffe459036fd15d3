"""BASELINE config C3 on one B200: partial-aggregation AllReduce, 8 virtual
ranks, stragglers {3, 6} with a CONTROLLED lag (a one-thread %globaltimer spin
on their own stream, adapcc_spin -- it takes no SM time from the collective),
driven by the online coordinator (break-even rule on the readiness board,
P:L129-137) with late join.

Per size (25 / 50 / 100 MiB fp32 per rank, the DDP bucket sizes of C3) and lag
t_s in {0, 0.25, 0.5, 1, 2} x T_full:
  T_wait   = t_s + the full AllReduce (stream-ordered after the straggler)
  T_adapcc = coordinator with the calibrated break-even buying cost
             (phase 1 + phase 2 measured on this box)
  T_eager  = coordinator that proceeds at its first cycle (late join makes
             phase 1 cheap to start)
each the median of --runs device-timed runs (CUDA events from the straggler's
start to the end of the last call), measured twice (repeat A / B).

    python scripts/bench_c3.py --out gpurun_out/c3_r02.json [--modes staged,direct]
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
from paper_conf_icdcs_zhaozw24_b200 import coordinator as C  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

N, R, LATE = 8, {0, 1, 2, 4, 5, 7}, (3, 6)


def ev():
    return torch.cuda.Event(enable_timing=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="25,50,100")
    ap.add_argument("--modes", default="staged,direct")
    ap.add_argument("--lags", default="0,0.25,0.5,1,2")
    ap.add_argument("--runs", type=int, default=7)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    out = {"what": "C3 partial aggregation with a controlled straggler, online coordinator + late join",
           "ranks": N, "ready": sorted(R), "stragglers": list(LATE), "rows": []}
    cs = torch.cuda.Stream(priority=-1)
    side = torch.cuda.Stream()
    for mode in a.modes.split(","):
        for mib in [int(s) for s in a.sizes.split(",")]:
            count = (mib << 20) // 4
            comm = pkg.Communicator.loopback(N, mode=mode, scratch_bytes=(2 * (mib << 20) + (64 << 20))
                                             if mode == "staged" else 64 << 20)
            comm.set_strategy("allreduce", G.allreduce_stars(N, chunk=262144))
            xs = [torch.randn(count, device="cuda") for _ in range(N)]
            ys = [torch.empty_like(x) for x in xs]

            def timed(fn, reps=5):
                torch.cuda.synchronize()
                ts = []
                for _ in range(reps):
                    e0, e1 = ev(), ev()
                    e0.record(cs)
                    fn()
                    e1.record(cs)
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1) * 1e-3)
                return statistics.median(ts)

            with torch.cuda.stream(cs):
                full = lambda: comm.allreduce_lb(xs, ys, stream=cs)  # noqa: E731
                full()
                t_full = timed(full)
                # phase 1 with nobody joining, then the whole complement: the buying cost
                comm.allreduce_lb(xs, ys, ready=R, late="join", stream=cs)
                comm.allreduce_lb(xs, ys, ready=R, late="complement", stream=cs)
                t_p1 = timed(lambda: comm.allreduce_lb(xs, ys, ready=R, late="join", stream=cs))
                t_p12 = timed(lambda: (comm.allreduce_lb(xs, ys, ready=R, late="join", stream=cs),
                                       comm.allreduce_lb(xs, ys, ready=R, late="complement", stream=cs)))
            buy = t_p12

            def policy(buy_s):
                def make():
                    p = C.Coordinator(N, "allreduce", count * 4, 100e9, 2e-6)
                    p.buy_cost = lambda k: buy_s
                    return p
                return make

            coord = {"break_even": C.OnlineCoordinator(comm, policy(buy), cycle=2e-6),
                     "eager": C.OnlineCoordinator(comm, policy(0.0), cycle=2e-6)}

            def run_wait(ts_ns):
                torch.cuda.synchronize()
                e0, e1 = ev(), ev()
                e0.record(cs)
                comm.spin(ts_ns, stream=cs)
                comm.allreduce_lb(xs, ys, stream=cs)
                e1.record(cs)
                torch.cuda.synchronize()
                return e0.elapsed_time(e1) * 1e-3, None

            def run_coord(name, ts_ns):
                co = coord[name]
                t = co.ticket()
                for r in R:                             # the ready ranks finished before t = 0
                    comm.signal_ready(r, ticket=t, stream=cs)
                torch.cuda.synchronize()
                e0, e1 = ev(), ev()
                e0.record(side)
                comm.spin(ts_ns, stream=side)           # the stragglers' computation
                for r in LATE:
                    comm.signal_ready(r, ticket=t, stream=side)
                res = co.allreduce(lambda m, lt: comm.allreduce_lb(xs, ys, ready=m, late=lt, stream=cs))
                e1.record(cs)
                torch.cuda.synchronize()
                assert comm.get_async_error() == 0
                return e0.elapsed_time(e1) * 1e-3, res["action"]

            for lag in [float(x) for x in a.lags.split(",")]:
                ts_ns = int(lag * t_full * 1e9)
                row = {"mode": mode, "mib_per_rank": mib, "t_full_us": round(t_full * 1e6, 2),
                       "t_phase1_us": round(t_p1 * 1e6, 2), "t_phase1_plus_2_us": round(t_p12 * 1e6, 2),
                       "lag_over_t_full": lag, "lag_us": round(ts_ns / 1e3, 2)}
                for name, fn in (("wait", lambda: run_wait(ts_ns)),
                                 ("break_even", lambda: run_coord("break_even", ts_ns)),
                                 ("eager", lambda: run_coord("eager", ts_ns))):
                    reps = []
                    for rep in range(2):
                        res = [fn() for _ in range(a.runs)]
                        reps.append({"median_us": round(statistics.median(r[0] for r in res) * 1e6, 2),
                                     "actions": sorted({str(r[1]) for r in res})})
                    row[name] = {"repeat_a": reps[0], "repeat_b": reps[1],
                                 "repeat_spread": round(abs(reps[0]["median_us"] - reps[1]["median_us"]) /
                                                        max(reps[0]["median_us"], 1e-9), 4)}
                for name in ("break_even", "eager"):
                    row[name]["speedup_vs_wait"] = round(row["wait"]["repeat_a"]["median_us"] /
                                                         row[name]["repeat_a"]["median_us"], 3)
                out["rows"].append(row)
                print(json.dumps(row), flush=True)
            comm.finalize()
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
