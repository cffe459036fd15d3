"""Benchmark of the AdapCC B200 hot path -- prints ONE JSON line.

Metric (BASELINE.json): AllReduce busbw (GB/s) = algbw * 2(n-1)/n, algbw =
bytes per rank / time per call (nccl-tests convention).

  python bench.py                      # N=1: 8 virtual ranks on one B200 (loopback)
  python bench.py --gpus N             # N>1: re-launches itself under torch.distributed.run,
                                       #      one process per GPU, CUDA IPC (fails without N GPUs)
  torchrun --nproc-per-node N bench.py --gpus N   # the same, launched by the caller
  python bench.py --gpus N --test-same-gpu        # N>1 code path, N processes on cuda:0
  python bench.py --impl reference     # the CPU oracle timed on the host (reference arm)

N=1 workload: BASELINE config C2's multi-tree AllReduce at the paper's
microbenchmark size ("float data of 256 MB"): 8 ranks x 256 MiB fp32,
8 weighted star trees (one per rank, chunk 256 KiB), all ranks ready.  One B200
hosts all 8 ranks (loopback DIRECT plan: every input read once, every output
written once), so the kernel is HBM-bound and the roofline is HBM.
N>1: the same call through CUDA IPC over NVLink (STAGED protocol), NCCL timed
beside it on the same buffers.
"""

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "AllReduce busbw GB/s vs size at 2/4/8 B200 (% of 900 GB/s) vs NCCL"
UNIT = "GB/s"
NVLINK_NOMINAL = 900.0
ENGINE_NAMES = {0: "adapcc::engine_kernel (128-bit LDG/STG fold)",
                1: "adapcc::{ns}::engine_tma_kernel (TMA bulk-copy pipeline)",
                3: "adapcc::flat::flat_kernel (grid-stride over flag-free tasks)"}


def engine_name(engine, mode, dtype):
    ns = "tma_direct" if mode == "direct" else "tma_staged"
    return ENGINE_NAMES.get(engine, "?").format(ns=ns) + f"<{dtype}>"


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--vranks", type=int, default=8, help="virtual ranks at N=1")
    p.add_argument("--size-mib", type=float, default=256.0, help="bytes per rank (MiB)")
    p.add_argument("--dtype", choices=["f32", "bf16"], default="f32")
    p.add_argument("--mode", choices=["direct", "staged"], default="direct")
    p.add_argument("--chunk-kib", type=int, default=256)
    p.add_argument("--e2e-steps", type=int, default=16,
                   help="e2e steps: the first upload and the last download do not overlap, so K steps "
                        "reach at most K/(K+1) of the full-duplex PCIe bound")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-parity", action="store_true")
    p.add_argument("--no-sweep", action="store_true", help="skip the busbw-vs-size sweep")
    p.add_argument("--no-nccl-legs", action="store_true",
                   help="N>1: skip the NCCL_ALGO / NVLS leg runs (separate torchrun jobs)")
    p.add_argument("--nccl-leg", default=None, help=argparse.SUPPRESS)   # internal: one NCCL variant
    p.add_argument("--nvls-leg", action="store_true", help=argparse.SUPPRESS)   # internal: the NVLS leg
    p.add_argument("--test-same-gpu", action="store_true",
                   help="N>1 code-path check on a 1-GPU box: every rank on cuda:0, gloo, no NCCL leg "
                        "(numbers are NOT NVLink measurements)")
    return p.parse_args()


def dist_env():
    r = int(os.environ.get("RANK", "0"))
    w = int(os.environ.get("WORLD_SIZE", "1"))
    lr = int(os.environ.get("LOCAL_RANK", "0"))
    return r, w, lr


def busbw(bytes_per_rank, seconds, n):
    return bytes_per_rank / seconds / 1e9 * (2.0 * (n - 1) / n)


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def profile_traffic(key):
    """dram bytes per launch from the newest committed ncu --set full summary
    (profiles/ncu_summary_rNN.json, else the r01 ncu_summary.json), if any."""
    import glob
    paths = sorted(glob.glob(os.path.join(ROOT, "profiles", "ncu_summary_r*.json")), reverse=True)
    for path in paths + [os.path.join(ROOT, "profiles", "ncu_summary.json")]:
        try:
            with open(path) as f:
                v = json.load(f).get(key, {}).get("dram_bytes_per_launch")
            if v:
                return v
        except Exception:  # noqa: BLE001
            continue
    return None


def traffic_key(engine, mode):
    return f"allreduce_loopback_{mode}_{'tma' if engine == 1 else 'ldg'}"


class ClockSampler:
    """NVML clocks + throttle reasons sampled DURING the timed region."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            names = {
                getattr(pynvml, "nvmlClocksThrottleReasonHwSlowdown", 0x8): "hw_slowdown",
                getattr(pynvml, "nvmlClocksThrottleReasonHwThermalSlowdown", 0x40): "hw_thermal_slowdown",
                getattr(pynvml, "nvmlClocksThrottleReasonSwThermalSlowdown", 0x20): "sw_thermal_slowdown",
                getattr(pynvml, "nvmlClocksThrottleReasonSwPowerCap", 0x4): "sw_power_cap",
            }

            def loop():
                while not self._stop.is_set():
                    try:
                        self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                        bits = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                        for b, nm in names.items():
                            if bits & b:
                                self.reasons.add(nm)
                    except Exception:  # noqa: BLE001
                        pass
                    time.sleep(0.001)

            self._t = threading.Thread(target=loop, daemon=True)
            self._t.start()
        except Exception:  # noqa: BLE001
            self._t = None
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=2)

    def summary(self):
        s = sorted(self.samples)
        med = s[len(s) // 2] if s else None
        return {"sm_mhz": med, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(s)}


# ------------------------------------------------------------- size sweep
SWEEP_SIZES = [1 << s for s in range(10, 29, 2)]   # bytes per rank: 1 KiB .. 256 MiB, x4 steps


def time_point(fn, reduce_max=None, graph=True, fn_graph=None):
    """Per-call device time (ms) of back-to-back calls, two ways: plain
    enqueue on the current stream ("ms", host enqueue included when it is the
    bottleneck) and a CUDA graph of the same calls ("ms_graph", device time
    only; fn_graph, default fn, must enqueue on the current stream).
    >= ~10 ms per measurement.  reduce_max: max over ranks (N>1)."""
    import torch
    cur = torch.cuda.current_stream()
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(cur)
    fn()
    b.record(cur)
    torch.cuda.synchronize()
    one = max(a.elapsed_time(b), 1e-3)
    iters = int(min(1000, max(5, 10.0 / one)))
    if reduce_max:
        iters = int(reduce_max(float(iters), op="min"))   # same count on every rank
        reduce_max(0.0)                                   # barrier
    a.record(cur)
    for _ in range(iters):
        fn()
    b.record(cur)
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / iters
    if not graph:
        return (reduce_max(ms) if reduce_max else ms), None
    s = torch.cuda.Stream()
    s.wait_stream(cur)
    with torch.cuda.stream(s):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(iters):
                (fn_graph or fn)()
    torch.cuda.synchronize()
    if reduce_max:
        reduce_max(0.0)
    g.replay()
    torch.cuda.synchronize()
    if reduce_max:
        reduce_max(0.0)
    a.record(cur)
    g.replay()
    b.record(cur)
    torch.cuda.synchronize()
    msg = a.elapsed_time(b) / iters
    del g
    if reduce_max:
        ms, msg = reduce_max(ms), reduce_max(msg)
    return ms, msg


# ------------------------------------------------------------------ oracle leg
def pin_one_core():
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    except Exception:  # noqa: BLE001
        pass


def oracle_replay(xs, text, n, dtype):
    """The CPU oracle (as it stands) on the whole workload: (outputs, seconds)."""
    from oracle import collectives as oc
    t0 = time.perf_counter()
    ys = oc.allreduce(xs, text, set(range(n)), dtype)
    return ys, time.perf_counter() - t0


def cpu_baseline_block(xs, text, n, dtype, first_s, target_s=15.0):
    """The oracle timed on the bench workload itself (every rank's full
    tensor), one host core; `first_s` = the replay parity already timed."""
    es = 4 if dtype == "f32" else 2
    reps = max(0, min(20, int(round(target_s / max(first_s, 1e-6))) - 1))
    times = [first_s]
    pin_one_core()
    for _ in range(reps):
        times.append(oracle_replay(xs, text, n, dtype)[1])
    t = sum(times) / len(times)
    return {"value": round(busbw(len(xs[0]) * es, t, n), 4), "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"the full bench workload ({n} simulated ranks x {len(xs[0]) * es >> 20} MiB {dtype}, "
                      f"strategy-order replay), {len(times)} reps, mean {t:.2f} s, numpy single thread pinned "
                      f"to 1 core of {os.cpu_count()}"}


def run_reference(args):
    """Reference arm of this tier: the CPU oracle, as it stands, timed on the
    host on this arm's own workload (N ranks x size-mib per step, N = 8
    virtual ranks at --gpus 1).  Under torchrun only rank 0 runs it."""
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    from synth import rank_tensors
    r, w, _ = dist_env()
    if r != 0:
        return None
    ngpus = max(w, args.gpus)
    n = args.vranks if ngpus == 1 else ngpus
    es = 4 if args.dtype == "f32" else 2
    count = int(args.size_mib * (1 << 20)) // 16 * 16 // es
    xs = rank_tensors(args.dtype, count, n)
    text = G.allreduce_stars(n, chunk=args.chunk_kib * 1024)
    pin_one_core()
    for _ in range(args.warmup):
        oracle_replay(xs, text, n, args.dtype)
    times = [oracle_replay(xs, text, n, args.dtype)[1] for _ in range(args.steps)]
    t = sum(times) / len(times)
    v = busbw(count * es, t, n)
    sample = (f"the whole workload every step: {n} simulated ranks x {count * es >> 20} MiB {args.dtype} "
              f"(strategy-order replay of {n} star trees), numpy single thread pinned to 1 core of {os.cpu_count()}")
    return {
        "impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": UNIT,
        "n_gpus": ngpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": args.dtype,
        "data": "synthetic", "config": workload_config(args, n, ngpus),
        "cpu_baseline": {"value": round(v, 4), "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


def workload_config(args, n, world):
    nbytes = int(args.size_mib * (1 << 20))
    where = "loopback-vr" if world == 1 else "ipc-gpu"
    return {
        "workload": f"allreduce-{where}{n}-{args.dtype}-{nbytes >> 20}MiB-star{n}",
        "ranks": n, "virtual_ranks": world == 1, "bytes_per_rank": nbytes,
        "strategy": f"{n} star trees (one rooted at each rank), equal weights, chunk {args.chunk_kib} KiB",
        "mode": args.mode if world == 1 else "zero-copy direct (registered buffers)", "ready_mask": "all",
        "l2": f"inputs {n * nbytes >> 20} MiB per step > 126 MB L2 (no flush needed)",
        "parallelism": f"{'virtual ' if world == 1 else ''}dp{n}",
        "same_gpu": bool(world > 1 and getattr(args, "test_same_gpu", False)),
    }


# ---------------------------------------------------------------- our arm, N=1
def run_single(args):
    import numpy as np
    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    from synth import rank_tensors

    torch.cuda.set_device(0)
    n = args.vranks
    es = 4 if args.dtype == "f32" else 2
    nbytes = int(args.size_mib * (1 << 20)) // 16 * 16
    count = nbytes // es
    tdt = torch.float32 if args.dtype == "f32" else torch.bfloat16
    text = G.allreduce_stars(n, chunk=args.chunk_kib * 1024)

    # staged: each half needs ~S of slots + a flag region of half/32
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=max(64 << 20, 2 * nbytes + nbytes // 8 + (16 << 20))
                                     if args.mode == "staged" else 64 << 20, mode=args.mode)
    comm.set_strategy("allreduce", text)

    host_in = []
    for r in range(n):
        x = rank_tensors(args.dtype, count, 1, base=1000 + r)[0]
        t = torch.from_numpy(x)
        if args.dtype == "bf16":
            t = t.view(torch.int16)
        host_in.append(t.pin_memory())
    dx = [h.cuda().view(tdt) for h in host_in]
    dy = [torch.empty(count, dtype=tdt, device="cuda") for _ in range(n)]
    stream = torch.cuda.current_stream()

    for _ in range(args.warmup):
        comm.allreduce_lb(dx, dy)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    launches0 = comm.launch_count()
    with ClockSampler(0) as clk:
        torch.cuda.synchronize()
        t_begin = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_begin.record(stream)
        for i in range(args.steps):
            starts[i].record(stream)
            comm.allreduce_lb(dx, dy)
            ends[i].record(stream)
        t_end.record(stream)
        torch.cuda.synchronize()
    launches = comm.launch_count() - launches0
    assert comm.get_async_error() == 0
    total_ms = t_begin.elapsed_time(t_end)
    per = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    ms = total_ms / args.steps
    kern_ms = sum(per) / len(per)
    value = busbw(nbytes, ms / 1e3, n)

    # parity at the bench point: EVERY output element of every rank against
    # the oracle's strategy-order replay of the same inputs, bit-exact
    parity, xs_np, oracle_s = None, None, None
    if not args.no_parity or not args.no_cpu_baseline:
        xs_np = [h.numpy().view(np.uint16) if args.dtype == "bf16" else h.numpy() for h in host_in]
        ys, oracle_s = oracle_replay(xs_np, text, n, args.dtype)
        if not args.no_parity:
            parity = complete_parity(dy, ys, args.dtype)
        del ys

    # end to end: pinned host inputs -> device -> allreduce -> pinned host, every
    # step.  Steps are pipelined like a training loop's buckets: double-buffered
    # device tensors, H2D on one copy stream and D2H on another, so step i's
    # download overlaps step i+1's upload (PCIe is full duplex); per-step time
    # = span of all steps / steps.
    e2e_t = e2e_pipelined(comm, host_in, dx, dy, args.e2e_steps, tdt, lambda xs, ys: comm.allreduce_lb(xs, ys))
    pcie = pcie_bidir_gbs()
    pcie_ms = n * nbytes / (pcie * 1e9) * 1e3      # every step moves n*S each way

    peak, peak_src = load_peaks()
    sweep = None
    if not args.no_sweep:   # BASELINE metric is busbw vs size: every x4 size up to the bench size
        sweep = []
        warm = comm.prepare_allreduce_lb([t[:256] for t in dx], [t[:256] for t in dy])
        for _ in range(2000):      # host warm-up (clocks, caches) before the smallest point
            warm()
        torch.cuda.synchronize()
        for sb in [b for b in SWEEP_SIZES if b <= nbytes]:
            c = sb // es
            xs_, ys_ = [t[:c] for t in dx], [t[:c] for t in dy]
            call = comm.prepare_allreduce_lb(xs_, ys_)     # host fast path: one C call per AllReduce
            ms_, msg_ = time_point(call, fn_graph=lambda: comm.allreduce_lb(xs_, ys_))
            msp_, _ = time_point(lambda: comm.allreduce_lb(xs_, ys_), graph=False)
            sweep.append({"bytes_per_rank": sb, "us": round(ms_ * 1e3, 2), "us_graph": round(msg_ * 1e3, 2),
                          "us_api": round(msp_ * 1e3, 2),
                          "busbw": round(busbw(sb, ms_ / 1e3, n), 2),
                          "busbw_graph": round(busbw(sb, msg_ / 1e3, n), 2),
                          "hbm_frac_graph": round(2 * n * sb / (msg_ / 1e3) / 1e9 / peak, 4)})
        assert comm.get_async_error() == 0
    partial = None
    if not args.no_sweep and n == 8:
        # C3 (BASELINE configs[2]): partial aggregation with 2 stragglers out of 8 acting as relays, at
        # the gradient-bucket sizes -- phase 1 = the AllReduce of the 6 ready ranks (mask 0xB7, every rank
        # receives; traffic 6 S read + 8 S written), phase 2 = ACCUMULATE of the 2 late ranks (mask 0x48,
        # recv += sum; 2 S read + 8 S read and written).  Graph-timed on slices of the bench buffers.
        partial = []
        R1, R2 = {0, 1, 2, 4, 5, 7}, {3, 6}
        for mib in (16, 25, 64, 100):
            sb = (mib << 20) // 16 * 16
            if sb > nbytes:
                continue
            c = sb // es
            ys_ = [t[:c] for t in dy]
            x1 = [t[:c] if r in R1 else None for r, t in enumerate(dx)]
            x2 = [t[:c] if r in R2 else None for r, t in enumerate(dx)]
            _, m1 = time_point(lambda: comm.allreduce_lb(x1, ys_, ready=R1))
            e1 = comm.last_engine()
            _, m2 = time_point(lambda: comm.allreduce_lb(x2, ys_, ready=R2, accumulate=True))
            e2 = comm.last_engine()
            partial.append({"mib_per_rank": mib,
                            "phase1_us": round(m1 * 1e3, 2), "phase1_hbm_frac": round(14 * sb / (m1 / 1e3) / 1e9 / peak, 4),
                            "phase1_kernel": engine_name(e1, args.mode, args.dtype),
                            "phase2_us": round(m2 * 1e3, 2), "phase2_hbm_frac": round(18 * sb / (m2 / 1e3) / 1e9 / peak, 4),
                            "phase2_kernel": engine_name(e2, args.mode, args.dtype)})
        assert comm.get_async_error() == 0
    alg_bytes = 2 * n * nbytes   # every rank's input read once + output written once
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    out = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": args.dtype,
        "data": "synthetic (seeded N(0,1), synth/inputs.py)",
        "config": workload_config(args, n, 1),
        "algbw": round(nbytes / (ms / 1e3) / 1e9, 3),
        "pct_of_nvlink_900": None,
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": profile_traffic(traffic_key(comm.last_engine(), args.mode)),
                     "algorithmic_bytes_per_launch": alg_bytes, "peak_source": peak_src,
                     "kernel": engine_name(comm.last_engine(), args.mode, args.dtype),
                     "kernel_ms": round(kern_ms, 4)},
        "e2e": {"value": round(busbw(nbytes, e2e_t / 1e3, n), 3), "unit": UNIT,
                "h2d_bytes_per_step": n * nbytes, "d2h_bytes_per_step": n * nbytes,
                "ms_per_step": round(e2e_t, 3), "steps": args.e2e_steps,
                "how": "pinned H2D of all inputs + allreduce_lb + D2H of all outputs per step; steps "
                       "double-buffered with H2D and D2H on separate copy streams (full-duplex PCIe)",
                "pcie_bidir_GBps_per_direction": round(pcie, 1),
                "pcie_bound_ms_per_step": round(pcie_ms, 3),
                "pcie_roofline_frac": round(pcie_ms / e2e_t, 4),
                "pipeline_bound_frac": round(args.e2e_steps / (args.e2e_steps + 1), 4)},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "parity": parity,
        "nccl": None,
        "paper_context": PAPER_CONTEXT,
        "sweep": sweep,
        "partial_aggregation": partial,
        "partial_aggregation_how": "C3 shapes on this bench's buffers, CUDA graph of back-to-back calls: phase 1 "
                                   "= AllReduce over ready ranks {0,1,2,4,5,7} (relays 3, 6 receive), roofline "
                                   "traffic 14 S; phase 2 = ACCUMULATE of ranks {3,6} into every recvbuf, 18 S; "
                                   "fractions of the measured HBM copy peak (parity: tests/test_gpu_fullsize.py)",
        "sweep_how": "same call at every x4 size (slices of the bench buffers): back-to-back enqueue of a "
                     "prepared call (us: Communicator.prepare_allreduce_lb, one C call per AllReduce), of the "
                     "per-call API (us_api: allreduce_lb marshals its arguments every call), and a CUDA graph "
                     "of the same calls (us_graph, device time); busbw from us; sizes whose 2nS fit the "
                     "126 MB L2 run partly from L2",
    }
    if not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline_block(xs_np, text, n, args.dtype, oracle_s)
    comm.finalize()
    return out


def pcie_bidir_gbs(nbytes=256 << 20, reps=3):
    """Pinned host <-> device throughput with both directions busy at once
    (the e2e steps' regime): GB/s per direction."""
    import torch
    h = [torch.empty(nbytes, dtype=torch.uint8).pin_memory() for _ in range(2)]
    d = [torch.empty(nbytes, dtype=torch.uint8, device="cuda") for _ in range(2)]
    s = [torch.cuda.Stream(), torch.cuda.Stream()]
    cur = torch.cuda.current_stream()
    best = 0.0
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(cur)
        for x in s:
            x.wait_stream(cur)
        with torch.cuda.stream(s[0]):
            d[0].copy_(h[0], non_blocking=True)
        with torch.cuda.stream(s[1]):
            h[1].copy_(d[1], non_blocking=True)
        for x in s:
            cur.wait_stream(x)
        b.record(cur)
        torch.cuda.synchronize()
        best = max(best, nbytes / (a.elapsed_time(b) * 1e-3) / 1e9)
    return best


def e2e_pipelined(comm, host_in, dx, dy, steps, tdt, call, second=None):
    """Average per-step time (ms) of `steps` end-to-end steps, each: H2D of
    every input from pinned host memory, the collective, D2H of every output
    into pinned host memory.  Two device buffer sets; copies on their own
    streams; the collective on the current stream.  second = (dx2, dy2): the
    second buffer set (e.g. registered for zero-copy), else allocated here."""
    import torch
    cur = torch.cuda.current_stream()
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    if second is None:
        second = ([torch.empty_like(t) for t in dx], [torch.empty_like(t) for t in dy])
    bx = [dx, second[0]]
    by = [dy, second[1]]
    hout = [[torch.empty(t.numel(), dtype=host_in[0].dtype).pin_memory() for t in dy] for _ in range(2)]
    ev = lambda: torch.cuda.Event()  # noqa: E731
    ar_done = [None, None]
    out_done = [None, None]

    def step(i):
        b = i % 2
        with torch.cuda.stream(s_in):
            if ar_done[b] is not None:
                s_in.wait_event(ar_done[b])          # the collective of step i-2 read bx[b]
            for r, h in enumerate(host_in):
                bx[b][r].view(h.dtype).copy_(h, non_blocking=True)
            e_in = ev()
            e_in.record(s_in)
        cur.wait_event(e_in)
        if out_done[b] is not None:
            cur.wait_event(out_done[b])              # step i-2's download of by[b] finished
        call(bx[b], by[b])
        ar_done[b] = ev()
        ar_done[b].record(cur)
        with torch.cuda.stream(s_out):
            s_out.wait_event(ar_done[b])
            for r, t in enumerate(by[b]):
                hout[b][r].copy_(t.view(hout[b][r].dtype), non_blocking=True)
            out_done[b] = ev()
            out_done[b].record(s_out)

    for i in range(2):                                   # warm the streams and buffers
        step(i)
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True)
    z = torch.cuda.Event(enable_timing=True)
    a.record(cur)
    s_in.wait_stream(cur)
    for i in range(steps):
        step(i)
    cur.wait_stream(s_out)
    cur.wait_stream(s_in)
    z.record(cur)
    torch.cuda.synchronize()
    assert comm.get_async_error() == 0
    return a.elapsed_time(z) / steps


def complete_parity(dy, ys, dtype):
    """Bit mismatches of every output element of every rank (device tensors
    dy) against the oracle's outputs ys."""
    import numpy as np
    import torch
    bad = 0
    for y, e in zip(dy, ys):
        g = y.view(torch.int16).cpu().numpy().view(np.uint16) if dtype == "bf16" else y.cpu().numpy().view(np.uint32)
        bad += int(np.count_nonzero(g != (e.view(np.uint16) if dtype == "bf16" else e.view(np.uint32))))
    return {"complete": True, "elements_per_rank": int(dy[0].numel()), "ranks": len(dy), "mismatches": bad,
            "reference": "oracle.allreduce (strategy-order replay) on the same inputs, every element, bit-exact"}


# ---------------------------------------------------------------- our arm, N>1
def multi_complete_parity(comm, x, y, text, world, rank, count, dtype):
    """One fresh zero-copy AllReduce checked completely: rank 0 regenerates
    every rank's seeded input, replays the strategy with the oracle and
    compares its own output element by element; every other rank sends the
    SHA-256 of its whole output, which must equal the hash of the oracle's
    output for that rank (all outputs of an AllReduce are bitwise identical,
    but each rank is checked against its own expected bytes).  None on ranks > 0."""
    import hashlib

    import numpy as np
    import torch
    import torch.distributed as dist

    from synth import rank_tensors
    y.fill_(float("nan"))
    comm.collective_zc("allreduce", x, y, count)
    torch.cuda.synchronize()
    g = y.view(torch.int16).cpu().numpy().view(np.uint16) if dtype == "bf16" else y.cpu().numpy().view(np.uint32)
    got = [None] * world
    dist.all_gather_object(got, hashlib.sha256(g.tobytes()).hexdigest())
    if rank != 0:
        return None
    xs = [rank_tensors(dtype, count, 1, base=1000 + r)[0] for r in range(world)]
    ys, _ = oracle_replay(xs, text, world, dtype)
    e0 = ys[0].view(np.uint16) if dtype == "bf16" else ys[0].view(np.uint32)
    bad0 = int(np.count_nonzero(g != e0))
    bad_ranks = [q for q in range(1, world)
                 if got[q] != hashlib.sha256(ys[q].tobytes()).hexdigest()]
    return {"complete": True, "elements_per_rank": int(count), "ranks": world, "mismatches": bad0,
            "ranks_mismatched": ([0] if bad0 else []) + bad_ranks,
            "reference": "oracle.allreduce (strategy-order replay) of every rank's seeded input; rank 0 "
                         "element by element, ranks > 0 by SHA-256 of the whole output, bit-exact"}


PAPER_CONTEXT = {
    "claims": ["up to 2x communication speed-up vs NCCL (P:L7, P:L31, P:L319)",
               "up to 31% training throughput improvement vs NCCL (P:L7, P:L321)",
               "AllReduce 1.06x-1.29x vs NCCL / MSCCL (P:L291, P:L301)"],
    "hardware": "6 servers: 4 x (4 A100, NVLink, 100 Gbps RDMA) + 2 x (4 V100, NVLink, 50 Gbps), CUDA 11.3 (P:L279)",
    "note": "context only: a multi-server RDMA/TCP testbed with stragglers, not one NVSwitch node",
}
NCCL_LEGS = {"default": {}, "ring": {"NCCL_ALGO": "Ring"}, "tree": {"NCCL_ALGO": "Tree"},
             "nvls": {"NCCL_ALGO": "NVLS"}, "nvls_off": {"NCCL_NVLS_ENABLE": "0"}}


def p2p_ceiling(comm, world, rank, nbytes=64 << 20):
    """In-run NVLink ceiling (adapcc_link_probe, graph-captured): copy engine
    and TMA-store kernel, 1 -> 1 (every rank to its right neighbour at once, a
    permutation round) and 1 -> n-1 (rank 0 to everyone); seconds are the max
    over ranks; GB/s per direction of the sender."""
    import torch
    import torch.distributed as dist
    out = {}
    dev = "cpu" if dist.get_backend() == "gloo" else "cuda"
    for eng in ("sm", "ce"):
        t1 = comm.link_probe({(rank + 1) % world}, nbytes, engine=eng, iters=8)
        tf = comm.link_probe(set(range(1, world)) if rank == 0 else set(), nbytes, engine=eng, iters=4)
        t = torch.tensor([t1, tf], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t1, tf = float(t[0]), float(t[1])
        out[eng] = {"one_to_one_GBps": round(nbytes / t1 / 1e9, 1),
                    "one_to_all_GBps_per_dst": round(nbytes / tf / 1e9, 1),
                    "one_to_all_GBps_out": round((world - 1) * nbytes / tf / 1e9, 1)}
    out["bytes"] = nbytes
    return out


def run_nccl_leg(args):
    """One NCCL variant (environment set by the parent): busbw vs size for
    fp32 and bf16, max over ranks; rank 0 prints one JSON line."""
    import torch
    import torch.distributed as dist
    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    nbytes = int(args.size_mib * (1 << 20)) // 16 * 16
    buf = torch.randn(nbytes // 4, device="cuda")

    def reduce_max(v, op="max"):
        t = torch.tensor([v], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.MIN)
        return float(t.item())

    res = {}
    for dt, tdt, es in (("f32", torch.float32, 4), ("bf16", torch.bfloat16, 2)):
        pts = []
        z = buf.view(tdt)
        for sb in [b for b in SWEEP_SIZES if b <= nbytes]:
            zs = z[:sb // es]
            ms, _ = time_point(lambda: dist.all_reduce(zs), reduce_max, graph=False)
            pts.append({"bytes_per_rank": sb, "us": round(ms * 1e3, 2), "busbw": round(busbw(sb, ms / 1e3, world), 2)})
        res[dt] = pts
    if rank == 0:
        print(json.dumps({"nccl_leg": args.nccl_leg, "env": NCCL_LEGS[args.nccl_leg], "sweep": res,
                          "version": ".".join(map(str, torch.cuda.nccl.version()))}), flush=True)
    dist.destroy_process_group()
    return None


def leg_job(args, world, extra, env, name):
    """Rank 0, after the main run: one measurement as its own torchrun job of
    `world` ranks (fresh processes: NCCL reads its environment at start, and a
    failing leg cannot poison this process's CUDA context).  Returns the
    job's JSON line, or {"unavailable": why}."""
    e = dict(os.environ)
    for k in list(e):
        if k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "LOCAL_WORLD_SIZE", "MASTER_ADDR", "MASTER_PORT",
                 "GROUP_RANK", "GROUP_WORLD_SIZE", "ROLE_RANK", "ROLE_WORLD_SIZE", "ROLE_NAME") or \
                k.startswith("TORCHELASTIC_"):
            e.pop(k)
    e.update(env)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__),
           "--gpus", str(world), "--size-mib", str(args.size_mib), "--steps", str(args.steps),
           "--warmup", str(args.warmup), "--chunk-kib", str(args.chunk_kib), *extra]
    if args.test_same_gpu:
        cmd.append("--test-same-gpu")
    try:
        p = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600, env=e)
        lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
        if p.returncode == 0 and lines:
            return json.loads(lines[-1])
        tail = p.stderr.strip().splitlines()[-1] if p.stderr.strip() else ""
        return {"unavailable": f"{name}: rc={p.returncode}: {tail}"[:300]}
    except Exception as ex:  # noqa: BLE001
        return {"unavailable": f"{name}: {ex!r}"[:300]}


def nccl_legs(args, world):
    """Every NCCL variant as its own job (NCCL reads NCCL_ALGO / NCCL_NVLS_ENABLE when it starts)."""
    return {name: leg_job(args, world, ["--nccl-leg", name], env, name) for name, env in NCCL_LEGS.items()}


def run_nvls_leg(args):
    """NEXT-2 NVLS leg (its own job): the nvls strategy line -- copy in,
    multimem ld_reduce + st by the slice owners, copy out -- timed as the main
    leg (max over ranks), then checked: every rank's output must be the same
    bytes (SHA-256), and rank 0's output is within the any-order bound of the
    exact sum (reading R9: |y - sum| <= ((n-1) + 1) 2^-24 sum |x| for fp32) on
    a strided sample.  Rank 0 prints one JSON line; value None + reason when
    the box cannot build a multicast team."""
    import hashlib

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    from synth import rank_tensors
    rank, world, local = dist_env()
    dev = 0 if args.test_same_gpu else local
    torch.cuda.set_device(dev)
    if args.test_same_gpu:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    nbytes = int(args.size_mib * (1 << 20)) // 16 * 16
    count = nbytes // 4
    comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
    comm.config("timeout_ms", 30000)
    ok, why = comm.nvls_setup(2 * nbytes + (16 << 20))
    out = {"nvls_leg": True, "value": None, "reason": why or None, "unit": UNIT}
    if ok:
        comm.set_strategy("allreduce", G.allreduce_nvls(world, chunk=args.chunk_kib * 1024))
        xh = rank_tensors("f32", count, 1, base=1000 + rank)[0]
        x = torch.from_numpy(xh).cuda()
        y = torch.empty_like(x)
        for _ in range(args.warmup):
            comm.allreduce(x, y)
        dist.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(args.steps):
            comm.allreduce(x, y)
        b.record()
        torch.cuda.synchronize()
        dv = "cpu" if args.test_same_gpu else "cuda"
        t = torch.tensor([a.elapsed_time(b) / args.steps], dtype=torch.float64, device=dv)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        y.fill_(float("nan"))
        comm.allreduce(x, y)
        torch.cuda.synchronize()
        err = comm.get_async_error()
        g = y.cpu().numpy()
        hashes = [None] * world
        dist.all_gather_object(hashes, hashlib.sha256(g.tobytes()).hexdigest())
        out.update({"value": round(busbw(nbytes, ms / 1e3, world), 3), "ms_per_step": round(ms, 4),
                    "async_error": err, "path": "nvls line: multimem ld_reduce + st (STAGED copy in / out)"})
        if rank == 0:
            idx = np.unique(np.concatenate([np.arange(0, count, 4099), np.arange(max(0, count - 4096), count)]))
            xs = [rank_tensors("f32", count, 1, base=1000 + r)[0][idx].astype(np.float64) for r in range(world)]
            exact = np.sum(xs, axis=0)
            bound = world * 2.0 ** -24 * np.sum(np.abs(xs), axis=0)
            bad = int(np.count_nonzero(~(np.abs(g[idx].astype(np.float64) - exact) <= bound)))
            out["parity"] = {"complete": False, "sampled_elements": int(idx.size), "out_of_bound": bad,
                             "ranks_identical": len(set(hashes)) == 1,
                             "reference": "fp64 sum of every rank's seeded input (plain definition), "
                                          "any-order fp32 bound n 2^-24 sum|x| (reading R9)"}
    if rank == 0:
        print(json.dumps(out), flush=True)
    comm.finalize()
    dist.destroy_process_group()
    return None


def run_multi(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    from synth import rank_tensors

    rank, world, local = dist_env()
    if args.test_same_gpu:
        local = 0
        torch.cuda.set_device(0)
        dist.init_process_group("gloo")
    else:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    es = 4 if args.dtype == "f32" else 2
    nbytes = int(args.size_mib * (1 << 20)) // 16 * 16
    count = nbytes // es
    tdt = torch.float32 if args.dtype == "f32" else torch.bfloat16
    text = G.allreduce_stars(world, chunk=args.chunk_kib * 1024)
    comm = pkg.Communicator.init(scratch_bytes=max(1 << 30, 2 * nbytes + (64 << 20)), device=local)
    comm.set_strategy("allreduce", text)
    xh = torch.from_numpy(rank_tensors(args.dtype, count, 1, base=1000 + rank)[0])
    if args.dtype == "bf16":
        xh = xh.view(torch.int16)
    xh = xh.pin_memory()
    x = xh.cuda().view(tdt)
    y = torch.empty_like(x)
    stream = torch.cuda.current_stream()
    # zero-copy: x / y registered once (CUDA IPC), DIRECT plan over NVLink
    comm.register(x)
    comm.register(y)
    probes = p2p_ceiling(comm, world, rank)

    def timed(fn, steps):
        dist.barrier()
        torch.cuda.synchronize()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(steps):
            fn()
        b.record(stream)
        torch.cuda.synchronize()
        t = torch.tensor([a.elapsed_time(b) / steps], device="cpu" if args.test_same_gpu else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.barrier()
        return float(t.item())

    def ours():
        comm.collective_zc("allreduce", x, y, count)

    def ours_staged():
        comm.allreduce(x, y)

    z = x.clone()

    def nccl():
        if not args.test_same_gpu:
            dist.all_reduce(z)

    for _ in range(args.warmup):
        ours()
        ours_staged()
        nccl()
    torch.cuda.synchronize()
    l0 = comm.launch_count()
    with ClockSampler(local) as clk:
        ms = timed(ours, args.steps)
    launches = comm.launch_count() - l0
    ms_nccl = timed(nccl, args.steps)
    ms_staged = timed(ours_staged, args.steps)
    err = comm.get_async_error()

    # end to end (same pipelining as N=1): per rank H2D of its input, the
    # zero-copy collective, D2H of its output; the per-step time is the max
    # over ranks.  The second buffer pair is registered too.
    x2, y2 = torch.empty_like(x), torch.empty_like(y)
    comm.register(x2)
    comm.register(y2)

    def zc_call(xs, ys):
        comm.collective_zc("allreduce", xs[0], ys[0], count)

    dist.barrier()
    e2e_local = e2e_pipelined(comm, [xh], [x], [y], args.e2e_steps, tdt, zc_call, second=([x2], [y2]))
    t = torch.tensor([e2e_local], device="cpu" if args.test_same_gpu else "cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    e2e_t = float(t.item())
    value = busbw(nbytes, ms / 1e3, world)

    def reduce_max(v, op="max"):
        t = torch.tensor([v], dtype=torch.float64, device="cpu" if args.test_same_gpu else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.MIN)
        return float(t.item())

    sweep = None
    if not args.no_sweep:   # busbw vs size, ours (zero-copy) and NCCL on the same buffers, max over ranks
        sweep = {}
        # fp32 and bf16 (C2): the other dtype reuses the registered bytes (timing only)
        for sdt in [args.dtype] + [d for d in ("f32", "bf16") if d != args.dtype]:
            sdt_t = torch.float32 if sdt == "f32" else torch.bfloat16
            ses = 4 if sdt == "f32" else 2
            xv, yv, zv = x.view(sdt_t), y.view(sdt_t), z.view(sdt_t)
            pts = []
            for sb in [b for b in SWEEP_SIZES if b <= nbytes]:
                c = sb // ses
                xs_, ys_, zs_ = xv[:c], yv[:c], zv[:c]
                call = comm.prepare_collective_zc("allreduce", xs_, ys_, c)
                ms_, msg_ = time_point(call, reduce_max,
                                       fn_graph=lambda: comm.collective_zc("allreduce", xs_, ys_, c))
                pt = {"bytes_per_rank": sb, "us": round(ms_ * 1e3, 2), "us_graph": round(msg_ * 1e3, 2),
                      "busbw": round(busbw(sb, ms_ / 1e3, world), 2),
                      "busbw_graph": round(busbw(sb, msg_ / 1e3, world), 2)}
                if not args.test_same_gpu:
                    nms, _ = time_point(lambda: dist.all_reduce(zs_), reduce_max, graph=False)
                    pt.update({"nccl_us": round(nms * 1e3, 2), "nccl_busbw": round(busbw(sb, nms / 1e3, world), 2)})
                pts.append(pt)
            sweep[sdt] = pts
    parity = None if args.no_parity else multi_complete_parity(comm, x, y, text, world, rank, count, args.dtype)
    st = pkg.adapcc.plan_stats(text, count, args.dtype, (1 << world) - 1, rank=rank)
    peak_dir = probes["sm"]["one_to_one_GBps"]
    dir_bytes = st["remote_bytes"]   # = bytes crossing each link direction of this GPU (symmetric plan)
    res = None
    if rank == 0:
        res = {
            "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": args.dtype,
            "data": "synthetic (seeded N(0,1), synth/inputs.py)",
            "config": workload_config(args, world, world),
            "algbw": round(nbytes / (ms / 1e3) / 1e9, 3),
            "pct_of_nvlink_900": round(100 * value / NVLINK_NOMINAL, 2),
            "roofline": {"bound": "nvlink" if not args.test_same_gpu else "hbm (all ranks on one GPU)",
                         "achieved": round(dir_bytes / (ms / 1e3) / 1e9, 1), "peak": peak_dir,
                         "unit": "GB/s", "frac": round(dir_bytes / (ms / 1e3) / 1e9 / peak_dir, 4), "traffic": None,
                         "peak_source": "measured in this run: TMA-store probe 1 -> 1 per direction "
                                        "(adapcc_link_probe, max over ranks); 900 nominal",
                         "algorithmic_bytes_per_direction": dir_bytes,
                         "why": "zero-copy star plan, per GPU g: g's kernel pulls (n-1)/n S (its trees' "
                                "inputs) and pushes (n-1)/n S (their results), while peers pull g's "
                                "slices and push their results into g: 2(n-1)/n S in each direction, the "
                                "plan's remote bytes of g (loads + stores) by symmetry"},
            "e2e": {"value": round(busbw(nbytes, e2e_t / 1e3, world), 3), "unit": UNIT,
                    "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes,
                    "ms_per_step": round(e2e_t, 3), "steps": args.e2e_steps,
                    "how": "per rank: pinned H2D of its input + collective_zc + D2H of its output; steps "
                           "double-buffered (both pairs registered), copies on separate streams; max over ranks"},
            "gpu_launches": launches, "clocks": clk.summary(), "async_error": err, "parity": parity,
            "sweep": sweep,
            "sweep_how": "every x4 size up to the bench size, slices of the registered buffers; ours = "
                         "zero-copy AllReduce, nccl = dist.all_reduce on the same sizes; back-to-back "
                         "enqueue (us; NCCL likewise) and, ours only, a CUDA graph (us_graph); max over ranks",
            "path": "zero-copy DIRECT plan over CUDA IPC (registered buffers)",
            "p2p_ceiling": probes, "nvls": None, "paper_context": PAPER_CONTEXT,
            "staged": {"value": round(busbw(nbytes, ms_staged / 1e3, world), 3), "unit": UNIT,
                       "ms_per_step": round(ms_staged, 4),
                       "path": "STAGED protocol (landing + broadcast slots in IPC arenas)"},
            "nccl": None if args.test_same_gpu else {"value": round(busbw(nbytes, ms_nccl / 1e3, world), 3), "unit": UNIT,
                     "ms_per_step": round(ms_nccl, 4), "version": ".".join(map(str, torch.cuda.nccl.version()))},
        }
    comm.finalize()
    dist.destroy_process_group()
    if rank == 0:
        del x, y, z, x2, y2
        torch.cuda.empty_cache()
        # NVLS (NEXT-2) in its own job: the multimem path has not run on a multicast-capable box
        # before, so a failure there cannot take this line with it
        res["nvls"] = leg_job(args, world, ["--nvls-leg"], {}, "nvls")
        if not args.test_same_gpu and not args.no_nccl_legs:
            res["nccl_legs"] = nccl_legs(args, world)
    return res


def free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def self_launch(args):
    """--gpus N without a launcher: re-run this script as N ranks under
    torch.distributed.run (one process per GPU, 127.0.0.1 rendezvous).
    Without N visible GPUs it fails loudly unless --test-same-gpu is given
    (then all N ranks share cuda:0 and the numbers are not NVLink numbers)."""
    if not args.test_same_gpu:
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            print(f"bench.py: --gpus {args.gpus} needs {args.gpus} visible GPUs, found {have} "
                  f"(use --test-same-gpu to run the N-rank code path on one GPU)", file=sys.stderr)
            return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.run(cmd, cwd=ROOT).returncode


def main():
    args = parse_args()
    _, world, _ = dist_env()
    if args.gpus < 1:
        print("bench.py: --gpus must be >= 1", file=sys.stderr)
        return 2
    if "WORLD_SIZE" in os.environ and world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        return 2
    if args.nccl_leg:
        out = run_nccl_leg(args)
    elif args.nvls_leg:
        out = run_nvls_leg(args)
    elif args.impl == "reference":
        out = run_reference(args)        # CPU only: no launcher needed, rank 0 prints
    elif args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)
    elif world > 1:
        out = run_multi(args)
    else:
        out = run_single(args)
    if out is not None:
        print(json.dumps(out), flush=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())
