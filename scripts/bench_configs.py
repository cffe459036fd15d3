"""Measure every BASELINE.json config on one B200 (loopback virtual ranks).

    python scripts/bench_configs.py [--out gpurun_out/configs.json]

C1  AllReduce fp32 1 Mi elements, 2 ranks, single tree, chunk 256 KiB (DIRECT and STAGED)
C2  AllReduce 8 ranks at 256 MiB: fp32 and bf16, M = 1/2/4/8 star trees, double binary, ring
C3  partial AllReduce, 8 ranks, stragglers {3,6}: T_adapcc = end of phase 2 (phase 1 among the
    ready ranks at t=0 with relays, phase 2 ACCUMULATE once the stragglers are ready) vs
    T_wait = t_s + T_full, straggler lag t_s simulated by a 1-CTA spin kernel on a compute stream
C4  AlltoAll 8 ranks, [8][512][4096] bf16 per rank
C4v AlltoAllv MoE dispatch, 8 ranks x 4096 tokens x 4096 bf16, Zipf(a) top-1 routing, a in {0, 1.2, 2}
C5  AllGather of GPT-2-XL row shards, 48 layers x 4 weights, strategy swap at call 96
G1  local chunk reduction: Reduce of k in {2, 8} virtual 1 GiB inputs into one
    1 GiB output (one star tree rooted at 0), fp32 and bf16; GB/s = (k+1) S / t vs the HBM peak
Timing: CUDA events on the launching stream, warm-up first; busbw factors as nccl-tests.
Every config also checks parity on sampled outputs against the oracle.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "configs.json"))
    ap.add_argument("--only", default="C1,C2,C3,C4,C4v,C5,G1")
    a = ap.parse_args()

    import numpy as np
    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from oracle import collectives as oc
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    from synth import GPT2XL_LAYERS, rank_tensors

    def dev(x, dtype):
        t = torch.from_numpy(x)
        return t.view(torch.int16).cuda().view(torch.bfloat16) if dtype == "bf16" else t.cuda()

    def host_bits(t, dtype):
        return t.view(torch.int16).cpu().numpy().view(np.uint16) if dtype == "bf16" else \
            t.cpu().numpy().view(np.uint32)

    def timeit(fn, iters=20, warm=3):
        for _ in range(warm):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(iters):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / iters

    def timeit_graph(fn, iters=100, reps=5):
        """Device time per call with the host out of the loop (CUDA graph of
        `iters` back-to-back calls), SURVEY §8(d) d-5."""
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            fn()
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                for _ in range(iters):
                    fn()
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            g.replay()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / (iters * reps)

    def sampled_ok(ys, xs, text, R, count, dtype, k=2048):
        idx = np.unique(np.random.default_rng(5).integers(0, count, size=k))
        exp = oc.allreduce_elements([x[idx] if x is not None else None for x in xs], idx, count, text, R, dtype)
        eb = exp.view(np.uint16) if dtype == "bf16" else exp.view(np.uint32)
        ti = torch.from_numpy(idx).cuda()
        return all(np.array_equal(host_bits(y.index_select(0, ti), dtype), eb) for y in ys)

    out = {"gpu": torch.cuda.get_device_name(0), "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())}
    only = set(a.only.split(","))

    # ------------------------------------------------------------------ C1
    if "C1" in only:
        res = []
        n, count = 2, 1 << 20
        text = G.allreduce_trees([[-1, 0]], chunk=262144)
        xs = rank_tensors("f32", count, n)
        for mode in ("direct", "staged"):
            comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=64 << 20)
            comm.set_strategy("allreduce", text)
            dx = [dev(x, "f32") for x in xs]
            dy = [torch.empty_like(t) for t in dx]
            ms = timeit(lambda: comm.allreduce_lb(dx, dy), iters=200)
            ms_g = timeit_graph(lambda: comm.allreduce_lb(dx, dy))
            exp = oc.allreduce(xs, text, {0, 1}, "f32")
            ok = all(np.array_equal(host_bits(dy[g], "f32"), exp[g].view(np.uint32)) for g in range(n))
            res.append({"mode": mode, "us": round(ms * 1e3, 2), "busbw": round(count * 4 / ms / 1e6 * 1.0, 2),
                        "us_graph": round(ms_g * 1e3, 2), "busbw_graph": round(count * 4 / ms_g / 1e6, 2),
                        "parity_bit_exact": ok, "kernel": comm.last_engine()})
            comm.finalize()
        out["C1"] = res
        print("C1", res, flush=True)

    # ------------------------------------------------------------------ C2
    if "C2" in only:
        res = []
        n, nbytes = 8, 256 << 20
        comm = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=512 << 20)
        for dtype in ("f32", "bf16"):
            es = 4 if dtype == "f32" else 2
            count = nbytes // es
            xs = rank_tensors(dtype, count, n)
            dx = [dev(x, dtype) for x in xs]
            dy = [torch.empty_like(t) for t in dx]
            strategies = {f"star M={m}": G.allreduce_stars(n, roots=list(range(m))) for m in (1, 2, 4, 8)}
            strategies["double binary"] = G.allreduce_double_binary(n)
            strategies["ring"] = G.allreduce_ring(n)
            for name, text in strategies.items():
                if dtype == "bf16" and name not in ("star M=8",):
                    continue
                comm.set_strategy("allreduce", text)
                ms = timeit(lambda: comm.allreduce_lb(dx, dy), iters=10)
                bus = nbytes / ms / 1e6 * 2 * (n - 1) / n
                ok = sampled_ok(dy, xs, text, set(range(n)), count, dtype)
                res.append({"dtype": dtype, "strategy": name, "ms": round(ms, 4), "busbw": round(bus, 1),
                            "hbm_frac": round(2 * n * nbytes / ms / 1e6 / 6545.6, 4), "parity": ok,
                            "kernel": comm.last_engine()})
                print("C2", res[-1], flush=True)
            del dx, dy
        comm.finalize()
        out["C2"] = res

    # ------------------------------------------------------------------ C3
    if "C3" in only:
        res = []
        n = 8
        R1, R2 = {0, 1, 2, 4, 5, 7}, {3, 6}
        comm = pkg.Communicator.loopback(n, mode="staged", scratch_bytes=(2 * 100 << 20) + (64 << 20))
        s_comm = torch.cuda.Stream()
        s_comp = torch.cuda.Stream()
        # cycles per ms of the spin kernel
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.cuda._sleep(10_000_000)
        e1.record()
        torch.cuda.synchronize()
        cyc_per_ms = 10_000_000 / e0.elapsed_time(e1)
        for mib in (25, 50, 100):
            count = (mib << 20) // 4
            xs = rank_tensors("f32", count, n)
            dx = [dev(x, "f32") for x in xs]
            dy = [torch.empty_like(t) for t in dx]
            t_full_txt = G.allreduce_stars(n)
            variants = {
                "relays as roots (mask-aware weights)": (G.allreduce_mask_aware_stars(n, R1),
                                                         G.allreduce_mask_aware_stars(n, R2)),
                "paper-faithful (unweighted stars, relays per tuples)": (G.allreduce_stars(n), G.allreduce_stars(n)),
                "relays as leaves only": (G.allreduce_mask_aware_stars(n, R1, relays_as_roots=False),
                                          G.allreduce_mask_aware_stars(n, R2, relays_as_roots=False)),
            }
            comm.set_strategy("allreduce", t_full_txt)
            t_full = timeit(lambda: comm.allreduce_lb(dx, dy), iters=10)
            point = {"mib": mib, "T_full_ms": round(t_full, 4), "variants": {}}
            for vname, (t1, t2) in variants.items():
                comm.set_strategy("allreduce", t1)
                p1 = timeit(lambda: comm.allreduce_lb([x if r in R1 else None for r, x in enumerate(dx)], dy,
                                                      ready=R1), iters=10)
                comm.set_strategy("allreduce", t2)
                p2 = timeit(lambda: comm.allreduce_lb([x if r in R2 else None for r, x in enumerate(dx)], dy,
                                                      ready=R2, accumulate=True), iters=10)
                lags = {}
                for f in (0.0, 0.25, 0.5, 1.0, 2.0):
                    ts = f * t_full
                    # measured end-to-end: spin kernel (straggler compute) on s_comp, phase 1 on
                    # s_comm at t=0, phase 2 on s_comm after the straggler's event
                    torch.cuda.synchronize()
                    a0 = torch.cuda.Event(enable_timing=True)
                    a1 = torch.cuda.Event(enable_timing=True)
                    ready_ev = torch.cuda.Event()
                    a0.record(s_comm)
                    s_comp.wait_event(a0)
                    with torch.cuda.stream(s_comp):
                        if ts > 0:
                            torch.cuda._sleep(int(ts * cyc_per_ms))
                        ready_ev.record(s_comp)
                    with torch.cuda.stream(s_comm):
                        comm.set_strategy("allreduce", t1)
                        comm.allreduce_lb([x if r in R1 else None for r, x in enumerate(dx)], dy, ready=R1)
                        s_comm.wait_event(ready_ev)
                        comm.set_strategy("allreduce", t2)
                        comm.allreduce_lb([x if r in R2 else None for r, x in enumerate(dx)], dy, ready=R2,
                                          accumulate=True)
                        a1.record(s_comm)
                    torch.cuda.synchronize()
                    t_adapcc = a0.elapsed_time(a1)
                    t_wait = ts + t_full
                    lags[str(f)] = {"t_s_ms": round(ts, 4), "T_adapcc_ms": round(t_adapcc, 4),
                                    "T_wait_ms": round(t_wait, 4), "speedup": round(t_wait / t_adapcc, 3)}
                full = oc.allreduce_exact([x[:4096] for x in xs], set(range(n)), "f32")
                got = dy[0][:4096].cpu().numpy().astype(np.float64)
                point["variants"][vname] = {"phase1_ms": round(p1, 4), "phase2_ms": round(p2, 4),
                                            "lags": lags,
                                            "rel_err_vs_full_sum": float(np.max(np.abs(got - full)) /
                                                                         np.max(np.abs(full)))}
            # Per-piece late join (NEXT-1) on the DIRECT plan: phase 1 starts at t = 0 with the
            # stragglers as late candidates; their compute stream signals them ready after the lag, so
            # every piece claimed after that folds them in; phase 2 (LATE_COMPLEMENT) adds them only to
            # the pieces that had already passed.  T_wait uses the DIRECT plan's own T_full.
            dcomm = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
            dcomm.set_strategy("allreduce", G.allreduce_stars(n))
            t_full_d = timeit(lambda: dcomm.allreduce_lb(dx, dy), iters=10)
            for _ in range(2):  # warm the LATE_JOIN plan (phase 2 runs on the same plan)
                dcomm.allreduce_lb(dx, dy, ready=R1, late="join")
                dcomm.allreduce_lb(dx, dy, ready=R1, late="complement")
            torch.cuda.synchronize()
            lags = {}
            for f in (0.0, 0.25, 0.5, 1.0, 2.0):
                ts = f * t_full_d
                reps = []
                for _ in range(7):  # the inclusion point races the straggler's signal: median of 7
                    torch.cuda.synchronize()
                    a0 = torch.cuda.Event(enable_timing=True)
                    a1 = torch.cuda.Event(enable_timing=True)
                    ready_ev = torch.cuda.Event()
                    ticket = dcomm.late_ticket() + 1
                    a0.record(s_comm)
                    s_comp.wait_event(a0)
                    with torch.cuda.stream(s_comp):
                        if ts > 0:
                            torch.cuda._sleep(int(ts * cyc_per_ms))
                        for r in sorted(R2):
                            dcomm.signal_ready(rank=r, ticket=ticket, stream=s_comp)
                        ready_ev.record(s_comp)
                    with torch.cuda.stream(s_comm):
                        dcomm.allreduce_lb(dx, dy, ready=R1, late="join")
                        s_comm.wait_event(ready_ev)
                        dcomm.allreduce_lb(dx, dy, ready=R1, late="complement")
                        a1.record(s_comm)
                    torch.cuda.synchronize()
                    reps.append(a0.elapsed_time(a1))
                t_adapcc = sorted(reps)[len(reps) // 2]
                t_wait = ts + t_full_d
                lags[str(f)] = {"t_s_ms": round(ts, 4), "T_adapcc_ms": round(t_adapcc, 4),
                                "T_wait_ms": round(t_wait, 4), "speedup": round(t_wait / t_adapcc, 3)}
            assert dcomm.get_async_error() == 0
            full = oc.allreduce_exact([x[:4096] for x in xs], set(range(n)), "f32")
            got = dy[0][:4096].cpu().numpy().astype(np.float64)
            point["variants"]["late join per piece (DIRECT, NEXT-1)"] = {
                "T_full_direct_ms": round(t_full_d, 4), "lags": lags,
                "rel_err_vs_full_sum": float(np.max(np.abs(got - full)) / np.max(np.abs(full)))}
            dcomm.finalize()
            res.append(point)
            print("C3", json.dumps(point)[:400], flush=True)
            del dx, dy
        comm.finalize()
        out["C3"] = res

    # ------------------------------------------------------------------ C4
    if "C4" in only:
        res = []
        n, cnt = 8, 512 * 4096
        text = G.alltoall_direct(n, chunk=1 << 20)
        xs = rank_tensors("bf16", n * cnt, n, base=2000)
        for mode in ("direct", "staged"):
            comm = pkg.Communicator.loopback(n, mode=mode, scratch_bytes=(2 * n * cnt * 2 + (64 << 20)))
            comm.set_strategy("alltoall", text)
            dx = [dev(x, "bf16") for x in xs]
            dy = [torch.empty_like(t) for t in dx]
            ms = timeit(lambda: comm.alltoall_lb(dx, dy), iters=20)
            nbytes = n * cnt * 2
            exp = oc.alltoall(xs, text, set(range(n)), "bf16", [np.zeros(n * cnt, np.uint16)] * n)
            ok = all(np.array_equal(host_bits(dy[d], "bf16"), exp[d]) for d in range(n))
            res.append({"mode": mode, "ms": round(ms, 4),
                        "busbw": round(nbytes / ms / 1e6 * (n - 1) / n, 1),
                        "hbm_frac": round(2 * n * nbytes / ms / 1e6 / 6545.6, 4), "parity": ok,
                        "kernel": comm.last_engine()})
            print("C4", res[-1], flush=True)
            comm.finalize()
        out["C4"] = res

    # ------------------------------------------------------------------ C4v
    # AlltoAllv MoE dispatch (NEXT-4): 8 ranks x 4096 tokens x hidden 4096 bf16 per rank, top-1
    # routing with Zipf(a) expert popularity (a = 0: uniform), DIRECT plan; algorithmic bytes =
    # every token read once and written once; busbw counts the tokens that leave their rank.
    if "C4v" in only:
        from synth.inputs import moe_counts
        res = []
        n, tok, hid = 8, 4096, 4096
        text = G.alltoall_direct(n, chunk=1 << 20)
        for a_zipf in (0.0, 1.2, 2.0):
            counts = moe_counts(n, tok, hid, zipf_a=a_zipf)
            send = [sum(counts[s]) for s in range(n)]
            recv = [sum(counts[s][d] for s in range(n)) for d in range(n)]
            xs = [rank_tensors("bf16", send[s], 1, base=2200 + s)[0] for s in range(n)]
            comm = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
            comm.set_strategy("alltoall", text)
            dx = [dev(x, "bf16") for x in xs]
            dy = [torch.empty(recv[d], dtype=torch.bfloat16, device="cuda") for d in range(n)]
            ms = timeit_graph(lambda: comm.alltoallv_lb(dx, dy, counts))
            prev = [np.zeros(recv[d], np.uint16) for d in range(n)]
            exp = oc.alltoallv(xs, counts, text, set(range(n)), "bf16", prev)
            comm.alltoallv_lb(dx, dy, counts)
            torch.cuda.synchronize()
            ok = all(np.array_equal(host_bits(dy[d], "bf16"), exp[d]) for d in range(n))
            moved = sum(counts[s][d] for s in range(n) for d in range(n) if s != d) * 2
            total = sum(send) * 2
            res.append({"zipf_a": a_zipf, "max_recv_tokens": max(recv) // hid, "min_recv_tokens": min(recv) // hid,
                        "ms_graph": round(ms, 4), "busbw_per_rank": round(moved / n / ms / 1e6, 1),
                        "hbm_frac": round(2 * total / ms / 1e6 / 6545.6, 4), "parity": ok,
                        "kernel": comm.last_engine()})
            print("C4v", res[-1], flush=True)
            comm.finalize()
        out["C4v"] = res

    # ------------------------------------------------------------------ C5
    if "C5" in only:
        res = []
        for n in (2, 4, 8):
            comm = pkg.Communicator.loopback(n, mode="staged", scratch_bytes=256 << 20)
            t_a, t_b = G.allgather_stars(n, chunk=262144), G.allgather_chains(n, chunk=1 << 20)
            shards = {}
            for wi, (name, rows, cols) in enumerate(GPT2XL_LAYERS):
                cnt = rows // n * cols
                xs = rank_tensors("bf16", cnt, n, base=3000 + wi)
                shards[name] = ([dev(x, "bf16") for x in xs],
                                [torch.empty(n * cnt, dtype=torch.bfloat16, device="cuda") for _ in range(n)],
                                xs)
            comm.set_strategy("allgather", t_a)
            for name in shards:   # warm plans of strategy A
                comm.allgather_lb(shards[name][0], shards[name][1])
            torch.cuda.synchronize()
            evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(192)]
            swap_host_ms = None
            for call in range(192):
                name = GPT2XL_LAYERS[call % 4][0]
                if call == 96:
                    h0 = time.perf_counter()
                    comm.set_strategy("allgather", t_b)
                    swap_host_ms = (time.perf_counter() - h0) * 1e3
                evs[call][0].record()
                comm.allgather_lb(shards[name][0], shards[name][1])
                evs[call][1].record()
            torch.cuda.synchronize()
            t = [s.elapsed_time(e) for s, e in evs]
            bus = []
            for call in range(192):
                name = GPT2XL_LAYERS[call % 4][0]
                out_bytes = shards[name][1][0].numel() * 2
                bus.append(out_bytes / t[call] / 1e6 * (n - 1) / n)
            ok = True
            for name, (_, dy, xs) in shards.items():
                cat = np.concatenate(xs)
                ok &= all(np.array_equal(host_bits(y, "bf16"), cat) for y in dy)
            res.append({"n": n, "busbw_median_A": round(float(np.median(bus[:96])), 1),
                        "busbw_median_B": round(float(np.median(bus[97:])), 1),
                        "call_ms_median_A": round(float(np.median(t[:96])), 4),
                        "call_ms_median_B": round(float(np.median(t[97:])), 4),
                        "first_call_after_swap_ms": round(t[96], 4),
                        "set_strategy_host_ms": round(swap_host_ms, 4), "parity": bool(ok)})
            print("C5", res[-1], flush=True)
            comm.finalize()
        out["C5"] = res

    # ------------------------------------------------------------------ G1
    if "G1" in only:
        res = []
        pk = os.path.join(ROOT, "MEASURED_PEAKS.json")
        peak = json.load(open(pk))["hbm_gbs"] if os.path.exists(pk) else 6650.0
        nbytes = 1 << 30
        for dtype in ("f32", "bf16"):
            es = 4 if dtype == "f32" else 2
            count = nbytes // es
            tdt = torch.float32 if dtype == "f32" else torch.bfloat16
            for k in (2, 8):
                comm = pkg.Communicator.loopback(k, mode="direct", scratch_bytes=64 << 20)
                text = G.reduce_trees([G.star_parent(k, 0)], chunk=1 << 20)
                comm.set_strategy("reduce", text)
                g = torch.Generator(device="cuda").manual_seed(7)
                dx = [torch.randn(count, device="cuda", generator=g).to(tdt) for _ in range(k)]
                dy = [torch.empty(count, device="cuda", dtype=tdt)] + [None] * (k - 1)
                ms = timeit(lambda: comm.reduce_lb(dx, dy, root=0), iters=10)
                gbs = (k + 1) * nbytes / ms / 1e6
                # parity: the single star's fold order (root's own input, then 1..k-1) at sampled indices
                idx = np.unique(np.random.default_rng(5).integers(0, count, size=2048))
                ti = torch.from_numpy(idx).cuda()
                vals = [host_bits(x.index_select(0, ti), dtype) for x in dx]
                vals = [v.view(np.float32) if dtype == "f32" else v for v in vals]
                exp = oc.allreduce_elements(vals, idx, count, G.allreduce_trees([G.star_parent(k, 0)]),
                                            set(range(k)), dtype)
                eb = exp.view(np.uint16) if dtype == "bf16" else exp.view(np.uint32)
                ok = bool(np.array_equal(host_bits(dy[0].index_select(0, ti), dtype), eb))
                res.append({"dtype": dtype, "k": k, "ms": round(ms, 4), "gbs": round(gbs, 1),
                            "hbm_frac": round(gbs / peak, 4), "parity": ok, "kernel": comm.last_engine()})
                print("G1", res[-1], flush=True)
                del dx, dy
                comm.finalize()
                torch.cuda.empty_cache()
        out["G1"] = res

    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__" and "--links" not in sys.argv:
    main()


def profile_links(out_path=None):
    """NEXT-2 on one GPU: the paper's alpha-beta probes applied to the
    engine's own copy path (2 virtual ranks, Broadcast = one K=1 copy) and to a
    plain device copy, then the cost model's chunk choice for NVLink numbers."""
    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import costmodel as CM
    from paper_conf_icdcs_zhaozw24_b200 import generator as G

    comm = pkg.Communicator.loopback(2, mode="direct", scratch_bytes=64 << 20)
    bufs = {}

    def engine_copy(nbytes):
        cnt = nbytes // 4
        if cnt not in bufs:
            bufs[cnt] = ([torch.ones(cnt, device="cuda")] * 2, [torch.empty(cnt, device="cuda") for _ in range(2)])
        xs, ys = bufs[cnt]
        comm.broadcast_lb(xs, ys, 0)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        comm.broadcast_lb(xs, ys, 0)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e-3

    def torch_copy(nbytes):
        a = torch.ones(nbytes // 4, device="cuda")
        b = torch.empty_like(a)
        b.copy_(a)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        b.copy_(a)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e-3

    res = {}
    for name, fn in (("engine_copy", engine_copy), ("torch_copy", torch_copy)):
        a, b, samples = CM.probe_link(fn, sizes=(1 << 16, 1 << 22), repeats=(1, 8))
        res[name] = {"alpha_us": round(a * 1e6, 3), "beta_GBps": round(1 / b / 1e9, 1) if b > 0 else None,
                     "note": "one GPU: 'link' = HBM read+write of the copy"}
    n = 8
    alpha, beta = CM.uniform_links(n, 3e-6, 1 / 770e9)
    best, scored = CM.best_chunk(lambda c: G.allreduce_stars(n, chunk=c), 256 << 20, alpha, beta)
    res["nvlink_model_256MiB_8ranks"] = {"alpha_us": 3.0, "link_GBps": 770,
                                         "best_chunk": best,
                                         "predicted_ms": {str(c): round(t * 1e3, 4) for t, c in scored}}
    comm.finalize()
    print("LINKS", json.dumps(res), flush=True)
    return res


if __name__ == "__main__" and "--links" in sys.argv:
    r = profile_links()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(r, open(os.path.join(ROOT, "gpurun_out", "links.json"), "w"), indent=1)
