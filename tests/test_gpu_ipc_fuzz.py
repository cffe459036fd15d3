"""Randomised parity sweep of the multi-process paths (-m gpu): 3 processes on
one GPU (CUDA IPC, gloo bootstrap), the seeded cases of test_gpu_fuzz.py with
n = 3 (kernels, LDG schedules, PDL and piece sizes included), each run through
the STAGED protocol and through the zero-copy DIRECT plan on registered
buffers; every process checks its own output bit-exactly.
ADAPCC_IPC_FUZZ_CASES sets the number of cases (default 240)."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
N = 3
CASES = int(os.environ.get("ADAPCC_IPC_FUZZ_CASES", "240"))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        import paper_conf_icdcs_zhaozw24_b200 as pkg
        from oracle import collectives as oc
        from synth import rank_tensors
        from tests.gpu_util import bits, to_dev, to_host
        from tests.test_gpu_fuzz import _case

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=N)
        dev = rank % torch.cuda.device_count()  # one GPU per rank when the box has them
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=256 << 20, device=dev)
        comm.config("timeout_ms", 60000)
        cap = 3 * (1 << 20) * N + 64
        bx = torch.zeros(cap, dtype=torch.int32, device="cuda")
        by = torch.zeros(cap, dtype=torch.int32, device="cuda")
        comm.register(bx)
        comm.register(by)
        tdt = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32}
        bad = []
        for seed in range(CASES):
            c = _case(seed, large=seed % 4 == 0, n=N)
            dtype, R, text, coll = c["dtype"], c["ready"], c["text"], c["coll"]
            count = min(c["count"], (1 << 20))
            per_rank = count * (N if coll in ("alltoall", "reducescatter") else 1)
            out_per_rank = count * (N if coll in ("alltoall", "allgather") else 1)
            xs = rank_tensors(dtype, per_rank, N, base=5000 + seed)
            prev = [rank_tensors(dtype, out_per_rank, 1, base=6000 + 7 * seed + g)[0] for g in range(N)]
            acc = coll == "allreduce" and seed % 3 == 0
            if coll == "allreduce":
                exp = oc.allreduce(xs, text, R, dtype, accumulate=acc, y_prev=prev)[rank]
            elif coll == "allgather":
                exp = oc.allgather(xs, text, R, dtype, prev)[rank]
            elif coll == "alltoall":
                exp = oc.alltoall(xs, text, R, dtype, prev)[rank]
            else:
                exp = oc.reducescatter(xs, text, R, dtype, y_prev=prev)[rank]
            comm.set_strategy(coll, text)
            comm.config("engine", c["engine"])
            for k in ("sched", "pdl", "piece_kib"):  # same seeded launch knobs on every rank
                comm.config(k, c[k])
            for path in ("staged", "zc"):
                if path == "staged":
                    x = to_dev(xs[rank], dtype)
                    y = to_dev(prev[rank], dtype)
                    if coll == "allreduce":
                        comm.allreduce(x, y, ready=R, accumulate=acc)
                    elif coll == "allgather":
                        comm.allgather(x, y, ready=R)
                    elif coll == "alltoall":
                        comm.alltoall(x, y, ready=R)
                    else:
                        comm.reducescatter(x, y, ready=R)
                else:
                    es = 2 if dtype == "bf16" else 4
                    x = bx.view(torch.uint8)[:per_rank * es].view(tdt[dtype])
                    y = by.view(torch.uint8)[:out_per_rank * es].view(tdt[dtype])
                    x.copy_(to_dev(xs[rank], dtype))
                    y.copy_(to_dev(prev[rank], dtype))
                    dist.barrier()   # every rank's inputs are in place before peers read them
                    torch.cuda.synchronize()
                    comm.collective_zc(coll, x, y, count, ready=R, accumulate=acc)
                torch.cuda.synchronize()
                if not np.array_equal(bits(to_host(y, dtype)), bits(exp)):
                    bad.append((seed, path, {k: v for k, v in c.items() if k != "text"}))
                if path == "zc":
                    dist.barrier()   # peers finished reading our buffers before the next case overwrites them
        err = comm.get_async_error()
        comm.finalize()
        q.put((rank, not bad and err == 0, f"err={err} bad={bad[:3]}"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_ipc_fuzz():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(N)]
    for p in procs:
        p.start()
    out = {}
    try:
        for _ in range(N):
            r, ok, msg = q.get(timeout=1200)
            out[r] = (ok, msg)
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(N):
        assert out[r][0], f"rank {r}: {out[r][1]}"
