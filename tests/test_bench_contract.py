"""bench.py keeps the driver's JSON-line contract (one line, required keys).

CPU: the reference arm (the oracle timed on the host).  GPU (-m gpu): our arm
at N=1 (loopback) and the N>1 code path with 2 processes on one GPU
(--test-same-gpu), each with sampled oracle parity at 0 mismatches.
"""

import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
        "scaling", "vs_baseline", "dtype", "data", "config", "e2e"}


def _run(cmd, timeout=600, env=None):
    e = dict(os.environ)
    e.update(env or {})
    p = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=e)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, p.stdout[-3000:]
    return json.loads(lines[0])


def test_reference_arm_contract():
    d = _run([sys.executable, "bench.py", "--impl", "reference", "--steps", "2", "--warmup", "1",
              "--size-mib", "4"])
    assert KEYS <= d.keys()
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "GB/s"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    # the oracle runs the arm's own workload (not a smaller sample under its label)
    assert d["config"]["workload"] == "allreduce-loopback-vr8-f32-4MiB-star8"
    assert d["config"]["bytes_per_rank"] == 4 << 20 and "4 MiB" in d["cpu_baseline"]["sample"]


def test_reference_arm_reports_n_gpus():
    d = _run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
              "--warmup", "1", "--size-mib", "1"])
    assert d["n_gpus"] == 2 and d["config"]["ranks"] == 2


def test_multi_gpu_without_gpus_fails_loudly():
    """--gpus N with fewer than N visible GPUs (this CPU box has none) must not
    fall back to a 1-GPU run: exit code != 0 and no JSON line."""
    e = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    p = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--steps", "1", "--warmup", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300, env=e)
    assert p.returncode != 0
    assert not [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert "--gpus 2" in p.stderr


@pytest.mark.gpu
def test_ours_single_gpu_contract():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    d = _run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3", "--size-mib", "16",
              "--no-cpu-baseline", "--e2e-steps", "2"])
    assert KEYS | {"roofline", "gpu_launches", "clocks", "parity"} <= d.keys()
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] == 3
    assert d["parity"]["complete"] and d["parity"]["mismatches"] == 0
    assert d["parity"]["elements_per_rank"] == (16 << 20) // 4 and d["parity"]["ranks"] == 8
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["achieved"] > 0 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert d["e2e"]["h2d_bytes_per_step"] == 8 * (16 << 20)
    sw = d["sweep"]   # busbw vs size: every x4 size from 1 KiB up to the bench size
    assert [p["bytes_per_rank"] for p in sw] == [1 << s for s in range(10, 25, 2)]
    assert all(p["busbw"] > 0 and p["busbw_graph"] > 0 for p in sw)


@pytest.mark.gpu
def test_ours_two_ranks_same_gpu_contract():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    # no launcher: bench.py re-launches itself as 2 ranks (both on cuda:0)
    d = _run([sys.executable, "bench.py", "--gpus", "2",
              "--steps", "3", "--warmup", "3", "--size-mib", "8", "--e2e-steps", "2", "--test-same-gpu"])
    assert KEYS | {"roofline", "gpu_launches", "parity", "staged"} <= d.keys()
    assert d["n_gpus"] == 2 and d["async_error"] == 0 and d["config"]["same_gpu"]
    assert d["parity"]["complete"] and d["parity"]["mismatches"] == 0 and d["parity"]["ranks"] == 2
    assert d["parity"]["ranks_mismatched"] == []
    for dt in ("f32", "bf16"):   # C2 sweeps both dtypes
        assert [p["bytes_per_rank"] for p in d["sweep"][dt]] == [1 << s for s in range(10, 24, 2)]
    assert d["p2p_ceiling"]["sm"]["one_to_one_GBps"] > 0 and d["roofline"]["peak"] > 0
    assert d["nvls"]["value"] is None and d["nvls"]["reason"]        # one GPU: no multicast team
    assert "2x" in d["paper_context"]["claims"][0]


def test_prepared_call_marshals_once():
    """PreparedCall converts every argument to its ctypes type once (host fast
    path); calling it re-issues exactly those arguments (CPU: a stub C function)."""
    import ctypes
    from paper_conf_icdcs_zhaozw24_b200.adapcc import PreparedCall
    seen = []

    @ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint64)
    def stub(h, n, m):
        seen.append((h, n, m))
        return 0
    pc = PreparedCall(stub, (ctypes.c_void_p(16), 1024, 0xFF), "stub")
    assert all(isinstance(a, ctypes._SimpleCData) for a in pc._args)
    pc()
    pc()
    assert seen == [(16, 1024, 0xFF)] * 2
