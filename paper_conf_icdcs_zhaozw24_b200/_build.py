"""Build libadapcc.so in-tree with nvcc for sm_100a (no JIT cache, no torch).

    python -m paper_conf_icdcs_zhaozw24_b200._build
"""

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libadapcc.so")
SOURCES = ["adapcc.cpp", "strategy.cpp", "plan.cpp", "engine.cu", "engine_tma_direct.cu",
           "engine_tma_staged.cu", "engine_flat.cu", "probe.cu"]
HEADERS = ["engine.cuh", "engine_common.cuh", "engine_tma_impl.cuh", "launch.hpp", "plan.hpp",
           "strategy.hpp"]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC,-Wall,-fvisibility=hidden",
    "-shared", "-cudart", "static", "-ldl",
]


def _nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.isabs(c) and os.path.exists(c) or not os.path.isabs(c)):
            return c
    return "nvcc"


def _stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "adapcc.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force=False, verbose=True, out=None, defines=()):
    """Compile libadapcc.so (or a tuning variant at `out` with extra -D defines)."""
    out = out or LIB
    if out == LIB and not defines and not force and not _stale():
        return LIB
    cmd = [_nvcc(), *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", os.path.join(ROOT, "include"),
           "-o", out + ".tmp", *[os.path.join(CSRC, f) for f in SOURCES]]
    if verbose:
        print("[adapcc build]", " ".join(cmd), flush=True)
    subprocess.run(cmd, check=True)
    os.replace(out + ".tmp", out)
    return out


if __name__ == "__main__":
    build(force="--force" in sys.argv)
