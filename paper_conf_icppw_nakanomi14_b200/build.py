"""Build librap.so in-tree with nvcc for sm_100a (no torch involved in the library)."""
from __future__ import annotations

import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "librap.so")
SOURCES = ["api.cu", "transpose.cu", "congestion.cu", "exchange.cu", "smem_bench.cu", "sweep_wide.cu", "sweep4.cu", "host_pipeline.cu", "transpose_rap16.cu"]
HEADERS = ["rap_rng.cuh", "rap_warp.cuh", "rap_internal.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: librap.so cannot be built")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "rap.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    # RAP_EXTRA_NVCC_FLAGS: launch-shape macros for tuning runs only (e.g. -DRAP_SWEEP_WARPS=8)
    extra = os.environ.get("RAP_EXTRA_NVCC_FLAGS", "").split()
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", *extra,
           "-shared", "-o", tmp, *[os.path.join(CSRC, f) for f in SOURCES]]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd, cwd=CSRC)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
