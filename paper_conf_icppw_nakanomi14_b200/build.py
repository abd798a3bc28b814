"""Build librap.so in-tree with nvcc for sm_100a (no torch involved in the library)."""
from __future__ import annotations

import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "librap.so")
SOURCES = ["api.cu", "transpose.cu", "congestion.cu", "exchange.cu", "smem_bench.cu", "sweep_wide.cu", "sweep4.cu", "host_pipeline.cu", "transpose_rap16.cu",
           "transpose64.cu", "pdl_registry.cu"]
HEADERS = ["rap_rng.cuh", "rap_warp.cuh", "rap_internal.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: librap.so cannot be built")


STAMP = LIB + ".flags"


def _flags() -> str:
    """The effective extra flags; a build with different flags (a tuning or ablation build left
    behind by tools/*.sh) is stale even when no source changed."""
    return " ".join(os.environ.get("RAP_EXTRA_NVCC_FLAGS", "").split())


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    try:
        if open(STAMP).read() != _flags():
            return True
    except OSError:
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "rap.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src: str, obj: str, extra, verbose: bool):
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", *extra,
           "-c", "-o", obj, os.path.join(CSRC, src)]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd, cwd=CSRC)


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every translation unit to an object (in parallel, one nvcc per unit: the template
    instantiations make a serial build take minutes) and link librap.so."""
    if not force and not _stale():
        return LIB
    from concurrent.futures import ThreadPoolExecutor
    # RAP_EXTRA_NVCC_FLAGS: launch-shape macros for tuning runs only (e.g. -DRAP_SWEEP_WARPS=8)
    extra = os.environ.get("RAP_EXTRA_NVCC_FLAGS", "").split()
    objdir = os.path.join(PKG, "build", f"obj{os.getpid()}")
    os.makedirs(objdir, exist_ok=True)
    objs = [os.path.join(objdir, f[:-3] + ".o") for f in SOURCES]
    with ThreadPoolExecutor(max_workers=min(len(SOURCES), os.cpu_count() or 4)) as ex:
        for f in [ex.submit(_compile, s, o, extra, verbose) for s, o in zip(SOURCES, objs)]:
            f.result()
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([_nvcc(), *ARCH, "-shared", "-o", tmp, *objs], cwd=CSRC)
    shutil.rmtree(objdir, ignore_errors=True)
    os.replace(tmp, LIB)
    with open(STAMP, "w") as f:
        f.write(_flags())
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
