"""Interleaved A/B of transpose kernels from several librap.so builds in ONE process (GPU box).

    python tools/ab_lib.py --libs /tmp/a.so:rap /tmp/b.so:rap /tmp/b.so:rap16 --n 16384 --dtype f64

Each `lib:layout` arm is timed as `--launches` back-to-back rap_transpose calls between one CUDA
event pair, arms interleaved round by round (box noise hits every arm alike); prints GB/s per
round and the median per arm.  The libraries are dlopen'ed side by side (RTLD_LOCAL).
"""
import argparse
import ctypes
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads  # noqa: E402

LAYOUTS = {"raw": 0, "pad": 1, "xor": 2, "ras": 3, "rap": 4, "rap16": 5, "rap64": 6}


def load(path):
    L = ctypes.CDLL(path)
    vp, i64, u32, u64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    L.rap_transpose.argtypes = [vp, vp, i64, i64, i64, i64, u32, i32, u64, vp]
    L.rap_transpose.restype = i32
    return L


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--libs", nargs="+", required=True)
    ap.add_argument("--n", type=int, default=16384)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--launches", type=int, default=20)
    a = ap.parse_args()
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    eb = 8 if a.dtype == "f64" else 4
    x = workloads.random_bits(a.n, a.n, dt, seed=0, device="cuda")
    y = torch.empty_like(x)
    ref = None
    libs = {}
    arms = []
    for spec in a.libs:
        path, lay = spec.rsplit(":", 1)
        if path not in libs:
            libs[path] = load(path)
        arms.append((spec, libs[path], LAYOUTS[lay]))
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    call = lambda L, lay: L.rap_transpose(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), a.n, a.n,
                                          a.n, a.n, eb, lay, 0, st)
    for spec, L, lay in arms:                      # correctness: every arm gives the same bits
        assert call(L, lay) == 0, spec
        torch.cuda.synchronize()
        bits = y.view(torch.int64 if eb == 8 else torch.int32).clone()
        if ref is None:
            ref = bits
        assert torch.equal(bits, ref), spec
    import subprocess
    smi = subprocess.Popen(["nvidia-smi", "-i", str(torch.cuda.current_device()),
                            "--query-gpu=clocks.sm,clocks.mem,power.draw,temperature.gpu,clocks_event_reasons.active",
                            "--format=csv,noheader,nounits", "-lms", "250"], stdout=subprocess.PIPE, text=True)
    res = {spec: [] for spec, _, _ in arms}
    nb = 2 * a.n * a.n * eb
    for r in range(a.rounds):
        for spec, L, lay in arms:
            for _ in range(3):
                call(L, lay)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for _ in range(a.launches):
                call(L, lay)
            e.record()
            torch.cuda.synchronize()
            res[spec].append(nb * a.launches / (s.elapsed_time(e) * 1e-3) / 1e9)
        print(f"round {r}: " + "  ".join(f"{k}={v[-1]:.0f}" for k, v in res.items()), flush=True)
    smi.terminate()
    samples = [ln.split(", ") for ln in smi.communicate()[0].strip().splitlines()]
    if samples:
        col = lambda i: sorted(float(x[i]) for x in samples if len(x) > 4)
        sm, mem, pw, tc = col(0), col(1), col(2), col(3)
        print(f"clocks: sm {sm[0]:.0f}..{sm[-1]:.0f} MHz (median {sm[len(sm) // 2]:.0f}), mem {mem[len(mem) // 2]:.0f} MHz, "
              f"power max {pw[-1]:.0f} W, temp max {tc[-1]:.0f} C, reasons {sorted(set(x[4] for x in samples if len(x) > 4))}")
    for k, v in res.items():
        print(f"{k:40s} median {statistics.median(v):7.1f} GB/s  min {min(v):7.1f}  max {max(v):7.1f}")


if __name__ == "__main__":
    main()
