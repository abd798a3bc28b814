"""e2e band-plan probe (GPU box): rap_transpose_host on the cfg4 (and cfg3) matrix for several
device workspaces (= band heights) from two librap.so builds (with / without the fill ramp),
interleaved rounds.   python tools/e2e_bands.py /tmp/a.so /tmp/b.so"""
import ctypes
import statistics
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

import workloads  # noqa: E402


def load(path):
    L = ctypes.CDLL(path)
    vp, i64, u32, i32, u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint32, ctypes.c_int, ctypes.c_uint64
    L.rap_transpose_host.argtypes = [vp, vp, i64, i64, i64, i64, u32, i32, u64, vp, ctypes.c_size_t, vp]
    L.rap_transpose_host.restype = i32
    return L


libs = [(p, load(p)) for p in sys.argv[1:]]
for (n, dt) in ((16384, torch.float64), (8192, torch.float32)):
    x = workloads.random_bits(n, n, dt, seed=0).pin_memory()
    y = torch.empty((n, n), dtype=dt).pin_memory()
    eb = x.element_size()
    ws_list = [16 << 20, 32 << 20, 48 << 20, 64 << 20, 96 << 20, 128 << 20, 1024 << 20]
    work = torch.empty(max(ws_list), dtype=torch.uint8, device="cuda")
    res = {}
    for r in range(3):
        for p, L in libs:
            for ws in ws_list:
                t0 = time.perf_counter()
                for _ in range(3):
                    rc = L.rap_transpose_host(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), n, n, n, n,
                                              eb, 4, 0, ctypes.c_void_p(work.data_ptr()), ws, None)
                    assert rc == 0
                el = (time.perf_counter() - t0) / 3
                res.setdefault((p, ws), []).append(2 * x.nbytes / el / 1e9)
    for (p, ws), v in res.items():
        print(f"{n} {str(dt)[6:]} {p:22s} ws {ws >> 20:5d} MiB  {statistics.median(v):6.1f} GB/s  ({min(v):.1f}-{max(v):.1f})",
              flush=True)
