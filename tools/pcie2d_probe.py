"""PCIe 2-D copy probe (GPU box): pinned D2H / H2D cudaMemcpy2DAsync throughput vs row width, the
shape rap_transpose_host's band downloads take (width = band rows x element bytes), and the fixed
cost of one rap_transpose_host call."""
import ctypes
import os
import sys
import time

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402

rt = ctypes.CDLL(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib", "libcudart.so.12"))
rt.cudaMemcpy2DAsync.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_size_t,
                                 ctypes.c_size_t, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p]
N = 256 << 20
torch.cuda.init()
host_big = torch.empty(2 * N, dtype=torch.uint8).pin_memory()
dev = torch.empty(N, dtype=torch.uint8, device="cuda")


def t_of(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


for width in (256, 512, 1024, 2048, 4096, 8192, 32768):
    h = N // width

    def d2h():
        assert rt.cudaMemcpy2DAsync(host_big.data_ptr(), 2 * width, dev.data_ptr(), width, width, h, 2, None) == 0

    def h2d():
        assert rt.cudaMemcpy2DAsync(dev.data_ptr(), width, host_big.data_ptr(), 2 * width, width, h, 1, None) == 0
    a, b = t_of(d2h), t_of(h2d)
    print(f"width {width:6d} B x {h:7d} rows: D2H 2-D {N / a / 1e9:5.1f} GB/s, H2D 2-D {N / b / 1e9:5.1f} GB/s", flush=True)

# the band download's real shape: 4 KiB of each 32 KiB output row (cfg3, 1024-row bands)
for width, pitch in ((4096, 32768), (2048, 32768), (256, 32768), (8192, 65536)):
    h = N // pitch

    def d2h():
        assert rt.cudaMemcpy2DAsync(host_big.data_ptr(), pitch, dev.data_ptr(), width, width, h, 2, None) == 0
    a = t_of(d2h)
    print(f"D2H 2-D width {width} B, host pitch {pitch} B: {width * h / a / 1e9:5.1f} GB/s", flush=True)

x = torch.zeros((64, 64), dtype=torch.float32).pin_memory()
y = torch.empty((64, 64), dtype=torch.float32).pin_memory()
t = t_of(lambda: rap.transpose_host(x, out=y), reps=50)
print(f"rap_transpose_host 64x64 call: {t * 1e6:.0f} us", flush=True)
