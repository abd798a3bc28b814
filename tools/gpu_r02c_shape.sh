#!/bin/bash
# Session 3 of round 2: sweep CTA shape A/B on the final kernel: 4 warps x 8 CTAs per SM (default)
# vs 8 warps x 4 CTAs -- the 8-warp build does not compile: its static shared memory passes the 48 KiB
# per-CTA limit for static allocations (the per-warp buffers scale with the warps)
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_w8.so "-DRAP_SWEEP_WARPS=8 -DRAP_SWEEP_MINB=4"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 7 --libs /tmp/s_def.so /tmp/s_w8.so > "$OUT/r02c_ab_sweep_shape.txt" 2>&1
