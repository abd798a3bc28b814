#!/bin/bash
# A/B of the cfg2 sweep kernel builds (tools/ab_sweep.py, interleaved rounds, 5e7 trials per launch):
# register budgets / CTA sizes / grid oversubscription around the default (RAP_SWEEP_MINB=7).
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_m8.so "-DRAP_SWEEP_MINB=8"
b /tmp/s_m5.so "-DRAP_SWEEP_MINB=5"
b /tmp/s_w8m3.so "-DRAP_SWEEP_WARPS=8 -DRAP_SWEEP_MINB=3"
b /tmp/s_w8m4.so "-DRAP_SWEEP_WARPS=8 -DRAP_SWEEP_MINB=4"
b /tmp/s_g4.so "-DRAP_SWEEP_GRID_MULT=4"
b /tmp/s_def.so ""
python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_m8.so /tmp/s_m5.so /tmp/s_w8m3.so /tmp/s_w8m4.so /tmp/s_g4.so 2>&1 | tee "$OUT/ab_sweep2.txt"
