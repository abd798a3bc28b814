#!/bin/bash
# A/B of the cfg2 sweep kernel builds (tools/ab_sweep.py, interleaved rounds, 5e7 trials per launch):
# the histogram increment through a kept shared-window address (RAP_SWEEP_HIST_SA) vs atomicAdd
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_gen.so "-DRAP_SWEEP_HIST_SA=0"
b /tmp/s_m7.so "-DRAP_SWEEP_MINB=7"
b /tmp/s_def.so ""
python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_gen.so /tmp/s_m7.so 2>&1 | tee "$OUT/ab_sweep6.txt"
