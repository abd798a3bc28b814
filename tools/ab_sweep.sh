#!/bin/bash
# A/B of the cfg2 sweep kernel builds (tools/ab_sweep.py, interleaved rounds, 5e7 trials per launch):
# the XOR-with-lane-selector on the FMA pipe (RAP_FMA_XOR) and register budgets.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_lop.so "-DRAP_FMA_XOR=0"
b /tmp/s_m7.so "-DRAP_SWEEP_MINB=7"
b /tmp/s_m6.so "-DRAP_SWEEP_MINB=6"
b /tmp/s_fma.so ""
python tools/ab_sweep.py --rounds 9 --libs /tmp/s_lop.so /tmp/s_fma.so /tmp/s_m7.so /tmp/s_m6.so 2>&1 | tee "$OUT/ab_sweep.txt"
