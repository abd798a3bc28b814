#!/bin/bash
# Session 3 of round 2: sweep A/B -- per-trial loop unrolled by 2 (RAP_SWEEP_UNROLL_M) and fewer
# CTAs per SM with more registers (RAP_SWEEP_MINB 7 / 6: the default's 64-register cap spills 44
# bytes); then the whole -m gpu suite on the default build
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_u2.so "-DRAP_SWEEP_UNROLL_M=2"
b /tmp/s_m7.so "-DRAP_SWEEP_MINB=7"
b /tmp/s_m6.so "-DRAP_SWEEP_MINB=6"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_u2.so /tmp/s_m7.so /tmp/s_m6.so > "$OUT/r02c_ab_sweep_unroll.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 2400 python -m pytest tests -m gpu -q -x > "$OUT/r02c_pytest_gpu.log" 2>&1
echo "pytest exit $?" >> "$OUT/r02c_pytest_gpu.log"
