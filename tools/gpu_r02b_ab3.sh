#!/bin/bash
# Session 2 of round 2: sweep A/B -- pre-multiplied banks (RAP_SWEEP_BANK4) x STS.128 result slots
# (RAP_SWEEP_RES_VEC); sweep parity tests on the default build
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_b0v0.so "-DRAP_SWEEP_BANK4=0 -DRAP_SWEEP_RES_VEC=0"
b /tmp/s_b1v0.so "-DRAP_SWEEP_RES_VEC=0"
b /tmp/s_b0v1.so "-DRAP_SWEEP_BANK4=0"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_b0v0.so /tmp/s_b1v0.so /tmp/s_b0v1.so > "$OUT/r02b_ab_bank4.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02b_pytest_sweep2.log" 2>&1
echo "pytest sweep exit $?" >> "$OUT/r02b_pytest_sweep2.log"
