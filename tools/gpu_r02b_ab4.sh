#!/bin/bash
# Session 2 of round 2: sweep A/B -- trial planes through shared memory (RAP_SWEEP_PLANES_SMEM) x
# vector counter clears (RAP_SWEEP_CLEAR_VEC); sweep parity tests on the default build
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_p0c0.so "-DRAP_SWEEP_PLANES_SMEM=0 -DRAP_SWEEP_CLEAR_VEC=0"
b /tmp/s_p0c1.so "-DRAP_SWEEP_PLANES_SMEM=0"
b /tmp/s_p1c0.so "-DRAP_SWEEP_CLEAR_VEC=0"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_p0c0.so /tmp/s_p0c1.so /tmp/s_p1c0.so > "$OUT/r02b_ab_planes.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02b_pytest_sweep3.log" 2>&1
echo "pytest sweep exit $?" >> "$OUT/r02b_pytest_sweep3.log"
