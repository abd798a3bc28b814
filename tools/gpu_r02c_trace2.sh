#!/bin/bash
# Session 3 of round 2: trace evaluator work-unit shape A/B around the new default (TK = 128 trace
# warps x TB = 32 trials): TB 16 x TK 128 / 256, TK 192; then the trace parity tests
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/t_tb16.so "-DRAP_TRACE_TB=16"
b /tmp/t_tb16k256.so "-DRAP_TRACE_TB=16 -DRAP_TRACE_TK=256"
b /tmp/t_tk192.so "-DRAP_TRACE_TK=192"
b /tmp/t_def.so ""
timeout 600 python tools/ab_trace.py --rounds 9 --libs /tmp/t_def.so /tmp/t_tb16.so /tmp/t_tb16k256.so /tmp/t_tk192.so > "$OUT/r02c_ab_trace2.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "trace" > "$OUT/r02c_pytest_trace2.log" 2>&1
echo "pytest exit $?" >> "$OUT/r02c_pytest_trace2.log"
