#!/bin/bash
# Session 3 of round 2: trace evaluator A/B -- counter addresses from 4 x bank (RAP_TRACE_BANK4)
# and trace warps per work unit (RAP_TRACE_TK 64 / 128 / 256: the per-trial P / r draws of a unit
# are shared by TK trace warps); then the trace / sweep / congestion parity tests of the default
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/t_b4off.so "-DRAP_TRACE_BANK4=0"
b /tmp/t_tk128.so "-DRAP_TRACE_TK=128"
b /tmp/t_tk256.so "-DRAP_TRACE_TK=256"
b /tmp/t_def.so ""
timeout 600 python tools/ab_trace.py --rounds 9 --libs /tmp/t_def.so /tmp/t_b4off.so /tmp/t_tk128.so /tmp/t_tk256.so > "$OUT/r02c_ab_trace.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "trace or sweep or congestion" > "$OUT/r02c_pytest_trace.log" 2>&1
echo "pytest exit $?" >> "$OUT/r02c_pytest_trace.log"
