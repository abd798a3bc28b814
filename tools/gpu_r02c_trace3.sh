#!/bin/bash
# Session 3 of round 2: trace evaluator A/B -- per-trial congestion kept by lane t and counted into a
# per-warp shared-memory histogram once per block (RAP_TRACE_HIST_SMEM); trace parity tests first
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "trace" > "$OUT/r02c_pytest_trace3.log" 2>&1
rc=$?
echo "pytest exit $rc" >> "$OUT/r02c_pytest_trace3.log"
[ $rc -ne 0 ] && exit 1
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/t_reg.so "-DRAP_TRACE_HIST_SMEM=0"
b /tmp/t_def.so ""
timeout 600 python tools/ab_trace.py --rounds 9 --libs /tmp/t_def.so /tmp/t_reg.so > "$OUT/r02c_ab_trace3.txt" 2>&1
