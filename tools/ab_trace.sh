#!/bin/bash
# A/B of the trace evaluator builds: shared-memory bank counters (RAP_TRACE_SMEM_BANKS) vs ballots
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/t_ballot.so "-DRAP_TRACE_SMEM_BANKS=0"
b /tmp/t_m3.so "-DRAP_TRACE32_MINB=3"
b /tmp/t_def.so ""
python tools/ab_trace.py --libs /tmp/t_def.so /tmp/t_ballot.so /tmp/t_m3.so 2>&1 | tee "$OUT/ab_trace.txt"
