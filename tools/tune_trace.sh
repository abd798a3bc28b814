#!/bin/bash
# Launch-shape sweep of the w = 32 trace evaluator (run on the GPU box via gpurun): rebuilds
# librap.so per variant (trials per unit TB, trace warps per unit TK, warps per CTA, min CTAs per
# SM) and times the bench trace workload (4096 trace warps x T trials x 5 schemes per step).
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
for v in ${VARIANTS:-"32 64 4 8" "32 32 4 8" "32 128 4 8" "64 64 4 8" "32 64 4 6" "16 64 4 8" "32 64 8 4"}; do
  set -- $v
  export RAP_EXTRA_NVCC_FLAGS="-DRAP_TRACE_TB=$1 -DRAP_TRACE_TK=$2 -DRAP_TRACE_WARPS=$3 -DRAP_TRACE32_MINB=$4"
  python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
  for T in 256 2048; do
    r=$(timeout 120 python bench.py --workload trace --no-cpu --no-e2e --trace-trials $T --steps 10 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['trace']['kernel_ms_median'],4))")
    echo "tb=$1 tk=$2 warps=$3 minb=$4 trials=$T : $r (G evaluations/s, kernel ms)" | tee -a "$OUT/tune_trace.txt"
  done
done
unset RAP_EXTRA_NVCC_FLAGS
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
