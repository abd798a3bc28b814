#!/bin/bash
# Launch-shape sweep of the default congestion-sweep kernel (run on the GPU box via gpurun):
# rebuilds librap.so per variant with RAP_EXTRA_NVCC_FLAGS and times 4e8 trials per step.
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
for v in ${VARIANTS:-"4 8 1" "4 8 2" "8 4 1" "2 16 1" "4 6 1" "4 4 1" "8 4 2"}; do
  set -- $v
  export RAP_EXTRA_NVCC_FLAGS="-DRAP_SWEEP_WARPS=$1 -DRAP_SWEEP_MINB=$2 -DRAP_SWEEP_GRID_MULT=$3"
  python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
  r=$(python bench.py --workload sweep --no-cpu --no-e2e --sweep-trials 400000000 --steps 3 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,4))")
  echo "warps=$1 minb=$2 grid_mult=$3 : $r G trials/s" | tee -a "$OUT/tune_sweep.txt"
done
unset RAP_EXTRA_NVCC_FLAGS
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
