#!/bin/bash
# Sweep kernel time vs batch size (in waves of the resident grid: 148 SMs x 8 CTAs x 4 warps x 32
# trials = 151552 trials): separates the per-launch fixed cost from the per-trial cost.
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
for w in 1 2 4 8 16 64; do
  n=$((151552 * w))
  python bench.py --workload sweep --no-cpu --no-e2e --sweep-trials $n --steps 20 --warmup 5 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print($w, $n, round(d['sweep']['kernel_ms_median']*1e3,2), 'us', round(d['value']/1e9,3), 'G trials/s')"
done | tee "$OUT/sweep_waves.txt"
