#!/bin/bash
# ncu capture of the w = 32 sweep and the trace evaluator (exported pages), plus the sweep A/B
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
B="python bench.py --no-e2e --no-cpu"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep32_kernel -s 3 -c 1 \
    -o "$OUT/prof_sweep" -f $B --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608 > "$OUT/ncu_sweep.log" 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:trace32_kernel -s 3 -c 1 \
    -o "$OUT/prof_trace" -f $B --workload trace --steps 1 --warmup 3 --trace-trials 2048 > "$OUT/ncu_trace.log" 2>&1
for rep in "$OUT"/*.ncu-rep; do
  stem=${rep%.ncu-rep}
  ncu -i "$rep" --page raw --csv > "$stem.raw.csv" 2>/dev/null
  ncu -i "$rep" --page source --csv --print-source sass > "$stem.source.csv" 2>/dev/null
  gzip -9 -f "$rep" "$stem.source.csv"
done
