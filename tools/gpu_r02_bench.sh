#!/bin/bash
# the bench lines only (after a profile refresh changed profiles/ncu_summary.json, which the
# roofline objects read): default, reference arm, sweep, trace
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
timeout 600 python bench.py --workload sweep > "$OUT/r02_bench_sweep.json" 2> "$OUT/r02_bench_sweep.err"
timeout 600 python bench.py --workload trace > "$OUT/r02_bench_trace.json" 2> "$OUT/r02_bench_trace.err"
