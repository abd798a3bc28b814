#!/bin/bash
# e2e workspace probe + the default bench line + the reference arm (one B200).
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python tools/e2e_probe.py > "$OUT/r02_e2e_probe.txt" 2>&1
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
timeout 600 python bench.py --workload sweep > "$OUT/r02_bench_sweep.json" 2> "$OUT/r02_bench_sweep.err"
timeout 600 python bench.py --workload trace > "$OUT/r02_bench_trace.json" 2> "$OUT/r02_bench_trace.err"
