#!/bin/bash
# Round-2 validation pass on one B200: smoke, the full -m gpu suite, the default bench line and
# the reference arm (outputs under gpurun_out/; the committed copies go to profiles/).
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > "$OUT/r02_gpu.txt"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$OUT/r02_smoke.log" 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x --durations=15 > "$OUT/r02_pytest_gpu.log" 2>&1
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
tail -3 "$OUT/r02_pytest_gpu.log"
