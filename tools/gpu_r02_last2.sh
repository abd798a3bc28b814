#!/bin/bash
# last check of round 2 after the rank-consistent soak fix: the multi-process GPU tests three times
# (the time-based soak loops let ranks drift a collective apart), then the whole -m gpu suite,
# smoke, and the default bench line
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$OUT/r02_smoke.log" 2>&1
for i in 1 2 3; do
  timeout 1200 python -m pytest tests/test_multiproc_gpu.py -m gpu -q -x > "$OUT/r02_multiproc_gpu_$i.log" 2>&1
  echo "exit $?" >> "$OUT/r02_multiproc_gpu_$i.log"
done
timeout 2400 python -m pytest tests -m gpu -q -x > "$OUT/r02_pytest_gpu.log" 2>&1
echo "pytest exit $?" >> "$OUT/r02_pytest_gpu.log"
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
