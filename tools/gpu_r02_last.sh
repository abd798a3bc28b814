#!/bin/bash
# last check of round 2 on the final tree: build + smoke + the -m gpu suite
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$OUT/r02_smoke.log" 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > "$OUT/r02_pytest_gpu.log" 2>&1
echo "pytest exit $?" >> "$OUT/r02_pytest_gpu.log"
