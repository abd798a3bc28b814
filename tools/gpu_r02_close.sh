#!/bin/bash
# closing pass of round 2 (one B200): smoke, the -m gpu suite, the profile refresh, then the bench
# lines against the refreshed captures (bench.py's roofline objects read profiles/ncu_summary.json,
# so the lines are re-run after tools/ncu_summary.py has been applied here -- see the README)
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$OUT/r02_smoke.log" 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > "$OUT/r02_pytest_gpu.log" 2>&1
tail -2 "$OUT/r02_pytest_gpu.log"
bash tools/gpu_profile_r02.sh "$OUT/p02" > "$OUT/p02.log" 2>&1
python tools/ncu_summary.py "$OUT/p02" profiles/ncu_summary.json r02 > "$OUT/ncu_summary.log" 2>&1
cp profiles/ncu_summary.json "$OUT/ncu_summary.json"
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
timeout 600 python bench.py --workload sweep > "$OUT/r02_bench_sweep.json" 2> "$OUT/r02_bench_sweep.err"
timeout 600 python bench.py --workload trace > "$OUT/r02_bench_trace.json" 2> "$OUT/r02_bench_trace.err"
du -sh "$OUT"
