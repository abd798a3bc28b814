#!/bin/bash
# full validation + measurement pass (one B200): smoke, the -m gpu suite, trace A/B, bench lines
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > "$OUT/r02_smoke.log" 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > "$OUT/r02_pytest_gpu.log" 2>&1
tail -2 "$OUT/r02_pytest_gpu.log"
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
timeout 600 python bench.py --workload sweep > "$OUT/r02_bench_sweep.json" 2> "$OUT/r02_bench_sweep.err"
timeout 600 python bench.py --workload trace > "$OUT/r02_bench_trace.json" 2> "$OUT/r02_bench_trace.err"
bash tools/gpu_profile_r02.sh "$OUT/p02" > "$OUT/p02.log" 2>&1
# (compute-sanitizer is closed on this GPU pool since session 3 of round 2: profiles/r02c_sanitizer_refused.txt;
#  the clean round-2 runs are profiles/r02_sanitizer.txt)
du -sh "$OUT"
