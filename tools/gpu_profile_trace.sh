#!/bin/bash
# ncu --set full capture of the w = 32 trace evaluator alone (4096 trace warps x 2048 trials x 5
# schemes per launch), the same command line as tools/gpu_profile.sh's trace entry.
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"trace(32)?_kernel" -s 2 -c 1 \
    -o "$OUT/prof_trace" -f python bench.py --no-e2e --no-cpu --workload trace --steps 1 --warmup 2 --trace-trials 2048 > "$OUT/ncu_trace.log" 2>&1
