#!/bin/bash
# ncu --set full capture of the default sweep kernel only (quick iteration on C1-C4).
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"sweep(32)?_kernel" -s 2 -c 1 \
    -o "$OUT/prof_sweep" -f python bench.py --no-e2e --no-cpu --workload sweep --steps 1 --warmup 2 \
    --sweep-trials 8388608 > "$OUT/ncu_sweep.log" 2>&1
