#!/bin/bash
# Round profiling pass (run on the GPU box via gpurun): launch list + one ncu --set full capture
# per kernel of interest.  Outputs land in gpurun_out/ and are summarised by tools/ncu_summary.py.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
B="python bench.py --no-e2e --no-cpu"
# every launch of a short default bench (warm-up included), device time per launch
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file "$OUT/launches.csv" $B --steps 5 --warmup 3 > /dev/null 2>&1
for lay in rap raw pad xor ras; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:transpose_kernel -s 3 -c 1 \
      -o "$OUT/prof_t32_$lay" -f $B --steps 1 --warmup 3 --layout $lay --sweep-trials 1024 > "$OUT/ncu_t32_$lay.log" 2>&1
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:transpose_kernel -s 3 -c 1 \
    -o "$OUT/prof_t64_rap" -f $B --workload cfg4 --steps 1 --warmup 3 > "$OUT/ncu_t64_rap.log" 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:transpose_rap16_kernel -s 3 -c 1 \
    -o "$OUT/prof_t64_rap16" -f $B --workload cfg4 --steps 1 --warmup 3 > "$OUT/ncu_t64_rap16.log" 2>&1
# steady-state DRAM bytes per launch: consecutive launches, no cache flush between them
timeout 600 ncu --cache-control none --clock-control none -k regex:transpose_kernel -s 3 -c 4 --csv \
    --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --log-file "$OUT/steady_t32.csv" $B --steps 4 --warmup 3 --sweep-trials 1024 > /dev/null 2>&1
timeout 600 ncu --cache-control none --clock-control none -k regex:transpose_kernel -s 3 -c 4 --csv \
    --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --log-file "$OUT/steady_t64.csv" $B --workload cfg4 --layout rap --steps 4 --warmup 3 > /dev/null 2>&1
timeout 600 ncu --cache-control none --clock-control none -k regex:transpose_rap16_kernel -s 3 -c 4 --csv \
    --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --log-file "$OUT/steady_t64_rap16.csv" $B --workload cfg4 --steps 4 --warmup 3 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"sweep(32)?_kernel" -s 2 -c 1 \
    -o "$OUT/prof_sweep" -f $B --workload sweep --steps 1 --warmup 2 --sweep-trials 8388608 > "$OUT/ncu_sweep.log" 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"sweep_match_kernel" -s 2 -c 1 \
    -o "$OUT/prof_sweep_match" -f $B --workload sweep --sweep-algo match --steps 1 --warmup 2 --sweep-trials 4194304 > "$OUT/ncu_sweep_match.log" 2>&1
# trace evaluator: 4096 warps x 2048 trials x 5 schemes per launch
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"trace(32)?_kernel" -s 2 -c 1 \
    -o "$OUT/prof_trace" -f $B --workload trace --steps 1 --warmup 2 --trace-trials 2048 > "$OUT/ncu_trace.log" 2>&1
ls -la "$OUT"
