#!/bin/bash
# Round-2 profiling pass (one B200): launch list of a short default bench, one ncu --set full
# capture per kernel of interest, steady-state DRAM bytes of the transposes.  Outputs under $OUT;
# summarised by tools/ncu_summary.py into profiles/ncu_summary.json.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
B="python bench.py --no-e2e --no-cpu"
# every launch of a short default bench (warm-up included), device time per launch
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv \
    --log-file "$OUT/launches.csv" $B --steps 4 --warmup 3 > /dev/null 2>&1
full() {  # full <stem> <kernel regex> <bench args...>
  local stem=$1 k=$2; shift 2
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$k" -s 3 -c 1 \
      -o "$OUT/$stem" -f $B "$@" > "$OUT/ncu_$stem.log" 2>&1
}
steady() {  # steady <stem> <kernel regex> <bench args...>
  local stem=$1 k=$2; shift 2
  timeout 900 ncu --cache-control none --clock-control none -k regex:"$k" -s 3 -c 4 --csv \
      --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --log-file "$OUT/$stem.csv" $B "$@" > /dev/null 2>&1
}
full prof_t64_rap "^transpose_kernel" --workload cfg4 --steps 1 --warmup 3
full prof_t64_rap64 "transpose64_kernel" --workload cfg4 --steps 1 --warmup 3
full prof_t64_rap16 "transpose_rap16_kernel" --workload cfg4 --steps 1 --warmup 3
for lay in rap raw pad xor ras; do
  full prof_t32_$lay "^transpose_kernel" --workload cfg3 --layout $lay --steps 1 --warmup 3 --sweep-trials 1024
done
full prof_sweep "sweep32_kernel" --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608
full prof_trace "trace32_kernel" --workload trace --steps 1 --warmup 3 --trace-trials 2048
steady steady_t64 "^transpose_kernel" --workload cfg4 --steps 4 --warmup 3
steady steady_t64_rap64 "transpose64_kernel" --workload cfg4 --steps 4 --warmup 3
steady steady_t64_rap16 "transpose_rap16_kernel" --workload cfg4 --steps 4 --warmup 3
steady steady_t32 "^transpose_kernel" --workload cfg3 --steps 4 --warmup 3 --sweep-trials 1024
ls -la "$OUT"
# export the pages the summary reads, keep compressed reports of the key kernels only (gpurun
# brings back at most 64 MiB)
for rep in "$OUT"/*.ncu-rep; do
  stem=${rep%.ncu-rep}
  ncu -i "$rep" --page raw --csv > "$stem.raw.csv" 2>/dev/null
  ncu -i "$rep" --page source --csv --print-source sass > "$stem.source.csv" 2>/dev/null
  case $(basename "$stem") in
    prof_t64_rap|prof_t32_rap|prof_sweep|prof_trace) gzip -9 -f "$rep" ;;
    *) rm -f "$rep" ;;
  esac
done
gzip -9 -f "$OUT"/*.source.csv
du -sh "$OUT"
