#!/bin/bash
# ncu captures of the cfg4 (16384^2 float64) transpose kernels: the 8-byte-slot RAP kernel
# (transpose64_kernel, layout rap64), RAP-16 and the two-plane RAP; full sets + steady-state DRAM bytes.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
B="python bench.py --no-e2e --no-cpu --workload cfg4"
for k in transpose64_kernel transpose_rap16_kernel transpose_kernel; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 \
      -o "$OUT/prof_$k" -f $B --steps 1 --warmup 3 > "$OUT/ncu_$k.log" 2>&1
  timeout 600 ncu --cache-control none --clock-control none -k regex:$k -s 3 -c 4 --csv \
      --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --log-file "$OUT/steady_$k.csv" $B --steps 4 --warmup 3 > /dev/null 2>&1
done
ls -la "$OUT"
