#!/bin/bash
# Session 3 of round 2: sweep A/B -- the lane-mode Fisher-Yates on the lane's byte P table in shared
# memory (RAP_SWEEP_FY_BYTES) instead of bit planes, with the other domains' Philox interleaved
# (RAP_SWEEP_FY_INTERLEAVE); sweep parity tests of the default first
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02c_pytest_sweep_fyb.log" 2>&1
rc=$?
echo "pytest exit $rc" >> "$OUT/r02c_pytest_sweep_fyb.log"
[ $rc -ne 0 ] && exit 1
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_planes.so "-DRAP_SWEEP_FY_BYTES=0"
b /tmp/s_noil.so "-DRAP_SWEEP_FY_INTERLEAVE=0"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_planes.so /tmp/s_noil.so > "$OUT/r02c_ab_sweep_fyb.txt" 2>&1
B="python bench.py --no-e2e --no-cpu"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"sweep32_kernel" -s 3 -c 1 \
    -o "$OUT/prof_sweep_fyb" -f $B --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608 > "$OUT/ncu_sweep_fyb.log" 2>&1
ncu -i "$OUT/prof_sweep_fyb.ncu-rep" --page raw --csv > "$OUT/prof_sweep_fyb.raw.csv" 2>/dev/null
ncu -i "$OUT/prof_sweep_fyb.ncu-rep" --page source --csv --print-source sass > "$OUT/prof_sweep_fyb.source.csv" 2>/dev/null
gzip -9 -f "$OUT/prof_sweep_fyb.source.csv"; rm -f "$OUT/prof_sweep_fyb.ncu-rep"
