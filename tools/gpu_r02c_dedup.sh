#!/bin/bash
# Session 3 of round 2: sweep A/B -- merged requests of the random access from a shared-memory cell
# bitmap (RAP_SWEEP_DEDUP_SMEM: one atom.shared.or) instead of __match_any_sync, and the histogram
# counted once per batch of 32 trials (RAP_SWEEP_BATCH_HIST); sweep parity tests of the default first
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02c_pytest_sweep_dedup.log" 2>&1
rc=$?
echo "pytest exit $rc" >> "$OUT/r02c_pytest_sweep_dedup.log"
[ $rc -ne 0 ] && exit 1
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_match.so "-DRAP_SWEEP_DEDUP_SMEM=0"
b /tmp/s_nobatch.so "-DRAP_SWEEP_BATCH_HIST=0"
b /tmp/s_old.so "-DRAP_SWEEP_DEDUP_SMEM=0 -DRAP_SWEEP_BATCH_HIST=0"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_match.so /tmp/s_nobatch.so /tmp/s_old.so > "$OUT/r02c_ab_sweep_dedup.txt" 2>&1
B="python bench.py --no-e2e --no-cpu"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"sweep32_kernel" -s 3 -c 1 \
    -o "$OUT/prof_sweep_dedup" -f $B --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608 > "$OUT/ncu_sweep_dedup.log" 2>&1
ncu -i "$OUT/prof_sweep_dedup.ncu-rep" --page raw --csv > "$OUT/prof_sweep_dedup.raw.csv" 2>/dev/null
ncu -i "$OUT/prof_sweep_dedup.ncu-rep" --page source --csv --print-source sass > "$OUT/prof_sweep_dedup.source.csv" 2>/dev/null
gzip -9 -f "$OUT/prof_sweep_dedup.source.csv"; rm -f "$OUT/prof_sweep_dedup.ncu-rep"
