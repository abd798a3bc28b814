#!/bin/bash
# Session 3 of round 2: sweep A/B -- branch-free per-trial histogram step (RAP_SWEEP_HIST_PRED:
# predicated result-slot STS.128, unconditional red.shared with a 0/1 increment) x lane-local
# leader test (RAP_SWEEP_LEAD_LANE: no VOTE); sweep parity tests on the default build
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_old.so "-DRAP_SWEEP_HIST_PRED=0 -DRAP_SWEEP_LEAD_LANE=0"
b /tmp/s_lead.so "-DRAP_SWEEP_HIST_PRED=0"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_old.so /tmp/s_lead.so > "$OUT/r02c_ab_sweep_pred.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02c_pytest_sweep_pred.log" 2>&1
echo "pytest sweep exit $?" >> "$OUT/r02c_pytest_sweep_pred.log"
B="python bench.py --no-e2e --no-cpu"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"sweep32_kernel" -s 3 -c 1 \
    -o "$OUT/prof_sweep_pred" -f $B --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608 > "$OUT/ncu_sweep_pred.log" 2>&1
ncu -i "$OUT/prof_sweep_pred.ncu-rep" --page raw --csv > "$OUT/prof_sweep_pred.raw.csv" 2>/dev/null
ncu -i "$OUT/prof_sweep_pred.ncu-rep" --page source --csv --print-source sass > "$OUT/prof_sweep_pred.source.csv" 2>/dev/null
gzip -9 -f "$OUT/prof_sweep_pred.source.csv" "$OUT/prof_sweep_pred.ncu-rep"
# (the sanitizer runs that followed were refused: compute-sanitizer is closed on this pool)
