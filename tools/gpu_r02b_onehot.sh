#!/bin/bash
# Session 2 of round 2: one-hot sweep maxima (RAP_SWEEP_ONEHOT) -- parity, A/B against the
# CREDUX.MAX build, capture; the default bench line with the RAP64 headline.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_max.so "-DRAP_SWEEP_ONEHOT=0"
b /tmp/s_oh.so ""
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion" > "$OUT/r02b_pytest_sweep.log" 2>&1
echo "pytest sweep exit $?" >> "$OUT/r02b_pytest_sweep.log"
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_oh.so /tmp/s_max.so > "$OUT/r02b_ab_onehot.txt" 2>&1
timeout 900 python bench.py > "$OUT/r02b_bench_default.json" 2> "$OUT/r02b_bench_default.err"
B="python bench.py --no-e2e --no-cpu"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep32_kernel -s 3 -c 1 \
    -o "$OUT/r02b_prof_sweep" -f $B --workload sweep --steps 1 --warmup 3 --sweep-trials 8388608 > "$OUT/r02b_ncu_sweep.log" 2>&1
for rep in "$OUT"/r02b_prof_*.ncu-rep; do
  stem=${rep%.ncu-rep}
  ncu -i "$rep" --page raw --csv > "$stem.raw.csv" 2>/dev/null
  ncu -i "$rep" --page source --csv --print-source sass > "$stem.source.csv" 2>/dev/null
  gzip -9 -f "$rep" "$stem.source.csv"
done
