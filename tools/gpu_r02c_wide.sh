#!/bin/bash
# Session 3 of round 2: the w != 32 sweeps without __match_any_sync (RAP_WIDE_DEDUP_ATOM for
# 32 < w <= 256, RAP_SWEEP_GENERIC_DEDUP for w < 32): parity tests of the default build first, an
# interleaved A/B per width, then the default bench line and the reference arm (the oracle
# sample is a 256 MiB band in both arms now)
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "sweep or congestion or wide or table" > "$OUT/r02c_pytest_wide.log" 2>&1
rc=$?
echo "pytest exit $rc" >> "$OUT/r02c_pytest_wide.log"
[ $rc -ne 0 ] && exit 1
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/w_old.so "-DRAP_WIDE_DEDUP_ATOM=0 -DRAP_SWEEP_GENERIC_DEDUP=0"
b /tmp/w_def.so ""
for w in 16 64 128 256; do
  n=$((w <= 16 ? 40000000 : (w <= 64 ? 8000000 : (w <= 128 ? 4000000 : 2000000))))
  echo "== w=$w" >> "$OUT/r02c_ab_wide.txt"
  timeout 600 python tools/ab_sweep.py --w $w --trials $n --rounds 5 --libs /tmp/w_def.so /tmp/w_old.so 2>&1 | tail -2 >> "$OUT/r02c_ab_wide.txt"
done
timeout 900 python bench.py > "$OUT/r02_bench_default.json" 2> "$OUT/r02_bench_default.err"
timeout 900 python bench.py --impl reference > "$OUT/r02_bench_ref.json" 2> "$OUT/r02_bench_ref.err"
