#!/bin/bash
# Session 3 of round 2: 32-bit transposes through column-pair 8-byte slots (RAP32_PAIR: the
# one-double-per-slot kernel on v(i,k) = (a[i][2k], a[i][2k+1])) -- parity tests of that build,
# then an interleaved A/B against the default 32-bit kernel (cfg3 8192^2 and 16384^2 fp32)
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/p_6.so "-DRAP32_PAIR=1 -DRAP32_PAIR_SR=6 -DRAP32_PAIR_MINB=2"
b /tmp/p_8.so "-DRAP32_PAIR=1 -DRAP32_PAIR_SR=8"
b /tmp/p_def.so ""
b /tmp/p_12.so "-DRAP32_PAIR=1"
RAP_EXTRA_NVCC_FLAGS="-DRAP32_PAIR=1" timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "transpose and not host and not 2pow32 and not aspect" > "$OUT/pair_pytest.log" 2>&1
echo "pytest exit $?" >> "$OUT/pair_pytest.log"
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/p_def.so:rap /tmp/p_12.so:rap /tmp/p_8.so:rap /tmp/p_6.so:rap > "$OUT/r02c_ab_pair.txt" 2>&1
python tools/ab_lib.py --rounds 7 --n 16384 --dtype f32 --libs /tmp/p_def.so:rap /tmp/p_12.so:rap /tmp/p_8.so:rap /tmp/p_6.so:rap > "$OUT/r02c_ab_pair_16k.txt" 2>&1
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1
