#!/bin/bash
# A/B: RAP / RAS tiles with wrapped 32-word rows ((j + sh) & 31 in the address, half the shared
# memory) against the unwrapped 64-word row windows, cfg3 fp32 and cfg4 fp64 (two planes).
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/w_wrap.so "-DRAP32_WRAP=1"
b /tmp/w_def.so ""
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/w_def.so:rap /tmp/w_wrap.so:rap /tmp/w_def.so:xor \
    /tmp/w_def.so:pad /tmp/w_wrap.so:ras /tmp/w_def.so:ras 2>&1 | tee "$OUT/ab_wrap32.txt"
python tools/ab_lib.py --rounds 9 --libs /tmp/w_def.so:rap /tmp/w_wrap.so:rap /tmp/w_def.so:rap16 2>&1 | tee "$OUT/ab_wrap64.txt"
