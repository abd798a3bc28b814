#!/bin/bash
# A/B of fp32 CTA / cluster shapes (PDL off), cfg3 8192^2 and a 16384^2 fp32 matrix
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/f_c8.so "-DRAP32_CL=8"
b /tmp/f_4x4c2.so "-DRAP32_SC=4 -DRAP32_CL=2 -DRAP32_MINB=1"
b /tmp/f_2x2c8.so "-DRAP32_SR=2 -DRAP32_SC=2 -DRAP32_CL=8 -DRAP32_MINB=4"
b /tmp/f_m3.so "-DRAP32_MINB=3"
b /tmp/f_4x4c4.so "-DRAP32_SC=4 -DRAP32_CL=4 -DRAP32_MINB=1"
b /tmp/f_def.so ""
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/f_def.so:rap /tmp/f_c8.so:rap /tmp/f_4x4c2.so:rap \
    /tmp/f_2x2c8.so:rap /tmp/f_m3.so:rap /tmp/f_4x4c4.so:rap 2>&1 | tee "$OUT/ab32s2.txt"
