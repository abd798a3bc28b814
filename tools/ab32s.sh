#!/bin/bash
# A/B of fp32 CTA / cluster shapes (PDL off), cfg3 8192^2 and a 16384^2 fp32 matrix
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/f_12a.so "-DRAP32_SR=12 -DRAP32_SC=1 -DRAP32_CL=1 -DRAP32_MINB=1"
b /tmp/f_12b.so "-DRAP32_SR=12 -DRAP32_SC=1 -DRAP32_CL=1 -DRAP32_MINB=2"
b /tmp/f_8c2.so "-DRAP32_SR=8 -DRAP32_SC=1 -DRAP32_CL=2 -DRAP32_MINB=2"
b /tmp/f_16.so "-DRAP32_SR=16 -DRAP32_SC=1 -DRAP32_CL=1 -DRAP32_MINB=1"
b /tmp/f_4x2c2.so "-DRAP32_CL=2"
b /tmp/f_def.so ""
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/f_def.so:rap /tmp/f_12a.so:rap /tmp/f_12b.so:rap \
    /tmp/f_8c2.so:rap /tmp/f_16.so:rap /tmp/f_4x2c2.so:rap 2>&1 | tee "$OUT/ab32s.txt"
python tools/ab_lib.py --rounds 7 --n 16384 --dtype f32 --libs /tmp/f_def.so:rap /tmp/f_12a.so:rap /tmp/f_12b.so:rap \
    /tmp/f_8c2.so:rap /tmp/f_16.so:rap /tmp/f_4x2c2.so:rap 2>&1 | tee "$OUT/ab32s_16k.txt"
