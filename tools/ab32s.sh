#!/bin/bash
# A/B of fp32 cluster sizes (PDL off), cfg3 8192^2 and 16384^2 fp32
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/f_c8.so "-DRAP32_CL=8"
b /tmp/f_c16.so "-DRAP32_CL=16"
b /tmp/f_8x2c8.so "-DRAP32_SR=8 -DRAP32_CL=8 -DRAP32_MINB=1"
b /tmp/f_4x1c16.so "-DRAP32_SC=1 -DRAP32_CL=16 -DRAP32_MINB=4"
b /tmp/f_2x2c16.so "-DRAP32_SR=2 -DRAP32_CL=16 -DRAP32_MINB=4"
b /tmp/f_def.so ""
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/f_def.so:rap /tmp/f_c8.so:rap /tmp/f_c16.so:rap \
    /tmp/f_8x2c8.so:rap /tmp/f_4x1c16.so:rap /tmp/f_2x2c16.so:rap 2>&1 | tee "$OUT/ab32s3.txt"
python tools/ab_lib.py --rounds 7 --n 16384 --dtype f32 --libs /tmp/f_def.so:rap /tmp/f_c8.so:rap /tmp/f_c16.so:rap \
    /tmp/f_8x2c8.so:rap 2>&1 | tee "$OUT/ab32s3_16k.txt"
