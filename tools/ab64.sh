#!/bin/bash
# A/B of build variants (tools/ab_lib.py, interleaved rounds).  cfg4: the 8-byte-slot RAP kernel
# (default build, and capped at 160 registers) against RAP-16 / two-plane RAP; cfg3: CTA / cluster shapes
# of the fp32 kernel with allocating loads + PDL.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {   # build librap.so with extra flags and copy it to $1
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/l_def.so ""
b /tmp/l_r160.so "-maxrregcount=160"
b /tmp/l_8x2.so "-DRAP32_SR=8 -DRAP32_SC=2 -DRAP32_CL=1 -DRAP32_MINB=1"
b /tmp/l_cl2.so "-DRAP32_CL=2"
b /tmp/l_cl1.so "-DRAP32_CL=1"
b /tmp/l_4x1.so "-DRAP32_SC=1 -DRAP32_MINB=4"
b /tmp/l_m3.so "-DRAP32_MINB=3"
python tools/ab_lib.py --rounds 11 --libs /tmp/l_def.so:rap64 /tmp/l_r160.so:rap64 /tmp/l_def.so:rap16 /tmp/l_def.so:rap 2>&1 | tee "$OUT/ab64f.txt"
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/l_def.so:rap /tmp/l_8x2.so:rap /tmp/l_cl2.so:rap /tmp/l_cl1.so:rap \
    /tmp/l_4x1.so:rap /tmp/l_m3.so:rap /tmp/l_def.so:pad /tmp/l_def.so:xor 2>&1 | tee "$OUT/ab32f.txt"
