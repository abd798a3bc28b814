#!/bin/bash
# A/B of the two-plane fp64 (cfg4 RAP) CTA / cluster shapes with allocating loads + PDL
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/p_6c2.so "-DRAP64P_SR=6 -DRAP64P_CL=2 -DRAP64P_MINB=2"
b /tmp/p_4c4.so "-DRAP64P_SR=4 -DRAP64P_CL=4 -DRAP64P_MINB=3"
b /tmp/p_6c1.so "-DRAP64P_SR=6 -DRAP64P_MINB=2"
b /tmp/p_12c2.so "-DRAP64P_SR=12 -DRAP64P_CL=2"
b /tmp/p_8c1.so "-DRAP64P_SR=8"
b /tmp/p_def.so ""
python tools/ab_lib.py --rounds 9 --libs /tmp/p_def.so:rap /tmp/p_6c2.so:rap /tmp/p_4c4.so:rap /tmp/p_6c1.so:rap \
    /tmp/p_12c2.so:rap /tmp/p_8c1.so:rap /tmp/p_def.so:rap16 2>&1 | tee "$OUT/ab64p.txt"
