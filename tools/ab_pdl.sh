#!/bin/bash
# A/B: early loads under PDL (opt-in build) vs PDL with the wait before the first load (default) vs no PDL
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/d_early.so "-DRAP_PDL_EARLY=1"
b /tmp/d_nopdl.so "-DRAP_PDL=0"
b /tmp/d_def.so ""
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/d_early.so:rap /tmp/d_def.so:rap /tmp/d_nopdl.so:rap \
    /tmp/d_def.so:xor 2>&1 | tee "$OUT/ab_pdl32.txt"
python tools/ab_lib.py --rounds 9 --libs /tmp/d_early.so:rap /tmp/d_def.so:rap /tmp/d_nopdl.so:rap /tmp/d_def.so:rap16 2>&1 | tee "$OUT/ab_pdl64.txt"
