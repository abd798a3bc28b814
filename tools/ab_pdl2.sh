#!/bin/bash
# A/B (longer): programmatic dependent launch on / off, cfg3 fp32 and cfg4 fp64, three layouts
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/d_nopdl.so "-DRAP_PDL=0"
b /tmp/d_def.so ""
python tools/ab_lib.py --rounds 21 --n 8192 --dtype f32 --libs /tmp/d_def.so:rap /tmp/d_nopdl.so:rap /tmp/d_def.so:pad /tmp/d_nopdl.so:pad 2>&1 | tee "$OUT/ab_pdl32b.txt"
python tools/ab_lib.py --rounds 15 --libs /tmp/d_def.so:rap /tmp/d_nopdl.so:rap /tmp/d_def.so:rap16 /tmp/d_nopdl.so:rap16 2>&1 | tee "$OUT/ab_pdl64b.txt"
