#!/bin/bash
# Session 2 of round 2: STS.128 result slots A/B (RAP_SWEEP_RES_VEC) + size-matched copy probe
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_vec.so "-DRAP_SWEEP_RES_VEC=1"
b /tmp/s_def.so ""
timeout 600 python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_vec.so > "$OUT/r02b_ab_resvec.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python tools/copy_probe.py > "$OUT/r02b_copy_probe.txt" 2>&1
