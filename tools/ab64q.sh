#!/bin/bash
# the three 64-bit RAP encodings with PDL off (default build), cfg4 16384^2 and 11584^2 float64
set -u
OUT=${1:-gpurun_out}
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1
cp paper_conf_icppw_nakanomi14_b200/librap.so /tmp/q_def.so
python tools/ab_lib.py --rounds 15 --libs /tmp/q_def.so:rap /tmp/q_def.so:rap64 /tmp/q_def.so:rap16 2>&1 | tee "$OUT/ab64q.txt"
python tools/ab_lib.py --rounds 15 --libs /tmp/q_def.so:rap64 /tmp/q_def.so:rap16 /tmp/q_def.so:rap 2>&1 | tee "$OUT/ab64q_rev.txt"
python tools/ab_lib.py --rounds 9 --n 11584 --libs /tmp/q_def.so:rap /tmp/q_def.so:rap64 /tmp/q_def.so:rap16 2>&1 | tee "$OUT/ab64q_11k.txt"
