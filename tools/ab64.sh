#!/bin/bash
# A/B of the cfg4 kernels: 8-byte-slot RAP with LDG.128 row-pair groups vs one LDG.64 per row,
# a few CTA shapes, against RAP-16 and the two-plane RAP2P (tools/ab_lib.py, interleaved rounds).
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {   # build librap.so with extra flags and copy it to $1
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/l_groups.so "-DRAP64_ROWS=0"
b /tmp/l_sr8.so "-DRAP64_SR=8"
b /tmp/l_sr13.so "-DRAP64_SR=13"
b /tmp/l_rows.so ""
python tools/ab_lib.py --rounds 9 --libs /tmp/l_rows.so:rap /tmp/l_groups.so:rap /tmp/l_sr8.so:rap /tmp/l_sr13.so:rap \
   /tmp/l_rows.so:rap16 /tmp/l_rows.so:rap2p /tmp/l_rows.so:pad /tmp/l_rows.so:xor /tmp/l_rows.so:raw 2>&1 | tee "$OUT/ab64.txt"
