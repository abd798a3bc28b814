#!/bin/bash
# band plan probe of rap_transpose_host (tools/e2e_bands.py): fill ramp on / off
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/e_noramp.so "-DRAP_HOST_RAMP_DIV=0"
b /tmp/e_def.so ""
python tools/e2e_bands.py /tmp/e_def.so /tmp/e_noramp.so 2>&1 | tee "$OUT/e2e_bands.txt"
