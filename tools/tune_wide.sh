#!/bin/bash
# Register budget sweep of the warp-per-trial wide sweep (32 < w <= 256): min CTAs per SM.
for m in ${VARIANTS:-1 2 3 4}; do
  RAP_EXTRA_NVCC_FLAGS="-DRAP_WIDE_MINB=$m" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
  echo "minb=$m"; timeout 100 python tools/wide_rate.py 2>&1 | grep -E "w=(64|128|256)"
done
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)"
