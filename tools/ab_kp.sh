#!/bin/bash
# 32-bit transposes through row-pair planes (RAP32_KP): parity tests of that build, then an
# interleaved A/B against the default 32-bit kernel (cfg3 8192^2 and 16384^2 fp32)
set -u
OUT=${1:-gpurun_out}
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/k_6.so "-DRAP32_KP=1 -DRAP32_KP_SR=6 -DRAP32_KP_MINB=2"
b /tmp/k_4c4.so "-DRAP32_KP=1 -DRAP32_KP_SR=4 -DRAP32_KP_CL=4 -DRAP32_KP_MINB=3"
b /tmp/k_def.so ""
b /tmp/k_12.so "-DRAP32_KP=1"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "transpose and not host and not 2pow32 and not aspect" > "$OUT/kp_pytest.log" 2>&1
tail -2 "$OUT/kp_pytest.log"
python tools/ab_lib.py --rounds 11 --n 8192 --dtype f32 --libs /tmp/k_def.so:rap /tmp/k_12.so:rap /tmp/k_6.so:rap /tmp/k_4c4.so:rap \
    /tmp/k_12.so:xor /tmp/k_12.so:pad 2>&1 | tee "$OUT/ab_kp.txt"
python tools/ab_lib.py --rounds 7 --n 16384 --dtype f32 --libs /tmp/k_def.so:rap /tmp/k_12.so:rap /tmp/k_6.so:rap /tmp/k_4c4.so:rap 2>&1 | tee "$OUT/ab_kp_16k.txt"
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1
