#!/bin/bash
# A/B of the cfg2 sweep kernel builds (tools/ab_sweep.py, interleaved rounds, 5e7 trials per launch):
# shared-memory bank counters (RAP_SWEEP_SMEM_BANKS) vs ballots, and register budgets.
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
b() {
  RAP_EXTRA_NVCC_FLAGS="$2" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1 && cp paper_conf_icppw_nakanomi14_b200/librap.so $1
}
b /tmp/s_ballot.so "-DRAP_SWEEP_SMEM_BANKS=0"
b /tmp/s_m8.so "-DRAP_SWEEP_MINB=8"
b /tmp/s_m6.so "-DRAP_SWEEP_MINB=6"
b /tmp/s_def.so ""
python tools/ab_sweep.py --rounds 9 --libs /tmp/s_def.so /tmp/s_ballot.so /tmp/s_m8.so /tmp/s_m6.so 2>&1 | tee "$OUT/ab_sweep3.txt"
