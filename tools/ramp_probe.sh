python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 100 python tools/pcie2d_probe.py 2>&1 | tail -5
for d in 0 2 4 16; do
  RAP_EXTRA_NVCC_FLAGS="-DRAP_HOST_RAMP_DIV=$d" python -c "from paper_conf_icppw_nakanomi14_b200 import build as b; b.build(force=True)" >/dev/null 2>&1
  echo "ramp div $d"; timeout 100 python tools/e2e_probe.py 2>&1 | grep -E "ws MiB (64|128)"
done
