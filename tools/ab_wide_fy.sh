python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "wide or table2" 2>&1 | tail -1
echo "lane-mode FY:"; timeout 100 python tools/wide_rate.py 2>&1 | grep -E "w= *(64|128|256)"
RAP_EXTRA_NVCC_FLAGS="-DRAP_WIDE_LANE_FY=0" python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1
echo "chain FY:"; timeout 100 python tools/wide_rate.py 2>&1 | grep -E "w= *(64|128|256)"
# restore the default library (the build stamp also forces this on the next build() call)
python -c "import sys; sys.path.insert(0, '.'); from paper_conf_icppw_nakanomi14_b200 import build; build.build(force=True)" >/dev/null 2>&1
