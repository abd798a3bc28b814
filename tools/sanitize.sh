#!/bin/bash
# NOTE: compute-sanitizer is closed on the GPU pool (profiles/r02c_sanitizer_refused.txt); kept for other machines
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize.py (small calls of every kernel)
OUT=${1:-gpurun_out/r02_sanitizer.txt}
python -c "import __graft_entry__ as g; g.build()"
: > "$OUT"
for tool in memcheck racecheck synccheck; do
  echo "== compute-sanitizer --tool $tool python tools/sanitize.py" >> "$OUT"
  timeout 1200 compute-sanitizer --tool $tool python tools/sanitize.py 2>&1 | grep -E "workload done|SUMMARY|Error|error|Hazard|hazard" | head -40 >> "$OUT"
done
cat "$OUT"
