set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "transpose or perm" 2>&1 | tail -15
timeout 300 python bench.py --workload cfg4 --steps 20 --warmup 5 --no-e2e --no-cpu > gpurun_out/cfg4.json 2>gpurun_out/cfg4.err; tail -3 gpurun_out/cfg4.err
python -c "import json;d=json.load(open('gpurun_out/cfg4.json'));print(d['value'], d.get('layouts_gbs'), d['clocks'])"
timeout 300 python bench.py --workload layouts --steps 20 --warmup 5 --no-e2e --no-cpu > gpurun_out/layouts.json 2>&1
python -c "import json;d=json.load(open('gpurun_out/layouts.json'));print(d['value'], d.get('layouts_gbs'), d['clocks'])"
