#!/bin/bash
# GPU parity tests, default bench, config-4 and config-2 p=5% cases of the sweep (prof 2 breakdown)
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms'])"
timeout 900 python tools/sweep.py --only 4 --k 12 --prof 2 --out gpurun_out/sw4.json > gpurun_out/sw4.log 2>&1; echo "sw4 rc=$?"
python -c "
import json
for r in json.load(open('gpurun_out/sw4.json')): print(r['case'], r['steady_ms_median'], r.get('phase_ms_steady_mean'), r['restore_ok'])"
