#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_contract.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 1500 python tools/sweep.py --only 4 --k 30 --out gpurun_out/sw4.json > gpurun_out/sw4.log 2>&1; echo "sw4 rc=$?"
python - <<'PY'
import json
for r in json.load(open('gpurun_out/sw4.json')):
    print(r['case'], 'dev', r['device_ms_steady_mean'], 'wall', r['wall_ms_steady_mean'], 'wall_med', r['wall_ms_steady_median'], r['host_ms_steady_mean'], 'growths', r['table_growths'], 'pre_max', r['host_pre_ms_max'], 'tab_max', r['host_table_growth_ms_max'], 'arena_max', r['host_arena_growth_ms_max'], 'steady_gbs', r['steady_gbs'], 'wall_gbs', r['steady_wall_gbs'])
PY
timeout 600 python bench.py --no-cpu-baseline --p 0.05 --e2e-steps 1 > gpurun_out/bench_p5.log 2>&1; echo "bench p5 rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_p5.log').read().strip().splitlines()[-1])
print('bench p5', d['value'], d['ms_per_step'], d['phase_ms'])"
