#!/bin/bash
# config 4 and config 2 p=5% with host timers (wall vs device), table growth counts
timeout 1500 python tools/sweep.py --only 4 --k 30 --out gpurun_out/sw4.json > gpurun_out/sw4.log 2>&1; echo "sw4 rc=$?"
python - <<'PY'
import json
for r in json.load(open('gpurun_out/sw4.json')):
    print(r['case'], 'dev', r['device_ms_steady_mean'], 'wall', r['wall_ms_steady_mean'], 'wall_med', r['wall_ms_steady_median'], r['host_ms_steady_mean'], 'growths', r['table_growths'], 'steady_gbs', r['steady_gbs'], 'wall_gbs', r['steady_wall_gbs'], 'gen_s', r['gen_s'])
PY
