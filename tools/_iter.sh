#!/bin/bash
# quick iteration on the GPU box: cfg4 + cfg2 per-phase breakdown, traces, bench line
timeout 300 python tools/sweep.py --only 4 --prof 2 --k 8 --out gpurun_out/it_cfg4.json > gpurun_out/it4.log 2>&1
timeout 300 python tools/sweep.py --only 2 --prof 2 --k 10 --out gpurun_out/it_cfg2.json > gpurun_out/it2.log 2>&1
python -c "
import json
for f in ['gpurun_out/it_cfg4.json','gpurun_out/it_cfg2.json']:
    for r in json.load(open(f)): print(r['case'], r['steady_ms_median'], r['phase_ms_steady_mean'], 'restore', r['restore_last_gbs'], r['restore_ok'])
"
rm -f gpurun_out/tr4.*; CFG=4 K=4 CKPT_TRACE=gpurun_out/tr4 timeout 300 python tools/profile_step.py > /dev/null 2>&1
python tools/trace_kernels.py gpurun_out/tr4; python tools/trace_view.py gpurun_out/tr4 2>&1 | tail -6
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('BENCH', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'], d['roofline']['k1_ms'], d['restore'])"
