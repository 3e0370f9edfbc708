#!/bin/bash
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
python tools/ab_k1.py paper_conf_icpp_tanlmtmbctn23_b200/libckpt.so
rm -f gpurun_out/tr.*; CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > /dev/null 2>&1
python tools/trace_kernels.py gpurun_out/tr
python - <<'PY'
import numpy as np, glob
f=sorted(glob.glob('gpurun_out/tr.*.bin'))[-1]
a=np.fromfile(f,dtype=np.uint64).reshape(-1,4).astype(np.int64)
k1=a[a[:,3]==100]; t0=k1[:,0].min(); ex=(k1[:,2]-t0)/1e3
print('K1 block exit percentiles', np.percentile(ex,[0,5,50,95,100]).round(1))
PY
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('BENCH', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'], d['roofline']['k1_ms'], d['restore']['gbs'])"
timeout 300 python tools/sweep.py --only 4 --prof 2 --k 6 --out gpurun_out/it_cfg4.json 2>&1 | tail -1 | cut -c1-300
