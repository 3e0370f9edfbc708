#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for P in 0.01 0.05; do
echo "P=$P prof1"; P=$P PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
done
echo "cfg4 prof1"; CFG=4 K=10 PROF=1 timeout 900 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'], d['restore']['ok'], d['restart_import']['ok'], d['paper_throughput'])"
