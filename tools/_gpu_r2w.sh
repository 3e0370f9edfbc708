#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for i in 1 2; do
for lib in libckpt_base.so libckpt.so; do
CKPT_LIB=$L/$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_$lib.$i.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_$lib.$i.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'], d['phase_ms']['total_replay'], d['paper_throughput']['ok'], d['restore']['ok'])"
done
done
