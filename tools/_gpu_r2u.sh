#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for PR in 1 0; do
echo "P=0.01 prof$PR"; P=0.01 PROF=$PR timeout 600 python tools/ab_k1.py $L/libckpt_nopdl.so $L/libckpt.so $L/libckpt_nopdl.so $L/libckpt.so
done
for i in 1 2; do
for lib in libckpt_nopdl.so libckpt.so; do
CKPT_LIB=$L/$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_$lib.$i.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_$lib.$i.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'], d['roofline']['k1_ms'])"
done
done
