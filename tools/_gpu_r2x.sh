#!/bin/bash
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_modes.py tests/test_gpu_variants.py tests/test_gpu_shift_insert.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for P in 0.01 0.05; do echo "P=$P prof2"; P=$P PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt_nolines.so $L/libckpt.so; done
echo "cfg4 prof2"; CFG=4 K=10 PROF=2 timeout 900 python tools/ab_k1.py $L/libckpt_nolines.so $L/libckpt.so
for lib in libckpt_nolines.so libckpt.so libckpt_nolines.so libckpt.so; do
CKPT_LIB=$L/$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_x.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_x.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'])"
done
