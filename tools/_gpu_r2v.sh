#!/bin/bash
timeout 900 python -m pytest tests/test_bench_contract.py -m gpu -x -q > gpurun_out/pytest_bc.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_bc.log
for i in 1 2 3; do
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench.$i.log 2>&1; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench.$i.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms'], d['roofline']['k1_ms'], d['roofline']['frac'], d['gpu_launches'], d['checkpoint0'])"
done
