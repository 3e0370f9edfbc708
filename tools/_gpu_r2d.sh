#!/bin/bash
# K1 insert warp (batched, backlog to K1b): parity subset, bench p=1% and p=5%, trace.
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_contract.py tests/test_gpu_import.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for P in 0.01 0.05 0.001; do
timeout 600 python bench.py --no-cpu-baseline --p $P --e2e-steps 1 > gpurun_out/bench_p$P.log 2>&1; echo "bench p=$P rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_p$P.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms'])"
done
CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > gpurun_out/trace_step.log 2>&1; echo "trace rc=$?"
python tools/trace_kernels.py gpurun_out/tr > gpurun_out/trace_kernels.txt 2>&1; cat gpurun_out/trace_kernels.txt
python tools/trace_view.py gpurun_out/tr > gpurun_out/trace_view.txt 2>&1; tail -6 gpurun_out/trace_view.txt
