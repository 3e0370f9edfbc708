#!/bin/bash
# Baseline: GPU tests, bench, in-kernel trace of config-2 steady checkpoints, host gap probe.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-400
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms'])"
CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > gpurun_out/trace_step.log 2>&1; echo "trace rc=$?"
python tools/trace_kernels.py gpurun_out/tr > gpurun_out/trace_kernels.txt 2>&1; cat gpurun_out/trace_kernels.txt
python tools/trace_view.py gpurun_out/tr > gpurun_out/trace_view.txt 2>&1; tail -6 gpurun_out/trace_view.txt
timeout 300 python tools/gap_probe.py > gpurun_out/gap.log 2>&1; echo "gap rc=$?"; tail -5 gpurun_out/gap.log
