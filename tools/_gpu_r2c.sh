#!/bin/bash
# Round 2: K1 insert warp — full GPU suite, bench, p=5% case, in-kernel trace, memcheck.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms'], d['restore']['ok'], d['restart_import']['ok'])"
timeout 600 python bench.py --no-cpu-baseline --p 0.05 --e2e-steps 1 > gpurun_out/bench_p5.log 2>&1; echo "bench p5 rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_p5.log').read().strip().splitlines()[-1])
print('bench p5', d['value'], d['ms_per_step'], d['phase_ms'])"
CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > gpurun_out/trace_step.log 2>&1; echo "trace rc=$?"
python tools/trace_kernels.py gpurun_out/tr > gpurun_out/trace_kernels.txt 2>&1; cat gpurun_out/trace_kernels.txt
python tools/trace_view.py gpurun_out/tr > gpurun_out/trace_view.txt 2>&1; tail -6 gpurun_out/trace_view.txt
SAN_BIG=0 timeout 1200 compute-sanitizer --tool memcheck --print-limit 50 python tools/sanitize_driver.py > gpurun_out/sanitize_memcheck.log 2>&1; echo "sanitize memcheck rc=$?"; tail -4 gpurun_out/sanitize_memcheck.log
