#!/bin/bash
# Round 2: boundary-contract tests, bench (config 2 default; config 5 at 16 GiB in place), sanitizers.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,memory.total --format=csv
free -g | head -2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu_contract.py tests/test_bench_contract.py tests/test_gpu_import.py -m gpu -x -q > gpurun_out/pytest_contract.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_contract.log
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-300
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['phase_ms']); print('cpu', d['cpu_baseline'])"
timeout 900 python bench.py --config 5 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg5.log 2>&1; echo "bench cfg5 rc=$?"; tail -3 gpurun_out/bench_cfg5.log | cut -c1-1500
for t in memcheck racecheck synccheck; do
  big=1; [ $t != memcheck ] && big=0
  SAN_BIG=$big timeout 1200 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_driver.py > gpurun_out/sanitize_$t.log 2>&1; echo "sanitize $t rc=$?"; tail -4 gpurun_out/sanitize_$t.log
done
