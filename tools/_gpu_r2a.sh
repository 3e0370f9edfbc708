#!/bin/bash
# Round 2, first call: GPU parity (incl. the full-size cases), smoke, default bench, ncu launch list.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv
nproc; lscpu | grep "Model name"
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -25 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench.log | cut -c1-800
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
python tools/launches.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1
grep ckpt gpurun_out/launches.txt | head -30
