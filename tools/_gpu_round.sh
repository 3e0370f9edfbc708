#!/bin/bash
# One gpurun call: GPU parity tests, smoke, default bench, ncu launch list of the bench, ncu full capture, sweep.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench.log | cut -c1-600
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
python tools/launches.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1
grep ckpt gpurun_out/launches.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"leaf_hash|insert_kernel|tree_kernel|gather|paint" -s 10 -c 6 -o gpurun_out/prof -f python tools/ncu_driver.py > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
python tools/ncu_summarize.py gpurun_out/prof.ncu-rep gpurun_out/ncu_summary.json > gpurun_out/ncu_full.txt 2>&1
cat gpurun_out/ncu_full.txt
if [ "$SWEEP" = "1" ]; then timeout 1500 python tools/sweep.py > gpurun_out/sweep.log 2>&1; echo "sweep rc=$?"; fi
timeout 900 python tools/oracle_time.py --out gpurun_out/oracle_time.json > gpurun_out/oracle_time.log 2>&1; echo "oracle_time rc=$?"
