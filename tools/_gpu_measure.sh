#!/bin/bash
# Round-2 measurement pass: GPU tests, smoke, bench (config 2 pipelined and --sync, config 5 in place, config 1,
# reference arm), pipelined vs synchronous lineages (tools/pipe_probe.py),
# ncu launch list and full captures (config 2 steady + per-config), sweep (configs 2-5, variants, methods),
# oracle timing, in-kernel trace, sanitizers, random-sector probe of the record table's access pattern.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv,noheader
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/rand_probe tools/rand_probe.cu && timeout 300 /tmp/rand_probe > gpurun_out/rand_probe.txt 2>&1; echo "rand_probe rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-200
timeout 900 python bench.py --config 5 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg5.log 2>&1; echo "bench5 rc=$?"
timeout 600 python bench.py --config 1 --bytes 1048576 --no-cpu-baseline > gpurun_out/bench_cfg1.log 2>&1; echo "bench1 rc=$?"
timeout 600 python bench.py --impl reference --steps 4 --warmup 3 > gpurun_out/bench_ref.log 2>&1; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
python tools/launches.py gpurun_out/launches.csv > gpurun_out/launches.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"leaf_hash|insert_kernel|tree_kernel|gather" -s 10 -c 6 -o gpurun_out/prof -f python tools/ncu_driver.py > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
python tools/ncu_summarize.py gpurun_out/prof.ncu-rep gpurun_out/ncu_summary.json > gpurun_out/ncu_full.txt 2>&1; cat gpurun_out/ncu_full.txt
ncu -i gpurun_out/prof.ncu-rep --page details --csv > gpurun_out/ncu_details.csv 2>/dev/null; gzip -f gpurun_out/ncu_details.csv
bash tools/ncu_configs.sh > gpurun_out/ncu_configs.log 2>&1; echo "ncu configs rc=$?"
timeout 2400 python tools/sweep.py --out gpurun_out/sweep.json > gpurun_out/sweep.log 2>&1; echo "sweep rc=$?"
timeout 1500 python tools/sweep.py --variants --out gpurun_out/variants.json > gpurun_out/variants.log 2>&1; echo "variants rc=$?"
timeout 1500 python tools/sweep.py --methods --out gpurun_out/methods.json > gpurun_out/methods.log 2>&1; echo "methods rc=$?"
for a in "" "P=0.05" "P=0.001" "CFG=3 C=32 B=4294967296 K=8" "CFG=3 C=4096 B=4294967296 K=8" "CFG=3 C=128 B=4294967296 K=8" "CFG=4 K=12"; do
  env $a STEPS=1 REPS=1 timeout 600 python tools/pipe_probe.py 2>&1 | head -2 | cut -c1-300
done > gpurun_out/pipeline.txt 2>&1; echo "pipeline rc=$?"; cat gpurun_out/pipeline.txt | grep "sync"
timeout 600 python bench.py --sync --no-cpu-baseline > gpurun_out/bench_sync.log 2>&1; echo "bench sync rc=$?"
timeout 900 python tools/oracle_time.py --out gpurun_out/oracle_time.json > gpurun_out/oracle_time.log 2>&1; echo "oracle_time rc=$?"
CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > gpurun_out/trace_step.log 2>&1; echo "trace rc=$?"
python tools/trace_kernels.py gpurun_out/tr > gpurun_out/trace_kernels.txt 2>&1; cat gpurun_out/trace_kernels.txt
python tools/trace_view.py gpurun_out/tr > gpurun_out/trace_view.txt 2>&1; tail -6 gpurun_out/trace_view.txt
rm -f gpurun_out/tr.*.bin
rm -f gpurun_out/*.ncu-rep   # summaries kept; the reports would exceed gpurun's 64 MiB copy-back
# compute-sanitizer: closed on the GPU pool late in round 2 (the wrapper exits 86); the logs of the last pass
# where it ran are kept in profiles/sanitize_r2/
for t in memcheck racecheck synccheck; do
  big=1; [ $t != memcheck ] && big=0
  SAN_BIG=$big timeout 1500 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_driver.py > gpurun_out/sanitize_$t.log 2>&1; echo "sanitize $t rc=$?"; tail -1 gpurun_out/sanitize_$t.log
done
