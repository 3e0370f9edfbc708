#!/bin/bash
# Bench-only A/B of library builds on one gpurun call (uninstrumented calls: PDL overlap intact):
# GPU parity with the current build, then `bench.py` alternating between the builds R times.
L=paper_conf_icpp_tanlmtmbctn23_b200
LIBS=${LIBS:-"$L/libckpt_base.so $L/libckpt.so"}
R=${R:-3}
BENCH_ARGS=${BENCH_ARGS:-""}
if [ -z "$NO_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
fi
for r in $(seq $R); do
  for lib in $LIBS; do
    CKPT_LIB=$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 $BENCH_ARGS > gpurun_out/bench_ab.log 2>&1
    python -c "
import json; d=json.loads(open('gpurun_out/bench_ab.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'], d['e2e']['value'])" || tail -5 gpurun_out/bench_ab.log
  done
done
