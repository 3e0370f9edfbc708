#!/bin/bash
# A/B of library builds on one gpurun call: GPU parity, then tools/ab_k1.py on config 2 (p = 1 %, 5 %),
# C = 32 and config 4, then the bench line, for every .so given (default: libckpt_base.so libckpt.so).
# Build the variants first, e.g.  python -c "from paper_conf_icpp_tanlmtmbctn23_b200 import _build;
# _build.build_variant('libckpt_base.so', [])"  from the reference commit (git stash).
L=paper_conf_icpp_tanlmtmbctn23_b200
LIBS=${LIBS:-"$L/libckpt_base.so $L/libckpt.so"}
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for P in 0.01 0.05; do echo "P=$P prof2"; P=$P PROF=2 timeout 600 python tools/ab_k1.py $LIBS; done
echo "C=32 prof1"; C=32 PROF=1 timeout 600 python tools/ab_k1.py $LIBS
echo "cfg4 prof1"; CFG=4 K=10 PROF=1 timeout 900 python tools/ab_k1.py $LIBS
for lib in $LIBS; do
  CKPT_LIB=$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_ab.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/bench_ab.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'])"
done
