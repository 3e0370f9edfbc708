#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py tests/test_gpu_modes.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for P in 0.01 0.05; do
echo "P=$P prof2"; P=$P PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
echo "P=$P prof1"; P=$P PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
done
echo "cfg4 prof2"; CFG=4 K=10 PROF=2 timeout 900 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
