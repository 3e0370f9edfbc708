#!/bin/bash
L=paper_conf_icpp_tanlmtmbctn23_b200
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_contract.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for P in 0.01 0.05 0.001; do
echo "P=$P prof1"; P=$P PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt.so $L/libckpt_noins.so $L/libckpt_ring8.so
done
echo "P=0.01 prof2"; P=0.01 PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt.so $L/libckpt_noins.so
