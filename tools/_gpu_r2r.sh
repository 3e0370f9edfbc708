#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_modes.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
for C in 32 64 128; do
echo "C=$C prof1"; C=$C PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
done
