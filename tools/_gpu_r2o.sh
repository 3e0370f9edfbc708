#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shift_insert.py tests/test_gpu_modes.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
L=paper_conf_icpp_tanlmtmbctn23_b200
echo "P=0.01 prof2"; P=0.01 PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
echo "P=0.05 prof2"; P=0.05 PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
echo "cfg4 prof2"; CFG=4 K=10 PROF=2 timeout 900 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
echo "cfg4 prof1"; CFG=4 K=10 PROF=1 timeout 900 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so
