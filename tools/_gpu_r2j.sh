#!/bin/bash
timeout 1200 python -m pytest tests/test_gpu_shift_insert.py -m gpu -x -q > gpurun_out/pytest_si.log 2>&1; echo "pytest si rc=$?"; tail -30 gpurun_out/pytest_si.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
