#!/bin/bash
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bw_probe tools/bw_probe.cu && timeout 120 /tmp/bw_probe > gpurun_out/bw_probe.txt 2>&1
cat gpurun_out/bw_probe.txt
rm -f gpurun_out/tr.*
CKPT_TRACE=gpurun_out/tr K=6 timeout 300 python tools/profile_step.py > gpurun_out/trace_step.log 2>&1
python tools/trace_kernels.py gpurun_out/tr > gpurun_out/trace_kernels.txt 2>&1; cat gpurun_out/trace_kernels.txt
python tools/trace_view.py gpurun_out/tr 2>&1 | tail -8
timeout 1500 python tools/sweep.py > gpurun_out/sweep.log 2>&1; echo "sweep rc=$?"
tail -3 gpurun_out/sweep.log | cut -c1-400
