for d in 0 512 1024 1536; do
  rm -f gpurun_out/tr.*
  CKPT_DBG=$d CKPT_TRACE=gpurun_out/tr K=6 python tools/profile_step.py > /dev/null 2>&1
  echo "dbg=$d"; python tools/trace_kernels.py gpurun_out/tr | tail -6
  CKPT_DBG=$d K=12 python tools/profile_step.py 2>&1 | grep "loop prof=False"
done
