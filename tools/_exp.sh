for d in 0 128; do
  rm -f gpurun_out/tr.*
  CKPT_DBG=$d CKPT_TRACE=gpurun_out/tr K=6 python tools/profile_step.py > /dev/null 2>&1
  echo "dbg=$d"; python tools/trace_kernels.py gpurun_out/tr | tail -6
  CKPT_DBG=$d python bench.py --steps 40 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('BENCH', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'], d['roofline']['k1_ms'])"
done
