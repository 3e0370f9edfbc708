for d in 0 2048; do
  rm -f gpurun_out/tr.*
  CKPT_DBG=$d CKPT_TRACE=gpurun_out/tr K=6 python tools/profile_step.py > /dev/null 2>&1
  echo "dbg=$d"; python tools/trace_kernels.py gpurun_out/tr | tail -2
  python - <<'PY'
import numpy as np
a=np.fromfile("gpurun_out/tr.5.bin",dtype=np.uint64).reshape(-1,4).astype(np.int64)
g=a[a[:,3]==77]
print("prefix",np.percentile((g[:,1]-g[:,0])/1e3,[50,90,100]).round(2),"rest",np.percentile((g[:,2]-g[:,1])/1e3,[50,90,99,100]).round(2))
PY
done
