K=4 ncu --set full --import-source on --clock-control none -k regex:gather_kernel --launch-skip 3 --launch-count 1 \
  -o gpurun_out/gather_full -f python tools/ncu_driver.py > gpurun_out/ncu_gather.log 2>&1
ncu -i gpurun_out/gather_full.ncu-rep --page raw --csv > gpurun_out/gather_raw.csv 2>/dev/null
tail -2 gpurun_out/ncu_gather.log
