# ncu full capture of the last checkpoint's tree kernels (phase 2 and 3) with source correlation
K=4 ncu --set full --import-source on --clock-control none -k regex:tree_kernel --launch-skip 6 --launch-count 2 \
  -o gpurun_out/tree_full -f python tools/ncu_driver.py > gpurun_out/ncu_tree.log 2>&1
ncu -i gpurun_out/tree_full.ncu-rep --page raw --csv > gpurun_out/tree_raw.csv 2>/dev/null
ncu -i gpurun_out/tree_full.ncu-rep --page details --csv > gpurun_out/tree_details.csv 2>/dev/null
tail -3 gpurun_out/ncu_tree.log
