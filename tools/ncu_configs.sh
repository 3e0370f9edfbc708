#!/bin/bash
# ncu --set full of one steady-state checkpoint per config (SURVEY §8(d) timing protocol):
# config 3 at C = 32 and C = 4096 (1 GiB), config 2 at p = 5 %, config 4 (duplicate-heavy), config 5 (16 GiB).
K='regex:leaf_hash|insert_kernel|tree_kernel|gather'
run() {  # name, env, driver
  env $2 timeout 1200 ncu --set full --clock-control none -k "$K" -s 15 -c 5 -o gpurun_out/ncu_$1 -f python $3 > gpurun_out/ncu_$1.log 2>&1
  echo "$1 rc=$?"
  python tools/ncu_summarize.py gpurun_out/ncu_$1.ncu-rep gpurun_out/ncu_$1.json > gpurun_out/ncu_$1.txt 2>&1
  cat gpurun_out/ncu_$1.txt
}
run cfg3_C32 "C=32 K=4" tools/ncu_driver.py
run cfg3_C4096 "C=4096 K=4" tools/ncu_driver.py
run cfg2_p5 "P=0.05 K=4" tools/ncu_driver.py
run cfg4 "K=4" tools/ncu_driver4.py
run cfg5_16GiB "B=17179869184 K=4" tools/ncu_driver.py
