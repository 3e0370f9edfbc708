#!/bin/bash
L=paper_conf_icpp_tanlmtmbctn23_b200
for i in 1 2 3; do
for lib in libckpt_base.so libckpt.so; do
CKPT_LIB=$L/$lib timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_$lib.$i.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_$lib.$i.log').read().strip().splitlines()[-1])
print('$lib', d['value'], d['ms_per_step'], d['phase_ms']['total_timed'])"
done
done
echo "P=0.01 prof1"; P=0.01 PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so $L/libckpt_base.so $L/libckpt.so
