#!/bin/bash
L=paper_conf_icpp_tanlmtmbctn23_b200
for P in 0.01 0.05; do
echo "P=$P prof2"; P=$P PROF=2 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt_ku1.so $L/libckpt.so $L/libckpt_ku4.so
done
echo "cfg4 prof2"; CFG=4 K=10 PROF=2 timeout 900 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt_ku1.so $L/libckpt.so $L/libckpt_ku4.so
