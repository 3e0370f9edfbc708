#!/bin/bash
L=paper_conf_icpp_tanlmtmbctn23_b200
for C in 32 64; do
echo "C=$C prof1"; C=$C PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt.so $L/libckpt_c4a.so $L/libckpt_c4b.so $L/libckpt_c3s.so
done
