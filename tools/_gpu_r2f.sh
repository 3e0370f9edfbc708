#!/bin/bash
L=paper_conf_icpp_tanlmtmbctn23_b200
for P in 0.01 0.05; do
echo "P=$P prof1"; P=$P PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt.so $L/libckpt_noins.so $L/libckpt_nopush.so $L/libckpt_noinsert.so $L/libckpt_poll1000.so
done
