#!/bin/bash
# K1 per chunk size, two builds (base: direct-load pass for C > 128 not a multiple of 128; new: TMA MODE3D 2)
L=paper_conf_icpp_tanlmtmbctn23_b200
for C in ${CS:-144 176 208 272 336 528 784 1040 1056 1088 1152 2064 2112 512 1024}; do echo "C=$C"; C=$C PROF=1 timeout 600 python tools/ab_k1.py $L/libckpt_base.so $L/libckpt.so; done
