"""Minimal steady-state driver for ncu: config-2 lineage (1 GiB, C=128, p=1%), K checkpoints.
Profile the LAST checkpoint's kernels with --launch-skip (K-1) per kernel regex."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, p = int(os.environ.get("B", 1 << 30)), int(os.environ.get("C", 128)), float(os.environ.get("P", 0.01))
K = int(os.environ.get("K", 4))
seed = W.seed_of(2)
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
W.DeviceGen.initial(2, bufs[0], B, seed)
for k in range(1, K):
    bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, p)
torch.cuda.synchronize()
ck = Checkpointer(C)
for k in range(K):
    d = ck.checkpoint(bufs[k])
print(d)
