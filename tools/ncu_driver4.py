"""Steady-state driver for ncu on config 4 (duplicate-heavy, host generator, 1 GiB, C = 128):
K checkpoints; profile the last checkpoint's kernels with --launch-skip."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, K = int(os.environ.get("B", 1 << 30)), int(os.environ.get("C", 128)), int(os.environ.get("K", 4))
g = W.DupHeavy(B, C, W.seed_of(4))
buf = torch.empty(B, dtype=torch.uint8, device="cuda")
ck = Checkpointer(C)
for k in range(K):
    buf.copy_(torch.from_numpy(g.next()))
    torch.cuda.synchronize()
    d = ck.checkpoint(buf)
print({x: d[x] for x in ("n_first", "n_temporal", "n_fixed", "n_first_regions", "n_shift_regions", "record_size",
                         "record_capacity")})
