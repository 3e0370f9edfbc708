import os, sys, statistics
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, p, K = 1 << 30, 128, float(os.environ.get("P", 0.01)), 16
seed = W.seed_of(2)
st = torch.cuda.Stream()
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
with torch.cuda.stream(st):
    W.DeviceGen.initial(2, bufs[0], B, seed, st)
    for k in range(1, K):
        bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, p, st)
st.synchronize()
ck = Checkpointer(C); ck.set_profiling(2)
pend = []
for k in range(K):
    pend.append(ck.submit(bufs[k], stream=st))
    if len(pend) >= 2: ck.wait(pend.pop(0), stream=st)
while pend: ck.wait(pend.pop(0), stream=st)
st.synchronize()
rows = [ck.phase_times(k) for k in range(4, K)]
for key in ("leaf_hash", "insert", "phase2", "phase3", "compact", "total"):
    print(key, round(statistics.median(r[key] for r in rows), 4))
