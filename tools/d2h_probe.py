import os, sys, time
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C = 1 << 30, 128
st = torch.cuda.Stream()
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(3)]
with torch.cuda.stream(st):
    W.DeviceGen.initial(2, bufs[0], B, 1, st)
    for k in (1, 2):
        bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(2, bufs[k], B, k, C, 1, 0.01, st)
st.synchronize()
ck = Checkpointer(C)
ds = [ck.checkpoint(b, stream=st) for b in bufs]
n = ds[2]["bytes"]
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d2h = torch.cuda.Stream()
for rep in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(d2h)
    for i in range(20):
        ck.diff_to_host_async(2, h, d2h, nbytes=n)
    e1.record(d2h); d2h.synchronize()
    print(f"arena diff D2H {n/1e6:.1f} MB: {20 * n / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s", flush=True)
t = torch.empty(n, dtype=torch.uint8, device="cuda")
for rep in range(2):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(d2h):
        e0.record(d2h)
        for i in range(20):
            h.copy_(t, non_blocking=True)
        e1.record(d2h)
    d2h.synchronize()
    print(f"cudaMalloc D2H: {20 * n / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s", flush=True)
big = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); hb = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with torch.cuda.stream(d2h):
    e0.record(d2h); hb.copy_(big, non_blocking=True); e1.record(d2h)
d2h.synchronize()
print(f"256 MB D2H: {(256 << 20) / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s")
