"""Where the time between two back-to-back checkpoints goes (host side), config 2.
Prints per-call means: Python wall of Checkpointer.checkpoint, the library's own host
phases (pre = entry -> first enqueue, enqueue, sync wait, post) and the device span."""
import os, sys, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, p, K = 1 << 30, 128, 0.01, 16
seed = W.seed_of(2)
st = torch.cuda.Stream()
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
with torch.cuda.stream(st):
    W.DeviceGen.initial(2, bufs[0], B, seed, st)
    for k in range(1, K):
        bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, p, st)
st.synchronize()
ck = Checkpointer(C)
ck.set_profiling(1)
for k in range(3):
    ck.checkpoint(bufs[k], stream=st)
walls, hp = [], []
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for k in range(3, K):
    t0 = time.perf_counter()
    ck.checkpoint(bufs[k], nbytes=B, stream=st, raw=True)
    walls.append(time.perf_counter() - t0)
    hp.append(ck.phase_times(k))
e1.record(st); st.synchronize()
n = K - 3
print("events ms/step %.4f" % (e0.elapsed_time(e1) / n))
print("python wall ms/call %.4f" % (1e3 * statistics.mean(walls)))
for key in ("total", "leaf_hash", "host_pre", "host_enqueue", "host_sync_wait", "host_post"):
    print("%-15s %.4f" % (key, statistics.mean(h[key] for h in hp)))

# A/B on fresh handles over the same lineage: raw C ABI call with prebuilt ctypes
# arguments vs Checkpointer.checkpoint (the binding's per-call Python cost)
import ctypes
from paper_conf_icpp_tanlmtmbctn23_b200 import ckpt as _ck
L = _ck.lib()
f = L.ckpt_checkpoint
sth = ctypes.c_void_p(st.cuda_stream)
ptrs = [ctypes.c_void_p(b.data_ptr()) for b in bufs]
nb = ctypes.c_uint64(B)
for rep in range(2):
    for kind in ("raw", "binding"):
        c2 = Checkpointer(C)
        c2.set_profiling(1)
        for k in range(3):
            c2.checkpoint(bufs[k], stream=st)
        outs = [_ck.CkptDiff() for _ in range(K)]
        hh = c2._h
        torch.cuda.synchronize()
        e0.record(st)
        if kind == "raw":
            for k in range(3, K):
                f(hh, ptrs[k], nb, sth, ctypes.byref(outs[k]))
        else:
            for k in range(3, K):
                c2.checkpoint(bufs[k], nbytes=B, stream=st, raw=True)
        e1.record(st); st.synchronize()
        print("%-8s events ms/step %.4f" % (kind, e0.elapsed_time(e1) / n))
        c2.close()
