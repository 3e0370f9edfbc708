"""Synchronous vs pipelined (ckpt_checkpoint_submit / _wait) lineages: device time per
checkpoint over K steps (CUDA events on the caller's stream), config 2 or 4.
Env: CFG (2), C (128), P (0.01), B (1 GiB), K (16)."""
import os, sys
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W

B, C, p = int(os.environ.get("B", 1 << 30)), int(os.environ.get("C", 128)), float(os.environ.get("P", 0.01))
cfg, K, Wm = int(os.environ.get("CFG", 2)), int(os.environ.get("K", 16)), 3
seed = W.seed_of(cfg)
st = torch.cuda.Stream()
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K + Wm)]
if cfg == 4:
    g = W.DupHeavy(B, C, seed)
    for b in bufs:
        b.copy_(torch.from_numpy(g.next()))
else:
    with torch.cuda.stream(st):
        W.DeviceGen.initial(cfg, bufs[0], B, seed, st)
        for k in range(1, K + Wm):
            bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(cfg, bufs[k], B, k, C, seed, p, st)
torch.cuda.synchronize()


def sync_run():
    ck = Checkpointer(C)
    for k in range(Wm):
        ck.checkpoint(bufs[k], stream=st)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for k in range(Wm, Wm + K):
        ck.checkpoint(bufs[k], stream=st, raw=True)
    e1.record(st); st.synchronize()
    ck.close()
    return e0.elapsed_time(e1) / K


DEPTH = int(os.environ.get("DEPTH", 2))   # calls in flight (the library's CKPT_PIPELINE_DEPTH or less)


def pipe_run():
    ck = Checkpointer(C)
    pend = []
    for k in range(Wm):
        pend.append(ck.submit(bufs[k], stream=st))
        if len(pend) >= DEPTH: ck.wait(pend.pop(0), stream=st)
    while pend: ck.wait(pend.pop(0), stream=st)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for k in range(Wm, Wm + K):
        pend.append(ck.submit(bufs[k], stream=st))
        if len(pend) >= DEPTH: ck.wait(pend.pop(0), stream=st, raw=True)
    while pend: ck.wait(pend.pop(0), stream=st, raw=True)
    e1.record(st); st.synchronize()
    ck.close()
    return e0.elapsed_time(e1) / K


for rep in range(int(os.environ.get("REPS", 3))):
    s, q = sync_run(), pipe_run()
    print(f"cfg{cfg} C={C} p={p}: sync {s:.4f} ms ({B / s / 1e6:.0f} GB/s)  pipelined {q:.4f} ms ({B / q / 1e6:.0f} GB/s)", flush=True)

for _rep in range(int(os.environ.get("STEPS", 0))):
    import time
    ck = Checkpointer(C)
    pend = None
    evs, ht = [], []
    for k in range(Wm + K):
        t0 = time.perf_counter()
        cid = ck.submit(bufs[k], stream=st)
        t1 = time.perf_counter()
        if pend is not None:
            ck.wait(pend, stream=st, raw=True)
        t2 = time.perf_counter()
        e = torch.cuda.Event(enable_timing=True); e.record(st); evs.append(e)
        ht.append((1e3 * (t1 - t0), 1e3 * (t2 - t1)))
        pend = cid
    ck.wait(pend, stream=st)
    st.synchronize()
    dev = [evs[k - 1].elapsed_time(evs[k]) for k in range(1, len(evs))]
    print("device ms per step:", " ".join(f"{x:.3f}" for x in dev))
    print("host wait ms:", " ".join(f"{x[1]:.3f}" for x in ht[1:]))
    ck.close()
