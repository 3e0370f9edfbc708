"""Per-call breakdown of ckpt_checkpoint on the GPU box (wall vs device span vs phases)."""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W

B, C, p = int(os.environ.get("B", 1 << 30)), int(os.environ.get("C", 128)), float(os.environ.get("P", 0.01))
K = int(os.environ.get("K", 10))
CFG = int(os.environ.get("CFG", 2))
seed = W.seed_of(CFG)
st = torch.cuda.Stream()
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
if CFG == 4:   # duplicate-heavy: host generator
    g = W.DupHeavy(B, C, seed)
    for k in range(K):
        bufs[k].copy_(torch.from_numpy(g.next()))
else:
    with torch.cuda.stream(st):
        W.DeviceGen.initial(CFG, bufs[0], B, seed, st)
        for k in range(1, K):
            bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(CFG, bufs[k], B, k, C, seed, p, st)
torch.cuda.synchronize()
st.synchronize()
for prof in (True, False):
    ck = Checkpointer(C)
    ck.set_profiling(prof)
    rows = []
    for k in range(K):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(st)
        d = ck.checkpoint(bufs[k], stream=st)
        e1.record(st)
        t1 = time.perf_counter()
        e1.synchronize()
        rows.append(dict(k=k, wall_ms=round(1e3 * (t1 - t0), 3), span_ms=round(e0.elapsed_time(e1), 3),
                         phases={k: round(v, 4) for k, v in ck.phase_times().items()}, nF=d["n_first_regions"], nS=d["n_shift_regions"],
                         cand=d["n_first"] + d["n_spatial"] + d["n_temporal"], bytes=d["bytes"]))
    for r in rows:
        print(json.dumps(r))
    # back-to-back loop
    t0 = time.perf_counter(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    ck2 = Checkpointer(C); ck2.set_profiling(prof)
    ck2.checkpoint(bufs[0], stream=st)
    e0.record(st); t0 = time.perf_counter()
    for k in range(1, K):
        ck2.checkpoint(bufs[k], stream=st)
    e1.record(st); e1.synchronize(); t1 = time.perf_counter()
    print("loop prof=%s: wall %.3f ms/step, events %.3f ms/step" % (prof, 1e3 * (t1 - t0) / (K - 1), e0.elapsed_time(e1) / (K - 1)))
    ck.close(); ck2.close()
