"""A/B of library builds on the config-2 lineage: python tools/ab_k1.py lib1.so lib2.so ...
Each build runs in its own process (CKPT_LIB); prints median K1 and whole-call event times."""
import json, os, subprocess, sys

CHILD = r'''
import os, sys, json, statistics
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, p, K = int(os.environ.get("B", 1 << 30)), int(os.environ.get("C", 128)), float(os.environ.get("P", 0.01)), 14
cfg = int(os.environ.get("CFG", 2))
seed = W.seed_of(cfg)
st = torch.cuda.Stream()
K = int(os.environ.get("K", K))
bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
if cfg == 4:
    g = W.DupHeavy(B, C, seed)
    for k in range(K):
        bufs[k].copy_(torch.from_numpy(g.next()))
    torch.cuda.synchronize()
else:
    with torch.cuda.stream(st):
        W.DeviceGen.initial(cfg, bufs[0], B, seed, st)
        for k in range(1, K):
            bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(cfg, bufs[k], B, k, C, seed, p, st)
    st.synchronize()
prof = int(os.environ.get("PROF", 1))
res = {}
for rep in range(2):
    ck = Checkpointer(C); ck.set_profiling(prof)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for k in range(3): ck.checkpoint(bufs[k], stream=st)
    e0.record(st)
    for k in range(3, K): ck.checkpoint(bufs[k], stream=st, raw=True)
    e1.record(st); st.synchronize()
    k1 = [ck.phase_times(k)["leaf_hash"] for k in range(3, K)]
    tot = [ck.phase_times(k)["total"] for k in range(3, K)]
    res = {"k1_ms": round(statistics.median(k1), 4), "call_ms": round(statistics.median(tot), 4),
           "loop_ms_per_step": round(e0.elapsed_time(e1) / (K - 3), 4)}
    if prof >= 2:
        for ph in ("insert", "phase2", "phase3", "compact"):
            res[ph] = round(statistics.median([ck.phase_times(k)[ph] for k in range(3, K)]), 4)
    ck.close()
print("RESULT", json.dumps(res))
'''

for lib in sys.argv[1:]:
    env = dict(os.environ, CKPT_LIB=os.path.abspath(lib))
    out = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
    line = [l for l in out.stdout.splitlines() if l.startswith("RESULT")]
    print(os.path.basename(lib), line[0][7:] if line else out.stderr[-400:], flush=True)
