"""A/B of library builds on restore: python tools/ab_restore.py lib1.so lib2.so ...
Each build runs in its own process (CKPT_LIB): a config-2 lineage (1 GiB, C = 128, p = 1 %,
K = 19) or config 4 (CFG=4, host generator, K = 10); restore(K-1) cold once, then warm
(median of 5, host wall time of the synchronous call), checked against the input."""
import json, os, subprocess, sys

CHILD = r'''
import os, sys, json, statistics, time
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
B, C, p = int(os.environ.get("B", 1 << 30)), 128, 0.01
cfg = int(os.environ.get("CFG", 2))
K = int(os.environ.get("K", 19 if cfg == 2 else 10))
seed = W.seed_of(cfg)
ck = Checkpointer(C)
buf = torch.empty(B, dtype=torch.uint8, device="cuda")
if cfg == 4:
    g = W.DupHeavy(B, C, seed)
for k in range(K):
    if cfg == 4:
        buf.copy_(torch.from_numpy(g.next()))
    elif k == 0:
        W.DeviceGen.initial(cfg, buf, B, seed)
    else:
        W.DeviceGen.mutate(cfg, buf, B, k, C, seed, p)
    torch.cuda.synchronize()
    ck.checkpoint(buf)
out = torch.empty_like(buf)
t0 = time.perf_counter(); ck.restore(K - 1, out); torch.cuda.synchronize(); cold = time.perf_counter() - t0
ok = bool(torch.equal(out, buf))
ts = []
for _ in range(5):
    out.zero_(); torch.cuda.synchronize()
    t0 = time.perf_counter(); ck.restore(K - 1, out); torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
ok = ok and bool(torch.equal(out, buf))
m = statistics.median(ts)
print("RESULT", json.dumps({"warm_ms": round(m * 1e3, 3), "warm_gbs": round(B / m / 1e9, 1), "cold_ms": round(cold * 1e3, 2), "ok": ok}))
'''

for lib in sys.argv[1:]:
    env = dict(os.environ, CKPT_LIB=os.path.abspath(lib))
    out = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
    line = [l for l in out.stdout.splitlines() if l.startswith("RESULT")]
    print(os.path.basename(lib), line[0][7:] if line else out.stderr[-400:], flush=True)
