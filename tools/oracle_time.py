#!/usr/bin/env python
"""Times the CPU oracle (as it stands: single-threaded C++, 1 core) per checkpoint on the
BASELINE configs it is planned for, on the host it runs on.

    python tools/oracle_time.py [--out gpurun_out/oracle_time.json]

  config 1: 1 MiB, C = 128, 10 checkpoints (the whole lineage)
  config 2: 1 GiB GDV-like, C = 128, p = 1 %, checkpoint 0 + 4 steady checkpoints
  config 4: duplicate-heavy at 64 MiB (host generator), C = 128, 10 checkpoints

Checkpoint 0 is reported separately; steady = mean over k >= 1. Inputs come from the
harness generators (host recipe; config 2 from the device twin when a GPU is present, the
same bytes). Test infrastructure: only reads oracle/, never the product path.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


def time_lineage(name, bufs, C):
    import oracle
    o = oracle.Oracle(C)
    ts = []
    for b in bufs:
        t0 = time.perf_counter()
        o.checkpoint(b)
        ts.append(time.perf_counter() - t0)
    B = bufs[0].size
    st = ts[1:]
    return {"case": name, "buffer_bytes": int(B), "chunk_bytes": C, "checkpoints": len(bufs),
            "ckpt0_s": round(ts[0], 4), "steady_s_mean": round(sum(st) / max(1, len(st)), 4),
            "steady_gbs": round(len(st) * B / max(1e-12, sum(st)) / 1e9, 4), "cores": 1}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "oracle_time.json"))
    a = ap.parse_args()
    import numpy as np
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    recs = []
    recs.append(time_lineage("cfg1_1MiB", [np.array(b) for b in W.lineage(1, 1 << 20, 128, 10)], 128))
    B2, K2, p2 = 1 << 30, 5, 0.01
    try:
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError
        t = torch.empty(B2, dtype=torch.uint8, device="cuda")
        seed = W.seed_of(2)
        W.DeviceGen.initial(2, t, B2, seed)
        bufs = [t.cpu().numpy()]
        for k in range(1, K2):
            W.DeviceGen.mutate(2, t, B2, k, 128, seed, p2)
            bufs.append(t.cpu().numpy())
        del t
    except Exception:
        bufs = [np.array(b) for b in W.lineage(2, B2, 128, K2, p=p2)]
    recs.append(time_lineage("cfg2_1GiB_p0.01", bufs, 128))
    del bufs
    recs.append(time_lineage("cfg4_64MiB", [np.array(b) for b in W.lineage(4, 64 << 20, 128, 10)], 128))
    host = {"cpu_model": cpu_model(), "nproc": os.cpu_count(), "threads_used": 1}
    out = {"host": host, "cases": recs}
    print(json.dumps(out))
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
