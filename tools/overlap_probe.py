"""Experiment: how much of the post-K1 chain could overlap the next K1? Two handles on two
streams, each checkpointing its own config-2 lineage from its own host thread (the library
call releases the GIL), against one handle alone. Prints aggregate GB/s."""
import os, sys, threading, time
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W

B, C, K = 1 << 30, 128, int(os.environ.get("K", 12))
seed = W.seed_of(2)


def lineage(sd):
    st = torch.cuda.Stream()
    bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
    with torch.cuda.stream(st):
        W.DeviceGen.initial(2, bufs[0], B, sd, st)
        for k in range(1, K):
            bufs[k].copy_(bufs[k - 1]); W.DeviceGen.mutate(2, bufs[k], B, k, C, sd, 0.01, st)
    st.synchronize()
    return bufs


L = [lineage(seed), lineage(seed + 1)]
W0 = 3


def run(nh):
    cks = [Checkpointer(C) for _ in range(nh)]
    sts = [torch.cuda.Stream() for _ in range(nh)]
    for i in range(nh):
        for k in range(W0):
            cks[i].checkpoint(L[i][k], stream=sts[i], raw=True)
    torch.cuda.synchronize()
    bar = threading.Barrier(nh + 1)

    def work(i):
        bar.wait()
        for k in range(W0, K):
            try:
                cks[i].checkpoint(L[i][k], stream=sts[i], raw=True)
            except Exception as e:
                print("handle", i, "checkpoint", k, "failed:", e, flush=True)
                raise
        sts[i].synchronize()
    th = [threading.Thread(target=work, args=(i,)) for i in range(nh)]
    for t in th: t.start()
    bar.wait()
    t0 = time.perf_counter()
    for t in th: t.join()
    dt = time.perf_counter() - t0
    n = nh * (K - W0)
    print(f"handles={nh} ckpts={n} {dt / n * 1e3:.4f} ms per checkpoint, aggregate {n * B / dt / 1e9:.0f} GB/s", flush=True)


if os.environ.get("INLINE"):
    ck = Checkpointer(C); st = torch.cuda.Stream()
    for k in range(K):
        ck.checkpoint(L[0][k], stream=st, raw=True); print("inline ok", k, flush=True)
for nh in (1, 2, 1, 2):
    run(nh)
