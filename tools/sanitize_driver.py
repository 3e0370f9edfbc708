#!/usr/bin/env python
"""Small lineages through every path of libckpt.so, for compute-sanitizer:

    compute-sanitizer --tool {memcheck,racecheck,synccheck} python tools/sanitize_driver.py

config 1 (1 MiB, 10 checkpoints), duplicate-heavy lineages in the Tree / List / Basic
methods (C = 64, ragged n), the variants (full first checkpoint, full-change switch, SHIFT-SHIFT insertion),
a multi-stage tree (n > 2^20 at C = 32), every restore, and a lineage import. Each diff
is compared with the CPU oracle so a sanitizer run is also a parity run.
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (test infrastructure: the checker)
from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer  # noqa: E402
from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W  # noqa: E402
from tests._lineages import dup_lineage  # noqa: E402


def run(name, bufs, C, mode=0, variant=None, check_import=False, pipe=False):
    B = bufs[0].size
    o = oracle.Oracle(C, mode=mode)
    ck = Checkpointer(C, mode)
    if variant:
        o.set_variant(*variant)
        ck.set_variant(*variant)
    devs = []
    pend = None
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        t = torch.from_numpy(np.ascontiguousarray(b)).cuda()
        devs.append(t)
        if pipe:   # ckpt_checkpoint_submit / _wait, two calls in flight
            cid = ck.submit(t, nbytes=B)
            if pend is not None:
                ck.wait(pend)
            pend = cid
        else:
            ck.checkpoint(t, nbytes=B)
    if pend is not None:
        ck.wait(pend)
    for k in range(len(bufs)):
        assert ck.diff_to_host(k) == o.diff(k), (name, k)
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(len(bufs)):
        ck.restore(k, out)
        assert torch.equal(out, devs[k]), (name, "restore", k)
    if check_import:
        b2 = Checkpointer(C, mode)
        if variant:
            b2.set_variant(*variant)
        for k in range(len(bufs)):
            b2.import_diff(ck.diff_to_host(k))
        b2.close()
    ck.close()
    print("ok", name, flush=True)


def main():
    oracle.build()
    torch.cuda.set_device(0)
    run("config1", list(W.lineage(1, 1 << 20, 128, 10)), 128, check_import=True)
    for mode in (0, 1, 2):
        run(f"dup_mode{mode}", dup_lineage(11, 3000 * 64 - 5, 64, K=6), 64, mode=mode, check_import=True)
    run("full_first", dup_lineage(12, 2000 * 64, 64, K=4), 64, variant=(1, 1000))
    run("switch", dup_lineage(13, 2000 * 64, 64, K=4, p_change=0.9), 64, variant=(2, 300), check_import=True)
    run("shift_insert", dup_lineage(14, 2000 * 64 - 3, 64, K=4, alphabet=2), 64, variant=(4, 1000), check_import=True)
    run("shift_insert_zero", [np.zeros(4096 * 32, dtype=np.uint8), np.full(4096 * 32, 3, dtype=np.uint8)], 32,
        variant=(4, 1000))
    run("config2_small", list(W.lineage(2, (1 << 22) + 100, 128, 4, p=0.05)), 128)
    run("pipelined_config2", list(W.lineage(2, (1 << 22) + 100, 128, 5, p=0.05)), 128, pipe=True)
    run("pipelined_dup", dup_lineage(15, 3000 * 64 - 5, 64, K=6, p_change=0.8), 64, pipe=True, check_import=True)
    if os.environ.get("SAN_BIG", "1") == "1":
        run("multistage_C32", list(W.lineage(1, (1 << 25) + 100, 32, 3, p=0.01)), 32)
    print("sanitize driver done", flush=True)


if __name__ == "__main__":
    main()
