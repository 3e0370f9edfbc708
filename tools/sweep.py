#!/usr/bin/env python
"""Measurement sweep over BASELINE.json configs 2-5 on one B200.

    python tools/sweep.py [--only 2,3,4,5] [--out gpurun_out/sweep.json]

Per case: one handle, one device buffer mutated in place between checkpoints (the
generator runs outside the library's events), per-checkpoint device time from the
library's CUDA events at profiling level 1 (events around the whole call only, PDL kept).
Reported: checkpoint 0 separately, steady state = sum_{k>=1} B / sum_{k>=1} t_k (§8(d)),
diff ratio with and without checkpoint 0, metadata ratio, Tree-vs-List entry
compaction, and restore(last) == the last input (byte equality on the device).

  cfg2: 1 GiB GDV-like, C = 128, K = 20, p in {0.001, 0.005, 0.01, 0.05}
  cfg3: 4 GiB GDV-like, p = 0.01, K = 10, C in {32 ... 4096}
  cfg4: 1 GiB duplicate-heavy (host generator, H2D before each checkpoint), C = 128, K = 50
  cfg5: 16 GiB GDV-like on one GPU, C = 128, p = 0.01, K = 10 (bench.py --gpus N runs
        the multi-GPU weak-scaling form at 1 GiB per rank)
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

GiB = 1 << 30


def run_case(name, cfg, B, C, K, p, stream, host_gen=None, prof=1, mode=0, d2h=False, variant=None):
    import torch
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    seed = W.seed_of(cfg)
    buf = torch.empty(B, dtype=torch.uint8, device="cuda")
    ck = Checkpointer(C, mode)
    if variant is not None:
        ck.set_variant(*variant)
    ck.set_profiling(prof)
    diffs, ts, walls, phases, d2hs = [], [], [], [], []
    hbuf = torch.empty(B + 64 + 12 * ((B + C - 1) // C) + 16, dtype=torch.uint8).pin_memory() if d2h else None
    t_gen = 0.0
    for k in range(K):
        g0 = time.perf_counter()
        with torch.cuda.stream(stream):
            if host_gen is not None:
                hb = torch.from_numpy(host_gen.next()).pin_memory()
                buf.copy_(hb, non_blocking=True)
            elif k == 0:
                W.DeviceGen.initial(cfg, buf, B, seed, stream)
            else:
                W.DeviceGen.mutate(cfg, buf, B, k, C, seed, p, stream)
        stream.synchronize()
        t_gen += time.perf_counter() - g0
        w0 = time.perf_counter()
        diffs.append(ck.checkpoint(buf, stream=stream))
        walls.append(time.perf_counter() - w0)
        pt = ck.phase_times(k)
        ts.append(pt["total"])
        phases.append(pt)
        if d2h:   # the paper's throughput includes one D2H of the consolidated diff
            h0 = time.perf_counter()
            ck.diff_to_host(k, hbuf)
            d2hs.append(time.perf_counter() - h0)
    out = torch.empty_like(buf)
    r0 = time.perf_counter()
    ck.restore(K - 1, out)
    torch.cuda.synchronize()
    rs_cold = time.perf_counter() - r0
    ok = bool(torch.equal(out, buf))
    out.zero_()
    torch.cuda.synchronize()
    r0 = time.perf_counter()
    ck.restore(K - 1, out)
    torch.cuda.synchronize()
    rs = time.perf_counter() - r0
    ok = ok and bool(torch.equal(out, buf))
    del out
    ck.close()
    del buf
    torch.cuda.empty_cache()
    st = diffs[1:]
    t_st = ts[1:]
    sum_b = sum(d["bytes"] for d in diffs)
    sum_b_st = sum(d["bytes"] for d in st)
    rec = {
        "case": name, "config": cfg, "buffer_bytes": B, "chunk_bytes": C, "checkpoints": K, "update_rate": p,
        "method": ["tree", "list", "basic"][mode],
        "variant": None if variant is None else {"flags": variant[0], "switch_permille": variant[1]},
        "full_diffs": sum(1 for d in diffs if d["n_first_regions"] == 1 and d["n_shift_regions"] == 0
                          and d["data_bytes"] == B and d["meta_bytes"] == 80),
        "steady_gbs": round((K - 1) * B / (sum(t_st) / 1e3) / 1e9, 1),
        "steady_ms_median": round(statistics.median(t_st), 4),
        "steady_ms_min": round(min(t_st), 4), "steady_ms_max": round(max(t_st), 4),
        "steady_wall_gbs": round((K - 1) * B / sum(walls[1:]) / 1e9, 1),
        "ckpt0_ms": round(ts[0], 3), "ckpt0_gbs": round(B / (ts[0] / 1e3) / 1e9, 1),
        "diff_ratio_all": round(K * B / max(1, sum_b), 3),
        "diff_ratio_steady": round((K - 1) * B / max(1, sum_b_st), 2),
        "diff_bytes_ckpt0": diffs[0]["bytes"], "diff_bytes_steady_mean": int(sum_b_st / max(1, K - 1)),
        "meta_over_diff_steady": round(sum(d["meta_bytes"] for d in st) / max(1, sum_b_st), 4),
        "meta_over_input_steady": round(sum(d["meta_bytes"] for d in st) / ((K - 1) * B), 6),
        "compaction_vs_list_steady": round(sum(d["list_entries"] for d in st) /
                                           max(1, sum(d["n_first_regions"] + d["n_shift_regions"] for d in st)), 3),
        "leaves_steady_mean": {x: int(sum(d[x] for d in st) / max(1, K - 1))
                               for x in ("n_first", "n_spatial", "n_temporal", "n_fixed")},
        "regions_steady_mean": {x: int(sum(d[x] for d in st) / max(1, K - 1))
                                for x in ("n_first_regions", "n_shift_regions")},
        "record_size": diffs[-1]["record_size"],
        "restore_last_s": round(rs, 5), "restore_cold_s": round(rs_cold, 4), "restore_last_gbs": round(B / rs / 1e9, 2), "restore_ok": ok,
        "gen_s": round(t_gen, 2),
        "profiling_level": prof,
    }
    if d2h:
        # "the size of the original data divided by the time it takes to create and copy
        # the incremental checkpoint from the GPU to the host memory" (steady checkpoints)
        rec["paper_throughput_gbs"] = round((K - 1) * B / (sum(t_st) / 1e3 + sum(d2hs[1:])) / 1e9, 1)
        rec["d2h_s_steady_mean"] = round(sum(d2hs[1:]) / max(1, K - 1), 6)
    # where the host wall time of a call goes (library host timers, include/ckpt.h [6..9]) and
    # how often the record table grew (capacity changes) — the wall vs device gap
    rec["host_ms_steady_mean"] = {x: round(sum(q[x] for q in phases[1:]) / max(1, K - 1), 4)
                                  for x in ("host_pre", "host_enqueue", "host_sync_wait", "host_post",
                                            "host_table_growth", "host_arena_growth")}
    rec["host_pre_ms_max"] = round(max(q["host_pre"] for q in phases[1:]), 3) if K > 1 else None
    rec["host_table_growth_ms_max"] = round(max(q["host_table_growth"] for q in phases[1:]), 3) if K > 1 else None
    rec["host_arena_growth_ms_max"] = round(max(q["host_arena_growth"] for q in phases[1:]), 3) if K > 1 else None
    rec["wall_ms_steady_mean"] = round(1e3 * sum(walls[1:]) / max(1, K - 1), 4)
    rec["wall_ms_steady_median"] = round(1e3 * statistics.median(walls[1:]), 4)
    rec["device_ms_steady_mean"] = round(sum(t_st) / max(1, K - 1), 4)
    rec["table_growths"] = sum(1 for a, b in zip(diffs, diffs[1:]) if b["record_capacity"] != a["record_capacity"])
    if prof >= 2:   # events between every kernel (breaks PDL overlap: a breakdown, not a rate)
        rec["phase_ms_steady_mean"] = {x: round(sum(q[x] for q in phases[1:]) / max(1, K - 1), 4)
                                       for x in ("leaf_hash", "insert", "phase2", "phase3", "compact", "total")}
    return rec


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="2,3,4,5")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.json"))
    ap.add_argument("--small", action="store_true", help="quick shapes (CI / smoke of the tool)")
    ap.add_argument("--prof", type=int, default=1, help="library profiling level (2: per-phase breakdown)")
    ap.add_argument("--k", type=int, default=0, help="override the number of checkpoints")
    ap.add_argument("--methods", action="store_true",
                    help="Fig. 4 analogue: Tree / List / Basic over C = 32..512 on config 2 (1 GiB, K = 10), "
                         "with the paper's create + D2H throughput")
    ap.add_argument("--variants", action="store_true",
                    help="NEXT #4: full first checkpoint on config 2, the full-change switch on configs 2 and 4")
    a = ap.parse_args()
    import torch
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream()
    only = {int(x) for x in a.only.split(",")}
    s = 64 if a.small else 1
    cases = []
    if 2 in only:
        for p in (0.001, 0.005, 0.01, 0.05):
            cases.append((f"cfg2_p{p}", 2, GiB // s, 128, 20, p, None))
    if 3 in only:
        for C in (32, 64, 128, 256, 512, 1024, 2048, 4096):
            cases.append((f"cfg3_C{C}", 3, 4 * GiB // s, C, 10, 0.01, None))
    if 4 in only:
        cases.append(("cfg4_dup_heavy", 4, GiB // s, 128, 50, 0.0, "dup"))
    if 5 in only:
        cases.append(("cfg5_16GiB_1gpu", 5, 16 * GiB // s, 128, 10, 0.01, None))
    cases = [c + (0, False, None) for c in cases]
    if a.methods:
        cases = []
        for C in (32, 64, 128, 256, 512):
            for m, nm in ((0, "tree"), (1, "list"), (2, "basic")):
                cases.append((f"methods_{nm}_C{C}", 2, GiB // s, C, 10, 0.01, None, m, True, None))
    if a.variants:
        cases = [
            ("var_full_first_cfg2_p0.01", 2, GiB // s, 128, 20, 0.01, None, 0, False, (1, 1000)),
            ("var_switch30_cfg2_p0.05", 2, GiB // s, 128, 20, 0.05, None, 0, False, (2, 30)),
            ("var_none_cfg4_dup_heavy", 4, GiB // s, 128, 20, 0.0, "dup", 0, False, None),
            ("var_switch850_cfg4_dup_heavy", 4, GiB // s, 128, 20, 0.0, "dup", 0, False, (2, 850)),
            ("var_shift_insert_cfg2_p0.01", 2, GiB // s, 128, 20, 0.01, None, 0, False, (4, 1000)),
            ("var_shift_insert_cfg4_dup_heavy", 4, GiB // s, 128, 20, 0.0, "dup", 0, False, (4, 1000)),
        ]
    recs = []
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    for name, cfg, B, C, K, p, hg, mode, d2h, var in cases:
        gen = W.DupHeavy(B, C, W.seed_of(cfg)) if hg == "dup" else None
        r = run_case(name, cfg, B, C, a.k or K, p, stream, gen, a.prof, mode, d2h, var)
        r["device"] = torch.cuda.get_device_name(0)
        print(json.dumps(r), flush=True)
        recs.append(r)
        with open(a.out, "w") as f:
            json.dump(recs, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
