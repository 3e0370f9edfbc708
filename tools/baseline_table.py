#!/usr/bin/env python
"""Regenerates BASELINE.md §3's results rows from profiles/ (sweep_rN.json, bench_rN.json,
bench_cfg1_rN.json, oracle_time_rN.json of the latest round that has each file) and
MEASURED_PEAKS.json:
    python tools/baseline_table.py            # rewrites the table rows in place"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = lambda *a: os.path.join(ROOT, *a)


def latest(stem):
    for r in (3, 2, 1):
        f = P("profiles", f"{stem}_r{r}.json")
        if os.path.exists(f):
            return f
    raise FileNotFoundError(stem)


def latest_txt(stem):
    for r in (3, 2, 1):
        f = P("profiles", f"{stem}_r{r}.txt")
        if os.path.exists(f):
            return f
    raise FileNotFoundError(stem)


def main():
    sw = {r["case"]: r for r in json.load(open(latest("sweep")))}
    bench = json.loads(open(latest("bench")).read())
    c1 = json.loads(open(latest("bench_cfg1")).read())
    ot = {c["case"]: c for c in json.load(open(latest("oracle_time")))["cases"]}
    try:
        meas = json.load(open(P("MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        meas = 6551.7
    spec = 8000.0
    pct = lambda v: f"{100 * v / spec:.0f} % / {100 * v / meas:.0f} %"
    f = lambda x: f"{x:,.0f}".replace(",", " ")
    o1, o2, o4 = ot["cfg1_1MiB"], ot["cfg2_1GiB_p0.01"], ot["cfg4_64MiB"]
    # pipelined lineages (tools/pipe_probe.py lines "cfgX C=.. p=..: sync .. ms (.. GB/s)  pipelined .. ms (.. GB/s)")
    pipe = {}
    try:
        import re
        for ln in open(latest_txt("pipeline")):
            m = re.match(r"cfg(\d) C=(\d+) p=([0-9.]+): sync [0-9.]+ ms \((\d+) GB/s\)\s+pipelined [0-9.]+ ms \((\d+) GB/s\)", ln)
            if m:
                pipe[(int(m[1]), int(m[2]), float(m[3]))] = (int(m[4]), int(m[5]))
    except FileNotFoundError:
        pass
    pv = lambda cfg, C, p: (f" (pipelined: {f(pipe[(cfg, C, p)][1])})" if (cfg, C, p) in pipe else "")
    rows = [f"| 1 (1 MiB, 1 %) | 1 | 128 | {c1['value']:.1f} ({c1['ms_per_step'] * 1000:.0f} µs per checkpoint: five "
            f"launches, latency-bound, a parity config) | — | {c1['value']:.1f} | {c1['checkpoint0']['gbs']} (untimed first "
            f"touch) | {c1['diff_ratio']} steady | {c1['meta_over_diff']} | {c1['compaction_vs_list']} | "
            f"{o1['steady_s_mean']:.4f} s (ckpt 0: {o1['ckpt0_s']:.4f} s) |"]
    for p, name in ((0.001, "2 (1 GiB GDV-like, p = 0.1 %)"), (0.005, "2 (p = 0.5 %)"), (0.01, "**2 (p = 1 %, headline)**"),
                    (0.05, "2 (p = 5 %)")):
        r = sw[f"cfg2_p{p}"]
        v = r["steady_gbs"]
        tail = (f"| {f(r['ckpt0_gbs'])} | {r['diff_ratio_all']:.1f} / {r['diff_ratio_steady']:.0f} | "
                f"{r['meta_over_diff_steady']:.3f} | {r['compaction_vs_list_steady']:.2f} |")
        if p == 0.01:
            b = bench["value"]
            sb = (bench.get("sync") or {}).get("value")
            sync_txt = f"; {f(sb)} one call at a time (`bench.py` `sync`)" if sb else ""
            rows.append(f"| {name} | 1 | 128 | **{f(b)}** (`bench.py`, pipelined calls){sync_txt}; {f(v)} (sweep, "
                        f"device time per synchronous call) | {pct(b)} (sweep: {pct(v)}) | {f(b)} {tail} "
                        f"{o2['steady_s_mean']:.2f} s (ckpt 0: {o2['ckpt0_s']:.2f} s) |")
        else:
            rows.append(f"| {name} | 1 | 128 | {f(v)}{pv(2, 128, p)} | {pct(v)} | {f(v)} {tail} — |")
    for C in (32, 64, 128, 256, 512, 1024, 2048, 4096):
        r = sw[f"cfg3_C{C}"]
        v = r["steady_gbs"]
        rows.append(f"| {'3 (4 GiB, p = 1 %)' if C == 32 else '3'} | 1 | {C} | {f(v)}{pv(3, C, 0.01)} | {pct(v)} | {f(v)} | "
                    f"{f(r['ckpt0_gbs'])} | {r['diff_ratio_all']:.1f} / {r['diff_ratio_steady']:.1f} | "
                    f"{r['meta_over_diff_steady']:.3f} | {r['compaction_vs_list_steady']:.2f} | n/a |")
    r = sw["cfg4_dup_heavy"]
    v = r["steady_gbs"]
    rows.append(f"| 4 (duplicate-heavy, 1 GiB, 50 checkpoints) | 1 | 128 | {f(v)}{pv(4, 128, 0.01)} | {pct(v)} | {f(v)} | "
                f"{f(r['ckpt0_gbs'])} | {r['diff_ratio_all']:.1f} / {r['diff_ratio_steady']:.1f} | "
                f"{r['meta_over_diff_steady']:.3f} | {r['compaction_vs_list_steady']:.2f} | "
                f"{o4['steady_s_mean']:.3f} s at 64 MiB (ckpt 0: {o4['ckpt0_s']:.3f} s) |")
    r = sw["cfg5_16GiB_1gpu"]
    v = r["steady_gbs"]
    rows.append(f"| 5 (16 GiB, p = 1 %) | 1 | 128 | {f(v)} | {pct(v)} | {f(v)} | {f(r['ckpt0_gbs'])} | "
                f"{r['diff_ratio_all']:.1f} / {r['diff_ratio_steady']:.0f} | {r['meta_over_diff_steady']:.3f} | "
                f"{r['compaction_vs_list_steady']:.2f} | n/a |")
    rows.append("| 5 (weak scaling) | 2/4/8 | 128 | not measurable here: every `gpurun` call and the round-end driver get "
                "one B200; `bench.py --gpus N` runs it (independent ranks, NCCL all-gather of the 32-B size records "
                "outside the timed region) | — | — | — | — | — | — | n/a |")
    path = P("BASELINE.md")
    s = open(path).read()
    a = s.index("| 1 (1 MiB, 1 %) | 1 | 128 |")
    b = s.index("\nNotes on the table")
    s = s[:a] + "\n".join(rows) + "\n" + s[b:]
    open(path, "w").write(s)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
