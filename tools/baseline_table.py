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
            rows.append(f"| {name} | 1 | 128 | **{f(v)}** (sweep, device time per call); **{f(b)}** (`bench.py`, host "
                        f"sync and call gap included) | {pct(v)} (bench: {pct(b)}) | {f(b)} {tail} "
                        f"{o2['steady_s_mean']:.2f} s (ckpt 0: {o2['ckpt0_s']:.2f} s) |")
        else:
            rows.append(f"| {name} | 1 | 128 | {f(v)} | {pct(v)} | {f(v)} {tail} — |")
    for C in (32, 64, 128, 256, 512, 1024, 2048, 4096):
        r = sw[f"cfg3_C{C}"]
        v = r["steady_gbs"]
        rows.append(f"| {'3 (4 GiB, p = 1 %)' if C == 32 else '3'} | 1 | {C} | {f(v)} | {pct(v)} | {f(v)} | "
                    f"{f(r['ckpt0_gbs'])} | {r['diff_ratio_all']:.1f} / {r['diff_ratio_steady']:.1f} | "
                    f"{r['meta_over_diff_steady']:.3f} | {r['compaction_vs_list_steady']:.2f} | n/a |")
    r = sw["cfg4_dup_heavy"]
    v = r["steady_gbs"]
    rows.append(f"| 4 (duplicate-heavy, 1 GiB, 50 checkpoints) | 1 | 128 | {f(v)} | {pct(v)} | {f(v)} | "
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
    b = s.index("\nNotes on the table:")
    s = s[:a] + "\n".join(rows) + "\n" + s[b:]
    open(path, "w").write(s)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
