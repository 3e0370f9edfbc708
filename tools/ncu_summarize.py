"""Summarise an `ncu --set full` report into profiles/ncu_summary.json (+ a text table).

Usage: python tools/ncu_summarize.py gpurun_out/prof.ncu-rep profiles/ncu_summary.json
"""
import csv
import io
import json
import subprocess
import sys

METRICS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "smsp__inst_executed.sum",
]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
              "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}


def main(rep, out_json):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(METRICS)],
                                  text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    summary = {}
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        name = d["Kernel Name"].split("(")[0].replace("void ", "").replace("ckpt::", "")
        base = name.split("<")[0]
        rec = {}
        for m in METRICS:
            v = d.get(m, "")
            try:
                x = float(v.replace(",", ""))
            except ValueError:
                continue
            scale = UNIT_SCALE.get(u.get(m, ""), 1.0)
            if m.startswith("dram__bytes"):
                rec[m] = x * scale
            elif m == "gpu__time_duration.sum":
                rec["duration_s"] = x * scale
            else:
                rec[m] = x
        if "dram__bytes_read.sum" in rec:
            rec["dram_bytes_per_launch"] = rec["dram__bytes_read.sum"] + rec.get("dram__bytes_write.sum", 0.0)
            if rec.get("duration_s"):
                rec["dram_gbs"] = rec["dram_bytes_per_launch"] / rec["duration_s"] / 1e9
        summary.setdefault(base, rec)   # first captured launch of each kernel
        summary[name] = rec
    with open(out_json, "w") as f:
        json.dump(summary, f, indent=1, sort_keys=True)
    for k, v in summary.items():
        print(f"{k:40s} {v.get('duration_s', 0)*1e6:9.1f} us  dram {v.get('dram_bytes_per_launch', 0)/1e6:10.2f} MB"
              f"  {v.get('dram_gbs', 0):8.1f} GB/s  sm {v.get('sm__throughput.avg.pct_of_peak_sustained_elapsed', 0):5.1f}%"
              f"  issue {v.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):5.1f}%")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
