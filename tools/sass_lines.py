"""Aggregate an ncu source page (SASS view) by CUDA source line.

    python tools/sass_lines.py REPORT.ncu-rep KERNEL_REGEX MANGLED_NAME CUBIN [--skip N] [--top 30]

ncu's SASS rows carry absolute addresses; nvdisasm -g of the same cubin carries function
offsets with `//## File "...", line N` comments. Offsets = address - first address of the
kernel, so both views line up when the cubin is the one that was profiled (-lineinfo build).
"""
import argparse
import collections
import csv
import io
import re
import subprocess


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("kernel")
    ap.add_argument("mangled")
    ap.add_argument("cubin")
    ap.add_argument("--skip", type=int, default=0)
    ap.add_argument("--top", type=int, default=30)
    a = ap.parse_args()
    txt = subprocess.check_output(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass",
                                   "--kernel-name", f"regex:{a.kernel}", "--launch-skip", str(a.skip),
                                   "--launch-count", "1"], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[1]
    data = rows[2:]
    i_s = hdr.index("Warp Stall Sampling (All Samples)")
    i_ex = hdr.index("Instructions Executed")
    base = int(data[0][0], 16)
    dis = subprocess.check_output(["nvdisasm", "-g", "-c", a.cubin], text=True, stderr=subprocess.DEVNULL)
    line_of = {}
    cur = None
    inside = False
    for ln in dis.splitlines():
        if ".section" in ln and ".text." in ln:
            inside = (".text." + a.mangled + ",") in ln
            cur = None
            continue
        if not inside:
            continue
        m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
        if m:
            cur = f"{m.group(1).split('/')[-1]}:{m.group(2)}"
            continue
        m = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
        if m and cur:
            line_of[int(m.group(1), 16)] = cur
    agg_s = collections.Counter()
    agg_i = collections.Counter()
    miss = 0
    for r in data:
        off = int(r[0], 16) - base
        key = line_of.get(off)
        if key is None:
            miss += 1
            key = "?"
        agg_s[key] += int(r[i_s]) if r[i_s].isdigit() else 0
        agg_i[key] += int(r[i_ex]) if r[i_ex].isdigit() else 0
    ts, ti = sum(agg_s.values()), sum(agg_i.values())
    print(f"samples {ts}  warp-instructions {ti}  unmapped rows {miss}/{len(data)}")
    print("by instructions:")
    for k, v in agg_i.most_common(a.top):
        print(f"  {k:24s} instr {v:>11d} ({100 * v / max(1, ti):5.1f}%)  samples {agg_s[k]:>6d} ({100 * agg_s[k] / max(1, ts):5.1f}%)")
    print("by stall samples:")
    for k, v in agg_s.most_common(a.top):
        print(f"  {k:24s} samples {v:>6d} ({100 * v / max(1, ts):5.1f}%)  instr {agg_i[k]:>11d}")


if __name__ == "__main__":
    main()
