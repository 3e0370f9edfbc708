"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list (median per kernel)."""
import csv, sys
from collections import defaultdict
rows = list(csv.reader(open(sys.argv[1])))
hdr = None
agg = defaultdict(list)
for r in rows:
    if 'Kernel Name' in r:
        hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        try:
            agg[d['Kernel Name'][:70]].append(float(d['Metric Value'].replace(',', '')))
        except ValueError:
            pass
for n, v in agg.items():
    v = sorted(v)
    print(f"{n:72s} n={len(v):4d} med={v[len(v)//2]/1e3:9.1f} us  min={v[0]/1e3:9.1f}")
