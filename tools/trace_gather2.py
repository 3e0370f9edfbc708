"""Per-tile gather timings from a CKPT_TRACE capture: python tools/trace_gather2.py <prefix>"""
import glob, sys
import numpy as np
f = sorted(glob.glob(sys.argv[1] + ".*.bin"), key=lambda x: int(x.split(".")[-2]))[-1]
a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
i77 = np.nonzero(a[:, 3] == 77)[0]
r0, r1 = a[i77], a[i77 + 1]
t0 = r0[:, 0].min()
dur = (r0[:, 2] - r0[:, 0]) / 1e3
pre = (r0[:, 1] - r0[:, 0]) / 1e3
print(f, "tiles", len(r0), "span us", (r0[:, 2].max() - t0) / 1e3)
print("per-tile dur med/p90/max", np.median(dur), np.percentile(dur, 90), dur.max(), "prefix part med", np.median(pre))
print("bytes per tile med/max", np.median(r1[:, 2]), r1[:, 2].max(), "total MB", r1[:, 2].sum() / 1e6)
blk = a[a[:, 3] == 105]
if len(blk):
    print("gather blocks", len(blk), "entry->wait med", np.median((blk[:, 1] - blk[:, 0]) / 1e3), "exit max", (blk[:, 2].max() - t0) / 1e3)
