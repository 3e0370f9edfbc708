import numpy as np, sys, glob
for f in sorted(glob.glob(sys.argv[1] + ".*.bin"))[-1:]:
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
    a = a[a[:, 3] > a[:, 0]]
    a = a[(a[:, 1] >= a[:, 0]) & (a[:, 3] - a[:, 0] < 10**6)]
    t0 = a[:, 0].min()
    print(f, "n", len(a), "kernel-start spread", (a[:, 0].max() - t0) / 1e3,
          "loads med", np.median(a[:, 2] - a[:, 1]) / 1e3, "insert med", np.median(a[:, 3] - a[:, 2]) / 1e3,
          "p90", np.percentile(a[:, 3] - a[:, 2], 90) / 1e3, "end max", (a[:, 3].max() - t0) / 1e3)
