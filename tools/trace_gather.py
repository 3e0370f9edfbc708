import numpy as np, sys, glob
for f in sorted(glob.glob(sys.argv[1] + ".*.bin"))[-1:]:
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
    g = a[a[:, 3] == 77]
    t0 = g[:, 0].min()
    print(f, "tiles", len(g), "start spread", (g[:, 0].max() - t0) / 1e3, "head med", np.median(g[:, 1] - g[:, 0]) / 1e3,
          "body med", np.median(g[:, 2] - g[:, 1]) / 1e3, "p90", np.percentile(g[:, 2] - g[:, 1], 90) / 1e3,
          "end max", (g[:, 2].max() - t0) / 1e3)
