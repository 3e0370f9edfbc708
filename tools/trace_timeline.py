import numpy as np, sys, glob
f = sorted(glob.glob(sys.argv[1] + ".*.bin"))[-1]
a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
t0 = None
rows = []
for ph in (2, 3):
    b = a[a[:, 3] == ph]
    st = b[:, 2] >> 32
    for sg in sorted(set(st.tolist())):
        m = b[st == sg]
        rows.append((f"phase{ph} stage{sg}", m[:, 0].min(), m[:, 1].max(), len(m)))
g = a[a[:, 3] == 77]
if len(g): rows.append(("gather", g[:, 0].min(), g[:, 2].max(), len(g)))
t0 = min(r[1] for r in rows)
for name, s, e, n in rows:
    print(f"{name:16s} n={n:5d}  start {(s - t0)/1e3:7.1f}  end {(e - t0)/1e3:7.1f} us")
for ph in (2, 3):
    idx = np.nonzero(a[:, 3] == 40 + ph)[0]
    for i in idx[:3]:
        g = a[i - 1]; q1 = a[i]; q2 = a[i + 1]
        print(f"phase{ph} upper group stage{g[2]>>32}: input {(q1[0]-g[0])/1e3:.2f} pass1 {(q1[1]-q1[0])/1e3:.2f} pass2 {(q1[2]-q1[1])/1e3:.2f} "
              f"labels/pass3 {(q2[0]-q1[2])/1e3:.2f} root {(q2[1]-q2[0])/1e3:.2f} rest {(g[1]-q2[1])/1e3:.2f} us")
