import numpy as np, sys, glob
for f in sorted(glob.glob(sys.argv[1] + ".*.bin")):
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4)
    if len(a) == 0: continue
    t0 = a[:, 0].min()
    for ph in (2, 3):
        b = a[a[:, 3] == ph]
        if len(b) == 0: continue
        st = b[:, 2] >> 32
        d = (b[:, 1] - b[:, 0]) / 1e3
        s = (b[:, 0] - t0) / 1e3; e = (b[:, 1] - t0) / 1e3
        print(f"{f} phase{ph}: groups={len(b)} stage0 dur med={np.median(d[st==0]):.1f} p90={np.percentile(d[st==0],90):.1f} max={d[st==0].max():.1f} us; "
              f"start span {s[st==0].min():.1f}-{s[st==0].max():.1f}; end max {e[st==0].max():.1f}")
        for sg in sorted(set(st.tolist()) - {0}):
            m = st == sg
            print(f"    stage{sg}: n={m.sum()} dur={d[m].round(1).tolist()[:4]} start={s[m].round(1).tolist()[:4]} end={e[m].round(1).tolist()[:4]}")
# intra-group breakdown: records 10+phase = {after input, after pass 1, after pass 2}
for f in sorted(glob.glob(sys.argv[1] + ".*.bin"))[-1:]:
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4)
    for ph in (2, 3):
        idx = np.nonzero(a[:, 3] == 10 + ph)[0]
        if len(idx) == 0: continue
        g = a[idx - 1].astype(np.int64); q = a[idx].astype(np.int64)
        print(f"phase{ph} per-tile median us: input {np.median(q[:,0]-g[:,0])/1e3:.2f}  pass1 {np.median(q[:,1]-q[:,0])/1e3:.2f}  "
              f"pass2 {np.median(q[:,2]-q[:,1])/1e3:.2f}  pass3+root+compaction {np.median(g[:,1]-q[:,2])/1e3:.2f}")

for f in sorted(glob.glob(sys.argv[1] + ".*.bin"))[-1:]:
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
    for ph in (2, 3):
        idx = np.nonzero(a[:, 3] == 20 + ph)[0]
        if len(idx) == 0: continue
        g = a[idx - 2]; q1 = a[idx - 1]; q2 = a[idx]
        print(f"phase{ph} tail split median us: pass3/labels {np.median(q2[:,0]-q1[:,2])/1e3:.2f} root {np.median(q2[:,1]-q2[:,0])/1e3:.2f} compaction {np.median(g[:,1]-q2[:,1])/1e3:.2f}")
