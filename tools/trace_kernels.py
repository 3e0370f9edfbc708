"""Kernel-level timeline of one traced checkpoint (CKPT_TRACE=<prefix>): per kernel, the
first block entry, the first/last return from griddepcontrol.wait and the last block exit,
in us from K1's first block entry. Usage: python tools/trace_kernels.py <prefix> [k]"""
import glob
import sys

import numpy as np

NAMES = {100: "K1 leaf", 101: "K1b insert", 111: "K1b worklist", 102: "tree phase 2", 103: "tree phase 3",
         104: "offsets", 105: "gather", 106: "data"}


def main():
    files = sorted(glob.glob(sys.argv[1] + ".*.bin"), key=lambda f: int(f.split(".")[-2]))
    f = files[int(sys.argv[2])] if len(sys.argv) > 2 else files[-1]
    a = np.fromfile(f, dtype=np.uint64).reshape(-1, 4).astype(np.int64)
    b = a[(a[:, 3] >= 100) & (a[:, 3] < 200)]
    t0 = b[b[:, 3] == 100][:, 0].min() if (b[:, 3] == 100).any() else b[:, 0].min()
    print(f)
    print(f"{'kernel':14s} {'blocks':>6s} {'entry':>8s} {'wait>=':>8s} {'wait<=':>8s} {'exit<=':>8s}  (us)")
    for code in sorted(set(b[:, 3].tolist()), key=lambda c: b[b[:, 3] == c][:, 0].min()):
        m = b[b[:, 3] == code]
        print(f"{NAMES.get(int(code), str(code)):14s} {len(m):6d} {(m[:, 0].min() - t0) / 1e3:8.2f} "
              f"{(m[:, 1].min() - t0) / 1e3:8.2f} {(m[:, 1].max() - t0) / 1e3:8.2f} {(m[:, 2].max() - t0) / 1e3:8.2f}")


if __name__ == "__main__":
    main()
