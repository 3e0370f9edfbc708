"""Small seeded lineages for CPU/GPU parity tests (harness only; no method arithmetic)."""
import numpy as np


def dup_lineage(seed, nbytes, C, K, alphabet=6, p_change=0.3, block_copy=True):
    """Tiny lineages full of spatial/temporal duplicates: each chunk is drawn from a
    small alphabet of contents, later checkpoints change some chunks, copy aligned
    blocks from older checkpoints, and sometimes keep chunks fixed."""
    rng = np.random.default_rng(seed)
    n = (nbytes + C - 1) // C
    alpha = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(alphabet)]
    bufs = []
    cur = np.zeros(n * C, dtype=np.uint8)
    for i in range(n):
        cur[i * C:(i + 1) * C] = alpha[rng.integers(alphabet)]
    bufs.append(cur[:nbytes].copy())
    for k in range(1, K):
        cur = cur.copy()
        for i in range(n):
            r = rng.random()
            if r < p_change / 2:
                cur[i * C:(i + 1) * C] = alpha[rng.integers(alphabet)]
            elif r < p_change:
                cur[i * C:(i + 1) * C] = rng.integers(0, 256, C, dtype=np.uint8)
        if block_copy and n >= 4:
            j = int(rng.integers(1, max(2, int(np.log2(n)))))
            blk = 1 << j
            if blk <= n:
                src_k = int(rng.integers(0, len(bufs)))
                a = int(rng.integers(0, n // blk)) * blk
                b = int(rng.integers(0, n // blk)) * blk
                old = np.zeros(n * C, dtype=np.uint8)
                old[:nbytes] = bufs[src_k]
                cur[b * C:(b + blk) * C] = old[a * C:(a + blk) * C]
        bufs.append(cur[:nbytes].copy())
    return bufs
