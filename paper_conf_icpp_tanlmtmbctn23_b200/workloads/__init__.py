"""Seeded synthetic checkpoint workloads (harness code — none of the method's arithmetic).

These generators serve BOTH the CUDA path and the CPU oracle; they are the only code
the two sides share (DESIGN.md §6 states the recipes and why they mirror the paper's
GDV workloads). Every random draw is the counter-based hash

    splitmix64(z) = mix(z), H(s, i) = splitmix64(s + (i+1)·0x9E3779B97F4A7C15)  (mod 2^64)
    H(s, a, b, ...) = H(H(s, a), b, ...)

so the host (numpy, this module) and the device (``gen.cu`` → ``libckptgen.so``)
produce identical bytes independently; ``tests/test_gpu_api.py::test_device_generators_match_host`` checks that.

Configs (BASELINE.json ``configs``):
  1  sparse random: B=1 MiB, C=128, K=10, 1 % Bernoulli chunk updates
  2  GDV-like: 1 GiB, rows of 73 u32 orbit counts (292 B), clustered row-run updates
  3  chunk sweep of config 2 (4 GiB, C=32..4096)
  4  duplicate-heavy: Zipf placements of a 512-block dictionary, shifted/temporal dups
  5  weak scaling: config 2 at 16 GiB per rank, seed + rank
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)
BASE_SEED = 20230807

ROW_ORBITS = 73                      # reading R18: 73 orbit counts per vertex (Table 1 sizes)
ROW_BYTES = 4 * ROW_ORBITS           # 292 B per GDV row
# 24 frequently-formed orbits (~10 of 30 graphlets form frequently); fixed list
FREQ_ORBITS = np.array([0, 1, 2, 3, 4, 5, 6, 7, 9, 10, 11, 12, 13, 15, 16, 17,
                        18, 19, 20, 21, 22, 23, 24, 25], dtype=np.int64)
ZERO_BLOCK_ROWS = 64                 # unprocessed-vertex blocks at checkpoint 0 (Gorder locality)
RUN_ROWS = 16                        # rows per update run at checkpoint k >= 1
N_PROTO = 256                        # prototype rows ("repeated substructures")


def seed_of(cfg: int, rank: int = 0) -> int:
    return BASE_SEED + cfg + rank


def threshold(p: float) -> int:
    """Integer threshold floor(p·2^64): a draw u is 'hit' iff u < threshold(p)."""
    return min(int(p * 2.0 ** 64), 2 ** 64 - 1)


def splitmix64(z):
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * M1
        z = z ^ (z >> np.uint64(27))
        z = z * M2
        z = z ^ (z >> np.uint64(31))
    return z


def H(s, *idx):
    """Counter-based hash H(s, a, b, ...) (module docstring)."""
    h = np.asarray(s, dtype=np.uint64)
    with np.errstate(over="ignore"):
        for a in idx:
            a = np.asarray(a, dtype=np.uint64)
            h = splitmix64(h + (a + np.uint64(1)) * GOLDEN)
    return h


def geo(x):
    """Geometric count with mean 3: number of leading non-zero 2-bit digits of x (0..32)."""
    x = np.asarray(x, dtype=np.uint64)
    alive = np.ones(x.shape, dtype=bool)
    cnt = np.zeros(x.shape, dtype=np.uint32)
    for j in range(32):
        d = (x >> np.uint64(62 - 2 * j)) & np.uint64(3)
        alive &= d != 0
        cnt += alive.astype(np.uint32)
    return cnt


# ------------------------------------------------------------------ config 1
def cfg1_initial(nbytes: int, seed: int) -> np.ndarray:
    """Checkpoint 0: u64 word w = H(seed, w), little-endian, truncated to nbytes."""
    nw = (nbytes + 7) // 8
    w = H(seed, np.arange(nw, dtype=np.uint64))
    return w.astype("<u8").view(np.uint8)[:nbytes].copy()


def cfg1_mutate(buf: np.ndarray, k: int, chunk_bytes: int, seed: int, p: float = 0.01) -> np.ndarray:
    """Checkpoint k >= 1, in place: chunk i updated iff H(seed,k,i) < p·2^64; the
    first u64 of an updated chunk is XORed with H(seed,k,i)|1 (a guaranteed change)."""
    nbytes = buf.size
    n = (nbytes + chunk_bytes - 1) // chunk_bytes
    u = H(H(seed, k), np.arange(n, dtype=np.uint64))
    hit = np.nonzero(u < np.uint64(threshold(p)))[0]
    for i in hit:
        x = int(u[i]) | 1
        off = int(i) * chunk_bytes
        for b in range(8):
            if off + b < nbytes and b < chunk_bytes:
                buf[off + b] ^= (x >> (8 * b)) & 0xFF
    return buf


# ------------------------------------------------------------------ config 2
def cfg2_rows(nbytes: int) -> int:
    return nbytes // ROW_BYTES


def cfg2_initial(nbytes: int, seed: int) -> np.ndarray:
    """GDV-like checkpoint 0: 64-row blocks all-zero with prob 1/2;
    otherwise a row copies one of 256 prototypes with prob 0.3, else draws its own
    geometric(mean 3) count for each of the 24 frequent orbits."""
    R = cfg2_rows(nbytes)
    counts = np.zeros((R, ROW_ORBITS), dtype=np.uint32)
    if R:
        r = np.arange(R, dtype=np.uint64)
        live = H(seed, 0, r // np.uint64(ZERO_BLOCK_ROWS)) >= np.uint64(1 << 63)
        proto = H(seed, 1, r) < np.uint64(threshold(0.3))
        P = H(seed, 2, r) % np.uint64(N_PROTO)
        q = np.arange(len(FREQ_ORBITS), dtype=np.uint64)
        proto_tab = geo(H(seed, 3, np.arange(N_PROTO, dtype=np.uint64)[:, None], q[None, :]))
        own = geo(H(seed, 4, r[:, None], q[None, :]))
        vals = np.where(proto[:, None], proto_tab[P.astype(np.int64)], own)
        vals = np.where(live[:, None], vals, 0).astype(np.uint32)
        counts[:, FREQ_ORBITS] = vals
    return _cfg2_bytes(counts, nbytes)


def _cfg2_bytes(counts: np.ndarray, nbytes: int) -> np.ndarray:
    out = np.zeros(nbytes, dtype=np.uint8)
    raw = counts.astype("<u4").view(np.uint8).reshape(-1)
    out[: raw.size] = raw
    return out


def cfg2_mutate(buf: np.ndarray, k: int, seed: int, p: float) -> np.ndarray:
    """Checkpoint k >= 1, in place: each run of 16 rows is updated with prob p; in an
    updated run each frequent-orbit count grows by 1 + (v & 3) with prob 1/4 (v = H(seed,6,k,r,q))."""
    R = cfg2_rows(buf.size)
    if R == 0:
        return buf
    counts = buf[: R * ROW_BYTES].view("<u4").reshape(R, ROW_ORBITS)
    nruns = (R + RUN_ROWS - 1) // RUN_ROWS
    runs = np.nonzero(H(seed, 5, k, np.arange(nruns, dtype=np.uint64)) < np.uint64(threshold(p)))[0]
    if runs.size == 0:
        return buf
    rows = (runs[:, None] * RUN_ROWS + np.arange(RUN_ROWS)[None, :]).reshape(-1)
    rows = rows[rows < R]
    q = np.arange(len(FREQ_ORBITS), dtype=np.uint64)
    v = H(seed, 6, k, rows.astype(np.uint64)[:, None], q[None, :])
    inc = np.where(v < np.uint64(1 << 62), (v & np.uint64(3)) + np.uint64(1), np.uint64(0)).astype(np.uint32)
    sub = counts[rows][:, FREQ_ORBITS] + inc
    blk = counts[rows]
    blk[:, FREQ_ORBITS] = sub
    counts[rows] = blk
    return buf


# ------------------------------------------------------------------ config 4
class DupHeavy:
    """Duplicate-heavy lineage (config 4), host-side (parity sizes 2^20 / 2^26; 1 GiB for tools/sweep.py).

    A dictionary of 512 blocks: 75 % have length C·2^j (j in 0..8), 25 % length
    C·m + r (unaligned). The buffer is a sequence of Zipf(1.1) placements; half of the
    power-of-two placements are first aligned to their own length (these subtree-aligned
    repeats collapse into one SHIFT region). Checkpoint k >= 1 swaps 2 % of adjacent
    placement pairs (shifted duplicates), replaces 1 % by a block used elsewhere
    (temporal duplicates) and re-randomises 0.2 % (first occurrences); the layout is then
    rebuilt, so content also moves."""

    NBLK = 512

    def __init__(self, nbytes: int, chunk_bytes: int, seed: int):
        self.B, self.C, self.seed = nbytes, chunk_bytes, seed
        b = np.arange(self.NBLK, dtype=np.uint64)
        aligned = (H(seed, 0, b) % np.uint64(4)) != 0
        j = (H(seed, 1, b) % np.uint64(9)).astype(np.int64)
        m = (H(seed, 2, b) % np.uint64(300)).astype(np.int64) + 1
        r = (H(seed, 3, b) % np.uint64(chunk_bytes)).astype(np.int64)
        self.blen = np.where(aligned, chunk_bytes * (1 << j), chunk_bytes * m + r).astype(np.int64)
        self.bpow2 = aligned
        ranks = np.arange(1, self.NBLK + 1, dtype=np.float64)
        pmf = ranks ** -1.1
        self.cdf = np.cumsum(pmf / pmf.sum())
        # initial item list: long enough to cover 2B of raw length (draws vectorised in
        # batches; item p uses H(seed, 5, p) and H(seed, 6, p) exactly as a scalar loop would)
        items = []
        total, p0 = 0, 0
        while total < 2 * nbytes:
            ps = np.arange(p0, p0 + 65536, dtype=np.uint64)
            u = H(seed, 5, ps).astype(np.float64) / 2.0 ** 64
            blks = np.minimum(np.searchsorted(self.cdf, u), self.NBLK - 1)
            als = self.bpow2[blks] & ((H(seed, 6, ps) % np.uint64(2)) == 0)
            lens = self.blen[blks]
            cum = total + np.cumsum(lens)
            stop = int(np.searchsorted(cum, 2 * nbytes)) + 1 if cum[-1] >= 2 * nbytes else len(ps)
            items.extend(("d", int(b), bool(a)) for b, a in zip(blks[:stop], als[:stop]))
            total = int(cum[stop - 1])
            p0 += 65536
        self.items = items
        self.k = 0
        self._dict_cache = {}   # dictionary block contents (fixed per block; perf-size lineages)

    def _content(self, item) -> np.ndarray:
        if item[0] == "d":
            blk = item[1]
            c = self._dict_cache.get(blk)
            if c is not None:
                return c
            key, ln = H(self.seed, 4, blk), int(self.blen[blk])
            nw = (ln + 7) // 8
            c = H(key, np.arange(nw, dtype=np.uint64)).astype("<u8").view(np.uint8)[:ln]
            self._dict_cache[blk] = c
            return c
        else:
            _, kk, pp, ln = item
            key = H(self.seed, 11, kk, pp)
        nw = (ln + 7) // 8
        return H(key, np.arange(nw, dtype=np.uint64)).astype("<u8").view(np.uint8)[:ln]

    def _len(self, item) -> int:
        return int(self.blen[item[1]]) if item[0] == "d" else item[3]

    def layout(self) -> np.ndarray:
        out = np.zeros(self.B, dtype=np.uint8)
        cur = 0
        for it in self.items:
            if cur >= self.B:
                break
            ln = self._len(it)
            if it[0] == "d" and it[2]:
                cur = (cur + ln - 1) // ln * ln
                if cur >= self.B:
                    break
            c = self._content(it)
            e = min(cur + ln, self.B)
            out[cur:e] = c[: e - cur]
            cur += ln
        return out

    def next(self) -> np.ndarray:
        """Returns the buffer of the next checkpoint (0, 1, 2, ...)."""
        if self.k > 0:
            k, s, P = self.k, self.seed, len(self.items)
            it = self.items
            ps = np.arange(P, dtype=np.uint64)
            swap = np.nonzero(H(s, 7, k, ps[0:P - 1:2]) < np.uint64(threshold(0.02)))[0] * 2
            for p in swap.tolist():
                it[p], it[p + 1] = it[p + 1], it[p]
            hit8 = H(s, 8, k, ps) < np.uint64(threshold(0.01))
            hit10 = H(s, 10, k, ps) < np.uint64(threshold(0.002))
            # sequential in p (a donor may be an item replaced earlier in this pass)
            for p in np.nonzero(hit8 | hit10)[0].tolist():
                if hit8[p]:
                    donor = it[int(H(s, 9, k, p)) % P]
                    if donor[0] == "d":
                        it[p] = ("d", donor[1], it[p][2] if it[p][0] == "d" else False)
                if hit10[p]:
                    it[p] = ("p", k, p, self._len(it[p]))
        self.k += 1
        return self.layout()


# ------------------------------------------------------------------ lineages
def lineage(cfg: int, nbytes: int, chunk_bytes: int, K: int, seed: int | None = None, p: float = 0.01):
    """Yields K host buffers (numpy uint8) of config cfg's lineage."""
    seed = seed_of(cfg) if seed is None else seed
    if cfg == 1:
        buf = cfg1_initial(nbytes, seed)
        yield buf.copy()
        for k in range(1, K):
            cfg1_mutate(buf, k, chunk_bytes, seed, p)
            yield buf.copy()
    elif cfg in (2, 3, 5):
        buf = cfg2_initial(nbytes, seed)
        yield buf.copy()
        for k in range(1, K):
            cfg2_mutate(buf, k, seed, p)
            yield buf.copy()
    elif cfg == 4:
        g = DupHeavy(nbytes, chunk_bytes, seed)
        for _ in range(K):
            yield g.next()
    else:
        raise ValueError(cfg)


# ------------------------------------------------------------------ device twins
class DeviceGen:
    """ctypes binding of libckptgen.so: the same generators, writing straight into a CUDA
    buffer (torch tensor or raw device pointer) on a stream."""

    _lib = None

    @classmethod
    def lib(cls):
        if cls._lib is None:
            import ctypes
            import os
            from .. import _build
            path = _build.lib_path("libckptgen.so")
            if not os.path.exists(path):
                raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
            L = ctypes.CDLL(path)
            vp, u32, u64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64
            L.gen_cfg1_initial.argtypes = [vp, u64, u64, vp]
            L.gen_cfg1_mutate.argtypes = [vp, u64, u32, u32, u64, u64, vp]
            L.gen_cfg2_initial.argtypes = [vp, u64, u64, u64, vp]
            L.gen_cfg2_mutate.argtypes = [vp, u64, u32, u64, u64, vp]
            L.gen_freq_orbits.argtypes = [vp]
            for f in ("gen_cfg1_initial", "gen_cfg1_mutate", "gen_cfg2_initial", "gen_cfg2_mutate", "gen_freq_orbits"):
                getattr(L, f).restype = ctypes.c_int
            cls._lib = L
        return cls._lib

    @staticmethod
    def _args(buf, stream):
        ptr = buf.data_ptr() if hasattr(buf, "data_ptr") else int(buf)
        st = stream.cuda_stream if hasattr(stream, "cuda_stream") else (int(stream) if stream else 0)
        return ptr, st

    @classmethod
    def freq_orbits(cls):
        arr = np.zeros(32, dtype=np.int32)
        n = cls.lib().gen_freq_orbits(arr.ctypes.data)
        return arr[:n].astype(np.int64)

    @classmethod
    def initial(cls, cfg: int, buf, nbytes: int, seed: int, stream=None):
        ptr, st = cls._args(buf, stream)
        if cfg == 1:
            rc = cls.lib().gen_cfg1_initial(ptr, nbytes, seed, st)
        elif cfg in (2, 3, 5):
            rc = cls.lib().gen_cfg2_initial(ptr, nbytes, seed, threshold(0.3), st)
        else:
            raise ValueError(f"config {cfg} has no device generator (host only)")
        if rc:
            raise RuntimeError(f"generator launch failed ({rc})")

    @classmethod
    def mutate(cls, cfg: int, buf, nbytes: int, k: int, chunk_bytes: int, seed: int, p: float, stream=None):
        ptr, st = cls._args(buf, stream)
        if cfg == 1:
            rc = cls.lib().gen_cfg1_mutate(ptr, nbytes, chunk_bytes, k, seed, threshold(p), st)
        elif cfg in (2, 3, 5):
            rc = cls.lib().gen_cfg2_mutate(ptr, nbytes, k, seed, threshold(p), st)
        else:
            raise ValueError(cfg)
        if rc:
            raise RuntimeError(f"generator launch failed ({rc})")
