"""restore(k) == checkpoint k, byte format (R13) and region invariants checked
against the raw buffers with memcmp only (independent of the oracle's record)."""
import struct

import numpy as np
import pytest

from tests._lineages import dup_lineage

FIRST, FIXED, SHIFT = 1, 2, 3


def check_diff_invariants(oracle_mod, o, bufs, k, C):
    B = len(bufs[k])
    n = (B + C - 1) // C
    raw = o.diff(k)
    d = oracle_mod.parse_diff(raw)
    assert d["magic"] == 0x44504B43 and d["version"] == 1 and d["id"] == k
    assert d["chunk_bytes"] == C and d["buf_bytes"] == B and d["n_leaves"] == n
    assert d["seed"] == 0
    meta = 64 + 4 * len(d["first"]) + 12 * len(d["shift"])
    assert raw[meta:d["meta_bytes"]] == bytes(d["meta_bytes"] - meta)  # zero pad
    assert len(raw) == d["meta_bytes"] + d["data_bytes"]
    blen = lambda u: min(o.hi(u) * C, B) - o.lo(u) * C
    regions = [(o.lo(u), o.hi(u), FIRST, u, None) for u in d["first"]] + \
              [(o.lo(u), o.hi(u), SHIFT, u, (v, c)) for (u, v, c) in d["shift"]]
    # each list sorted by lo; regions disjoint
    assert [o.lo(u) for u in d["first"]] == sorted(o.lo(u) for u in d["first"])
    assert [o.lo(s[0]) for s in d["shift"]] == sorted(o.lo(s[0]) for s in d["shift"])
    regions.sort()
    covered = np.zeros(n, dtype=bool)
    for lo, hi, _, _, _ in regions:
        assert not covered[lo:hi].any()
        covered[lo:hi] = True
    # covered chunks == non-FIXED chunks (memcmp against checkpoint k-1)
    cur = bufs[k]
    for i in range(n):
        a, b = i * C, min((i + 1) * C, B)
        fixed = k > 0 and bytes(cur[a:b]) == bytes(bufs[k - 1][a:b])
        assert covered[i] == (not fixed), i
    # data == FIRST regions' bytes in lo order; SHIFT content equals its source content
    data = b"".join(bytes(cur[o.lo(u) * C:o.lo(u) * C + blen(u)]) for u in d["first"])
    assert d["data"] == data
    for (u, v, c) in d["shift"]:
        assert c <= k and blen(u) == blen(v)
        assert bytes(cur[o.lo(u) * C:o.lo(u) * C + blen(u)]) == bytes(bufs[c][o.lo(v) * C:o.lo(v) * C + blen(v)])


@pytest.mark.parametrize("seed", range(60))
def test_restore_invariant_random_lineages(oracle_mod, seed):
    rng = np.random.default_rng(seed)
    C = int(rng.choice([32, 48, 64, 128]))
    n = int(rng.integers(1, 90))
    tail = int(rng.integers(0, C)) if rng.random() < 0.5 else 0
    nbytes = max(1, n * C - tail)
    bufs = dup_lineage(seed, nbytes, C, K=int(rng.integers(1, 6)))
    o = oracle_mod.Oracle(C)
    for b in bufs:
        o.checkpoint(b)
    for k, b in enumerate(bufs):
        assert o.restore(k) == bytes(b)
        check_diff_invariants(oracle_mod, o, bufs, k, C)


def test_size_change_rejected(oracle_mod):
    o = oracle_mod.Oracle(32)
    o.checkpoint(bytes(64))
    with pytest.raises(RuntimeError):
        o.checkpoint(bytes(96))
