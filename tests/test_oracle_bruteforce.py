"""Pins the oracle's leaf classification (Alg.1 l.1-23, reading R6) to a
brute-force memcmp definition, and the record size to its closed form."""
import numpy as np
import pytest

from tests._lineages import dup_lineage

FIRST, FIXED, SHIFT = 1, 2, 3


def brute_labels(bufs, C, o):
    """For content x: c*(x) = first checkpoint containing x; node*(x) = minimum node id
    holding x in c*. A non-FIXED leaf is FIRST iff (node, k) == (node*, c*)."""
    first_seen = {}
    out = []
    for k, b in enumerate(bufs):
        B = len(b)
        n = (B + C - 1) // C
        chunks = [bytes(b[i * C:min((i + 1) * C, B)]) for i in range(n)]
        nodes = [o.node_of_chunk(i) for i in range(n)]
        prev = None if k == 0 else [bytes(bufs[k - 1][i * C:min((i + 1) * C, B)]) for i in range(n)]
        cand = {}
        for i in range(n):
            if prev is not None and chunks[i] == prev[i]:
                continue
            x = chunks[i]
            if x not in first_seen:
                cand[x] = min(cand.get(x, 1 << 62), nodes[i])
        for x, u in cand.items():
            first_seen[x] = (u, k)
        lab = []
        for i in range(n):
            if prev is not None and chunks[i] == prev[i]:
                lab.append((FIXED, None))
            else:
                s = first_seen[chunks[i]]
                lab.append((FIRST, None) if s == (nodes[i], k) else (SHIFT, s))
        out.append(lab)
    return out, first_seen


@pytest.mark.parametrize("seed", range(40))
def test_leaf_classification_matches_bruteforce(oracle_mod, seed):
    rng = np.random.default_rng(1000 + seed)
    C = int(rng.choice([32, 48, 64]))
    nbytes = int(rng.integers(1, 40)) * C - int(rng.integers(0, C)) * int(rng.integers(0, 2))
    nbytes = max(nbytes, 1)
    bufs = dup_lineage(seed, nbytes, C, K=int(rng.integers(2, 6)))
    o = oracle_mod.Oracle(C)
    for b in bufs:
        o.checkpoint(b)
    want, first_seen = brute_labels(bufs, C, o)
    for k in range(len(bufs)):
        lab, sn, sc = o.leaf_labels(k)
        for i, (l, s) in enumerate(want[k]):
            assert lab[i] == l, (k, i)
            if l == SHIFT:
                assert (int(sn[i]), int(sc[i])) == s


@pytest.mark.parametrize("seed", range(20))
def test_record_growth_bound_and_leaf_entries(oracle_mod, seed):
    rng = np.random.default_rng(seed)
    C = 32
    n = int(rng.integers(1, 70))
    bufs = dup_lineage(500 + seed, n * C, C, K=4)
    o = oracle_mod.Oracle(C)
    prev_size = 0
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        st = o.stats(k)
        grow = o.record_size() - prev_size
        prev_size = o.record_size()
        # record = FIRST leaves + FIRST internal nodes, growth <= 2n-1
        assert grow == st["n_first"] + st["phase2_inserts"] == st["record_growth"]
        assert grow <= 2 * n - 1
        assert st["n_first"] + st["n_fixed"] + st["n_spatial"] + st["n_temporal"] == n
        assert st["list_entries"] == n - st["n_fixed"]
