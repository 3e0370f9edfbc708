"""Ideal-hash mode (exact content keys, no digests) must give byte-identical diffs
(R14: digest equality == content equality), and the tree geometry (R3) is checked by
brute force for complete and incomplete trees."""
import numpy as np
import pytest

from tests._lineages import dup_lineage


@pytest.mark.parametrize("seed", range(30))
def test_ideal_hash_mode_identical(oracle_mod, seed):
    rng = np.random.default_rng(300 + seed)
    C = int(rng.choice([32, 64]))
    n = int(rng.integers(1, 70))
    nbytes = max(1, n * C - (int(rng.integers(0, C)) if rng.random() < 0.3 else 0))
    bufs = dup_lineage(seed + 77, nbytes, C, K=4)
    a, b = oracle_mod.Oracle(C), oracle_mod.Oracle(C, ideal=True)
    for buf in bufs:
        a.checkpoint(buf)
        b.checkpoint(buf)
    for k in range(len(bufs)):
        assert a.diff(k) == b.diff(k)
        assert a.stats(k) == b.stats(k)


@pytest.mark.parametrize("n", list(range(1, 80)) + [127, 128, 129, 1000])
def test_geometry_inorder_contiguous(oracle_mod, n):
    o = oracle_mod.Oracle(16)
    o.checkpoint(bytes(16 * n))
    assert o.n_leaves == n
    leaves = [o.node_of_chunk(i) for i in range(n)]
    assert sorted(leaves) == list(range(n - 1, 2 * n - 1))    # bijection onto leaves
    # in-order traversal of the heap visits chunks 0..n-1 in order
    order = []

    def walk(u):
        if u >= n - 1:
            order.append(u)
            return
        walk(2 * u + 1)
        walk(2 * u + 2)
    walk(0)
    assert order == leaves
    for u in range(n - 1):                                      # children ranges concatenate
        l, r = 2 * u + 1, 2 * u + 2
        assert o.lo(u) == o.lo(l) and o.hi(l) == o.lo(r) and o.hi(r) == o.hi(u)
    assert o.lo(0) == 0 and o.hi(0) == n
    if n & (n - 1) == 0:
        assert leaves == list(range(n - 1, 2 * n - 1))          # Fig. 2: node = n-1+i
