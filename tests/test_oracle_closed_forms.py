"""Closed-form cases of the method pinning the
oracle's phases 2/3, emission and serialisation."""
import numpy as np
import pytest


def rand_chunks(rng, n, C):
    return [rng.integers(0, 256, C, dtype=np.uint8).tobytes() for _ in range(n)]


def align16(x):
    return (x + 15) // 16 * 16


@pytest.mark.parametrize("n", [1, 2, 3, 5, 8, 13, 16, 31, 64])
def test_all_distinct_then_unchanged(oracle_mod, n):
    C = 32
    rng = np.random.default_rng(n)
    buf = b"".join(rand_chunks(rng, n, C))
    o = oracle_mod.Oracle(C)
    o.checkpoint(buf)
    d0 = oracle_mod.parse_diff(o.diff(0))
    # fully unique checkpoint 0: the whole tree is FIRST -> one region, the root (R10)
    assert d0["first"] == [0] and d0["shift"] == []
    assert d0["data"] == buf and d0["data_bytes"] == len(buf)
    assert o.record_size() == 2 * n - 1
    o.checkpoint(buf)
    d1 = o.diff(1)
    assert len(d1) == 64                                     # unchanged -> header only
    p = oracle_mod.parse_diff(d1)
    assert p["first"] == [] and p["shift"] == [] and p["data_bytes"] == 0
    assert o.record_size() == 2 * n - 1


@pytest.mark.parametrize("n,i", [(8, 3), (16, 0), (16, 15), (13, 6), (64, 40)])
def test_one_changed_chunk(oracle_mod, n, i):
    C = 64
    rng = np.random.default_rng(7 * n + i)
    ch = rand_chunks(rng, n, C)
    o = oracle_mod.Oracle(C)
    o.checkpoint(b"".join(ch))
    before = o.record_size()
    ch[i] = rng.integers(0, 256, C, dtype=np.uint8).tobytes()
    o.checkpoint(b"".join(ch))
    d = oracle_mod.parse_diff(o.diff(1))
    assert d["first"] == [o.node_of_chunk(i)] and d["shift"] == []
    assert o.record_size() == before + 1
    assert len(o.diff(1)) == 80 + C                          # align16(64+4) + C


@pytest.mark.parametrize("n,j", [(8, 1), (16, 0), (16, 7), (32, 5)])
def test_two_sibling_chunks_changed(oracle_mod, n, j):
    C = 32
    rng = np.random.default_rng(100 + n + j)
    ch = rand_chunks(rng, n, C)
    o = oracle_mod.Oracle(C)
    o.checkpoint(b"".join(ch))
    before = o.record_size()
    ch[2 * j] = rng.integers(0, 256, C, dtype=np.uint8).tobytes()
    ch[2 * j + 1] = rng.integers(0, 256, C, dtype=np.uint8).tobytes()
    o.checkpoint(b"".join(ch))
    d = oracle_mod.parse_diff(o.diff(1))
    parent = (o.node_of_chunk(2 * j) - 1) // 2
    assert d["first"] == [parent] and d["shift"] == []
    assert o.record_size() == before + 3                     # two leaves + their parent


@pytest.mark.parametrize("h,j,a,b", [(4, 2, 0, 2), (4, 1, 3, 6), (5, 3, 1, 3), (6, 4, 0, 3), (3, 3, 0, 0)])
def test_aligned_block_copy_is_one_shift_region(oracle_mod, h, j, a, b):
    """An aligned 2^j-chunk block copied from an aligned block that was FIRST in
    checkpoint 0 collapses into ONE shifted-duplicate region."""
    n, C = 1 << h, 32
    rng = np.random.default_rng(h * 100 + j * 10 + a + b)
    ch = rand_chunks(rng, n, C)
    o = oracle_mod.Oracle(C)
    o.checkpoint(b"".join(ch))
    blk = 1 << j
    new = list(ch)
    new[b * blk:(b + 1) * blk] = ch[a * blk:(a + 1) * blk]
    o.checkpoint(b"".join(new))
    d = oracle_mod.parse_diff(o.diff(1))
    node_at = lambda pos: (1 << (h - j)) - 1 + pos            # node of the aligned block
    if a == b:
        assert d["first"] == [] and d["shift"] == []
    else:
        assert d["first"] == [] and d["shift"] == [(node_at(b), node_at(a), 0)]


@pytest.mark.parametrize("n", [2, 4, 7, 16, 33])
def test_all_zero_checkpoint0(oracle_mod, n):
    """Reading R9 (SHIFT-SHIFT parents absent from the record are not inserted):
    an all-zero checkpoint 0 gives 1 FIRST + (n-1) SHIFT leaf regions; the FIRST leaf
    is the minimum node id n-1 (R6), which is chunk 0 when n is a power of two."""
    C = 32
    o = oracle_mod.Oracle(C)
    o.checkpoint(bytes(n * C))
    d = oracle_mod.parse_diff(o.diff(0))
    z = n - 1
    assert d["first"] == [z]
    if n & (n - 1) == 0:
        assert z == o.node_of_chunk(0)
    assert sorted(s[0] for s in d["shift"]) == list(range(n, 2 * n - 1))
    assert all((s[1], s[2]) == (z, 0) for s in d["shift"])
    assert d["data"] == bytes(C)
    assert len(o.diff(0)) == align16(64 + 4 + 12 * (n - 1)) + C


def test_partial_last_chunk_only_matches_equal_length(oracle_mod):
    """R4: the last chunk is hashed at its true length, so a short last chunk equal to
    a prefix of another chunk is NOT a duplicate."""
    C = 32
    rng = np.random.default_rng(5)
    a = rng.integers(0, 256, C, dtype=np.uint8).tobytes()
    buf = a + a[:20]
    o = oracle_mod.Oracle(C)
    o.checkpoint(buf)
    lab, _, _ = o.leaf_labels(0)
    assert list(lab) == [1, 1]
    assert o.restore(0) == buf
