"""Pins of the oracle's List and Basic methods to plain
definitions: memcmp brute force, Figure 2's entry count, closed-form sizes, and the
restore invariant. Neither pin re-derives the oracle's own arithmetic: List entries are
checked against the brute-force leaf classification (tests/test_oracle_bruteforce.py),
Basic bitmaps against byte comparison with the previous buffer."""
import json
import os

import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_oracle_bruteforce import FIRST, FIXED, SHIFT, brute_labels
from tests.test_oracle_fig2 import GOLD, _content


def _chunks(b, C):
    n = (len(b) + C - 1) // C
    return [bytes(b[i * C:min((i + 1) * C, len(b))]) for i in range(n)]


def _random_case(seed):
    rng = np.random.default_rng(7000 + seed)
    C = int(rng.choice([32, 48, 64, 128]))
    nbytes = max(1, int(rng.integers(1, 60)) * C - int(rng.integers(0, C)) * int(rng.integers(0, 2)))
    return C, dup_lineage(300 + seed, nbytes, C, K=int(rng.integers(2, 6)))


@pytest.mark.parametrize("seed", range(30))
def test_list_entries_are_the_bruteforce_leaves(oracle_mod, seed):
    """List ("a full list of all first-time occurrences and shifted duplicates"):
    one entry per non-FIXED leaf in chunk order, FIRST/SHIFT and source as brute force says;
    data = the FIRST chunks in chunk order; size = align16(64 + 4 nF + 12 nS) + FIRST bytes."""
    C, bufs = _random_case(seed)
    o = oracle_mod.Oracle(C, mode=oracle_mod.MODE_LIST)
    for b in bufs:
        o.checkpoint(b)
    want, _ = brute_labels(bufs, C, o)
    for k, b in enumerate(bufs):
        d = oracle_mod.parse_diff(o.diff(k))
        assert d["flags"] == oracle_mod.MODE_LIST
        ch = _chunks(b, C)
        exp_f = [o.node_of_chunk(i) for i, (l, _) in enumerate(want[k]) if l == FIRST]
        exp_s = [(o.node_of_chunk(i),) + tuple(s) for i, (l, s) in enumerate(want[k]) if l == SHIFT]
        assert d["first"] == exp_f
        assert [tuple(x) for x in d["shift"]] == exp_s
        exp_data = b"".join(ch[i] for i, (l, _) in enumerate(want[k]) if l == FIRST)
        assert d["data"] == exp_data
        size = (64 + 4 * len(exp_f) + 12 * len(exp_s) + 15) // 16 * 16 + len(exp_data)
        assert len(o.diff(k)) == size
        assert o.restore(k) == bytes(b)


@pytest.mark.parametrize("seed", range(30))
def test_basic_bitmap_and_data_bruteforce(oracle_mod, seed):
    """Basic ("a bitmap to indicate what chunks are new and what chunks remain
    unchanged. It saves the bitmap and the new chunks"): bit i = chunk i differs from chunk i
    of the previous buffer (all set at checkpoint 0, P:198's full initial checkpoint)."""
    C, bufs = _random_case(seed)
    o = oracle_mod.Oracle(C, mode=oracle_mod.MODE_BASIC)
    for b in bufs:
        o.checkpoint(b)
    for k, b in enumerate(bufs):
        d = oracle_mod.parse_diff(o.diff(k))
        assert d["flags"] == oracle_mod.MODE_BASIC
        ch = _chunks(b, C)
        prev = _chunks(bufs[k - 1], C) if k else None
        changed = [i for i in range(len(ch)) if prev is None or ch[i] != prev[i]]
        assert d["changed"] == changed and d["n_changed"] == len(changed)
        data = b"".join(ch[i] for i in changed)
        assert d["data"] == data and d["data_bytes"] == len(data)
        n = len(ch)
        assert len(o.diff(k)) == (64 + 4 * ((n + 31) // 32) + 15) // 16 * 16 + len(data)
        assert o.restore(k) == bytes(b)


def test_fig2_list_has_seven_entries(oracle_mod):
    """the naive method "saves a metadata entry for each non-fixed duplicate chunk
    (referred to as the List method)" — 7 entries for Figure 2's second checkpoint."""
    g = json.load(open(GOLD))
    C = g["chunk_bytes"]
    cont = {nm: _content(nm, C) for nm in set(g["ckpt0"] + g["ckpt1"])}
    o = oracle_mod.Oracle(C, mode=oracle_mod.MODE_LIST)
    o.checkpoint(b"".join(cont[x] for x in g["ckpt0"]))
    o.checkpoint(b"".join(cont[x] for x in g["ckpt1"]))
    d = oracle_mod.parse_diff(o.diff(1))
    assert len(d["first"]) + len(d["shift"]) == g["ckpt1_list_entries"] == 7
    assert d["first"] == [7, 8, 9, 10]                      # I, J, K, L
    assert [tuple(x) for x in d["shift"]] == [(12, 7, 0), (13, 7, 1), (14, 8, 1)]
    # checkpoint 0 (taken fully, all distinct): one entry per chunk, no compaction
    d0 = oracle_mod.parse_diff(o.diff(0))
    assert d0["first"] == list(range(7, 15)) and d0["shift"] == []


@pytest.mark.parametrize("seed", range(10))
def test_methods_agree_where_they_must(oracle_mod, seed):
    """Tree and List carry the same first-occurrence data (the FIRST chunks in chunk order);
    Basic's changed-chunk count is the non-FIXED leaf count of the other two."""
    C, bufs = _random_case(100 + seed)
    o = {m: oracle_mod.Oracle(C, mode=m) for m in (oracle_mod.MODE_TREE, oracle_mod.MODE_LIST,
                                                   oracle_mod.MODE_BASIC)}
    for b in bufs:
        for x in o.values():
            x.checkpoint(b)
    for k in range(len(bufs)):
        t, l, bs = (oracle_mod.parse_diff(o[m].diff(k)) for m in (0, 1, 2))
        assert t["data"] == l["data"]
        st = o[0].stats(k)
        assert bs["n_changed"] == st["n_leaves"] - st["n_fixed"]
        assert len(l["first"]) + len(l["shift"]) == st["list_entries"]
        assert o[1].record_size() <= o[0].record_size()   # List keeps leaves only
