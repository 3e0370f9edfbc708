"""Pins the oracle's Tree-method variants (readings R22, R23):

  VAR_FULL_FIRST  checkpoint 0 "taken fully": Algorithm 1 runs as usual, so
                  the record is the one Fig. 2 describes, but the difference is the whole
                  buffer (one FIRST region, the root).
  VAR_FULL_SWITCH incremental checkpointing "deactivated" when the data "fully changes
                  during the checkpoint interval": at k >= 1, at least
                  switch_permille / 1000 of the leaves not FIXED -> a full difference, no
                  record operation, leaf digests still updated (l.21).

Pins: the full format built by hand from DESIGN.md §4; Fig. 2 with checkpoint 0 taken
fully (record = nodes 0-14; regions {1, 6, 12}); brute-force memcmp leaf
classification that ignores switched checkpoints; the switch threshold boundary; closed
forms for the checkpoint after a switch; restore(k) == input_k."""
import struct

import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_oracle_bruteforce import FIRST, FIXED, SHIFT

FULL_FIRST, FULL_SWITCH = 1, 2


def full_form(k, C, buf):
    """The full difference written out from the format (R22)."""
    B = len(buf)
    n = (B + C - 1) // C
    hdr = struct.pack("<IHHIIQQQQQII", 0x44504B43, 1, 3, k, C, B, n, 1, 0, B, 0, 0)
    meta = hdr + struct.pack("<I", 0)
    meta += b"\0" * (-len(meta) % 16)
    assert len(meta) == 80
    return meta + bytes(buf)


def fig2_bufs(C=32):
    rng = np.random.default_rng(2)
    A = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(8)]
    I, J, K, L = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(4)]
    return [np.concatenate(A), np.concatenate([I, J, K, L, A[4], A[0], I, J])]


def test_fig2_first_checkpoint_taken_fully(oracle_mod):
    """"a single first checkpoint that was taken fully and the historical record of
    unique hashes consists of all possible non-overlapping regions corresponding to the
    intermediate nodes 0-14"; the second checkpoint is regions 1, 6, 12."""
    C = 32
    b0, b1 = fig2_bufs(C)
    o = oracle_mod.Oracle(C)
    o.set_variant(FULL_FIRST)
    o.checkpoint(b0)
    assert o.diff(0) == full_form(0, C, b0)
    assert sorted((u, c) for _, u, c in o.record()) == [(u, 0) for u in range(15)]
    st = o.stats(0)
    assert (st["n_first_regions"], st["n_shift_regions"], st["data_bytes"], st["meta_bytes"]) == (1, 0, 8 * C, 80)
    assert st["n_first"] == 8 and st["record_growth"] == 15
    o.checkpoint(b1)
    d = oracle_mod.parse_diff(o.diff(1))
    assert d["flags"] == 0
    assert d["first"] == [1] and d["shift"] == [(12, 7, 0), (6, 3, 1)]
    assert o.restore(0) == b0.tobytes() and o.restore(1) == b1.tobytes()


def test_full_first_zero_buffer(oracle_mod):
    """An all-zero checkpoint 0 (1 FIRST + n-1 SHIFT leaf regions by default, R9) becomes
    one region; the record still holds only chunk 0's digest (Alg.1 runs unchanged)."""
    C, n = 64, 37
    buf = np.zeros(n * C, dtype=np.uint8)
    o = oracle_mod.Oracle(C)
    o.set_variant(FULL_FIRST)
    o.checkpoint(buf)
    assert o.diff(0) == full_form(0, C, buf)
    st = o.stats(0)
    assert st["n_first"] == 1 and st["n_spatial"] == n - 1 and o.record_size() == 1
    assert o.restore(0) == buf.tobytes()


def brute_labels_switch(bufs, C, o, switched):
    """brute_labels (test_oracle_bruteforce) with switched checkpoints never entering the
    record: c*(x) = first NON-switched checkpoint containing x at a non-FIXED leaf."""
    first_seen = {}
    out = []
    for k, b in enumerate(bufs):
        B = len(b)
        n = (B + C - 1) // C
        chunks = [bytes(b[i * C:min((i + 1) * C, B)]) for i in range(n)]
        nodes = [o.node_of_chunk(i) for i in range(n)]
        prev = None if k == 0 else [bytes(bufs[k - 1][i * C:min((i + 1) * C, B)]) for i in range(n)]
        fixed = [prev is not None and chunks[i] == prev[i] for i in range(n)]
        if switched[k]:
            out.append([(FIXED, None) if fixed[i] else (FIRST, None) for i in range(n)])
            continue
        cand = {}
        for i in range(n):
            if not fixed[i] and chunks[i] not in first_seen:
                cand[chunks[i]] = min(cand.get(chunks[i], 1 << 62), nodes[i])
        for x, u in cand.items():
            first_seen[x] = (u, k)
        lab = []
        for i in range(n):
            if fixed[i]:
                lab.append((FIXED, None))
            else:
                s = first_seen[chunks[i]]
                lab.append((FIRST, None) if s == (nodes[i], k) else (SHIFT, s))
        out.append(lab)
    return out


def changed_count(bufs, k, C):
    B = len(bufs[k])
    n = (B + C - 1) // C
    if k == 0:
        return n
    return sum(bytes(bufs[k][i * C:(i + 1) * C]) != bytes(bufs[k - 1][i * C:(i + 1) * C]) for i in range(n))


@pytest.mark.parametrize("seed", range(30))
def test_switch_matches_bruteforce(oracle_mod, seed):
    rng = np.random.default_rng(3000 + seed)
    C = int(rng.choice([32, 48, 64]))
    nbytes = max(1, int(rng.integers(1, 40)) * C - int(rng.integers(0, C)) * int(rng.integers(0, 2)))
    bufs = dup_lineage(seed, nbytes, C, K=int(rng.integers(3, 7)), p_change=float(rng.choice([0.2, 0.6, 0.95])))
    permille = int(rng.choice([0, 100, 400, 700, 1000]))
    flags = FULL_SWITCH | (FULL_FIRST if seed % 2 else 0)
    o = oracle_mod.Oracle(C)
    o.set_variant(flags, permille)
    for b in bufs:
        o.checkpoint(b)
    n = (nbytes + C - 1) // C
    switched = [k >= 1 and 1000 * changed_count(bufs, k, C) >= permille * n for k in range(len(bufs))]
    want = brute_labels_switch(bufs, C, o, switched)
    size = 0
    for k, b in enumerate(bufs):
        lab, sn, sc = o.leaf_labels(k)
        for i, (l, s) in enumerate(want[k]):
            assert lab[i] == l, (k, i)
            if l == SHIFT:
                assert (int(sn[i]), int(sc[i])) == s
        st = o.stats(k)
        if switched[k] or (k == 0 and flags & FULL_FIRST):
            assert o.diff(k) == full_form(k, C, b), k
        else:
            assert oracle_mod.parse_diff(o.diff(k))["flags"] == 0
        if switched[k]:
            assert st["record_growth"] == 0 and st["n_first"] == changed_count(bufs, k, C)
            assert st["n_spatial"] == st["n_temporal"] == 0
        assert st["n_first"] + st["n_fixed"] + st["n_spatial"] + st["n_temporal"] == n
        size += st["record_growth"]
    assert o.record_size() == size
    for k, b in enumerate(bufs):
        assert o.restore(k) == b.tobytes(), k


def test_switch_threshold_boundary(oracle_mod):
    """n = 16 leaves, permille = 250: 4 changed chunks switch, 3 do not (1000 c >= 250 n)."""
    C, n = 32, 16
    rng = np.random.default_rng(7)
    b0 = rng.integers(0, 256, n * C, dtype=np.uint8)
    o = oracle_mod.Oracle(C)
    o.set_variant(FULL_SWITCH, 250)
    o.checkpoint(b0)
    assert oracle_mod.parse_diff(o.diff(0))["flags"] == 0    # k = 0 is never switched
    assert o.record_size() == 2 * n - 1
    b1 = b0.copy()
    for i in (1, 5, 9):
        b1[i * C] ^= 0xFF
    o.checkpoint(b1)
    d1 = oracle_mod.parse_diff(o.diff(1))
    assert d1["flags"] == 0 and len(d1["first"]) == 3 and d1["shift"] == []
    b2 = b1.copy()
    for i in (0, 2, 4, 6):
        b2[i * C] ^= 0x0F
    o.checkpoint(b2)
    assert o.diff(2) == full_form(2, C, b2)
    st = o.stats(2)
    assert (st["n_first"], st["n_fixed"], st["record_growth"]) == (4, 12, 0)
    for k, b in enumerate([b0, b1, b2]):
        assert o.restore(k) == b.tobytes()


def test_after_switch_closed_forms(oracle_mod):
    """After a switched checkpoint k: (i) leaves equal to checkpoint k are FIXED (l.21 ran),
    so one changed chunk gives one FIRST leaf region, diff = 80 + C; (ii) content that
    first appeared in k is unknown to the record: moved elsewhere in k+1 it is FIRST."""
    C, n = 64, 32
    rng = np.random.default_rng(11)
    b0 = rng.integers(0, 256, n * C, dtype=np.uint8)
    o = oracle_mod.Oracle(C)
    o.set_variant(FULL_SWITCH, 1000)
    o.checkpoint(b0)
    g0 = o.record_size()
    b1 = rng.integers(0, 256, n * C, dtype=np.uint8)   # every chunk changes: switched
    o.checkpoint(b1)
    assert o.diff(1) == full_form(1, C, b1) and o.record_size() == g0
    b2 = b1.copy()
    b2[3 * C] ^= 1
    o.checkpoint(b2)
    assert len(o.diff(2)) == 80 + C
    d2 = oracle_mod.parse_diff(o.diff(2))
    assert d2["first"] == [o.node_of_chunk(3)] and d2["shift"] == []
    b3 = b2.copy()
    b3[7 * C:8 * C] = b1[20 * C:21 * C]                 # content first seen in switched ckpt 1
    o.checkpoint(b3)
    lab, _, _ = o.leaf_labels(3)
    assert lab[7] == FIRST
    b4 = b3.copy()
    b4[9 * C:10 * C] = b0[2 * C:3 * C]                  # content of ckpt 0: temporal SHIFT
    o.checkpoint(b4)
    lab, sn, sc = o.leaf_labels(4)
    assert lab[9] == SHIFT and (int(sn[9]), int(sc[9])) == (o.node_of_chunk(2), 0)
    for k, b in enumerate([b0, b1, b2, b3, b4]):
        assert o.restore(k) == b.tobytes()


def test_variant_rejections(oracle_mod):
    o = oracle_mod.Oracle(32, mode=oracle_mod.MODE_LIST)
    with pytest.raises(ValueError):
        o.set_variant(FULL_FIRST)
    o = oracle_mod.Oracle(32)
    with pytest.raises(ValueError):
        o.set_variant(FULL_SWITCH, 1001)
    with pytest.raises(ValueError):
        o.set_variant(8)                 # unknown flag bit (4 is the SHIFT-insert variant)
    o.checkpoint(np.zeros(64, dtype=np.uint8))
    with pytest.raises(ValueError):
        o.set_variant(FULL_FIRST)


def test_ideal_mode_variants_same_regions(oracle_mod):
    """Exact content keys give the same diffs under both variants (R14 pin, as for Tree)."""
    C = 48
    bufs = dup_lineage(77, 50 * C - 5, C, K=6, p_change=0.7)
    a, b = oracle_mod.Oracle(C), oracle_mod.Oracle(C, ideal=True)
    for o in (a, b):
        o.set_variant(FULL_FIRST | FULL_SWITCH, 500)
        for x in bufs:
            o.checkpoint(x)
    for k in range(len(bufs)):
        assert a.diff(k) == b.diff(k), k
