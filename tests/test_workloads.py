"""Host workload generators (harness): determinism and the statistical shape the
DESIGN.md §6 recipes promise; plus the oracle on the full config-1 lineage."""
import time

import numpy as np

from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W


def test_counter_hash_reference_values():
    # splitmix64 of 0 after one golden-ratio increment (the classic SplitMix64 first output)
    assert int(W.splitmix64(np.uint64(0x9E3779B97F4A7C15))) == 0xE220A8397B1DCDAF
    assert int(W.H(0, 0)) == 0xE220A8397B1DCDAF
    assert int(W.H(5, 1, 2)) == int(W.H(W.H(5, 1), 2))


def test_geo_mean_three():
    x = W.H(123, np.arange(200000, dtype=np.uint64))
    g = W.geo(x)
    assert abs(g.mean() - 3.0) < 0.05


def test_cfg1_change_fraction_and_determinism():
    B, C = 1 << 20, 128
    a = list(W.lineage(1, B, C, 4))
    b = list(W.lineage(1, B, C, 4))
    assert all((x == y).all() for x, y in zip(a, b))
    n = B // C
    for k in range(1, 4):
        ch = (a[k].reshape(n, C) != a[k - 1].reshape(n, C)).any(axis=1).sum()
        assert 40 < ch < 130        # E = 82 at p = 1 %


def test_cfg2_gdv_shape():
    B = 1 << 22
    bufs = list(W.lineage(2, B, 128, 3, p=0.05))
    R = W.cfg2_rows(B)
    c0 = bufs[0][:R * 292].view("<u4").reshape(R, 73)
    other = np.setdiff1d(np.arange(73), W.FREQ_ORBITS)
    assert (c0[:, other] == 0).all()
    zero_rows = (c0 == 0).all(axis=1).mean()
    assert 0.35 < zero_rows < 0.65
    assert (bufs[0][R * 292:] == 0).all()
    c2 = bufs[2][:R * 292].view("<u4").reshape(R, 73)
    assert (c2 >= c0).all() and (c2 > c0).any()    # counts only grow


def test_cfg4_dup_heavy_has_duplicates(oracle_mod):
    B, C = 1 << 20, 128
    bufs = list(W.lineage(4, B, C, 3))
    o = oracle_mod.Oracle(C)
    for b in bufs:
        o.checkpoint(b)
    st0, st1 = o.stats(0), o.stats(1)
    assert st0["n_spatial"] > 0.2 * st0["n_leaves"]      # many spatial duplicates
    assert st1["n_temporal"] > 0
    assert st0["n_first_regions"] + st0["n_shift_regions"] < st0["list_entries"]
    for k, b in enumerate(bufs):
        assert o.restore(k) == bytes(b)


def test_oracle_full_cfg1_lineage_fast(oracle_mod):
    B, C = 1 << 20, 128
    o = oracle_mod.Oracle(C)
    t = time.time()
    for b in W.lineage(1, B, C, 10):
        o.checkpoint(b)
    assert time.time() - t < 30
    st = o.stats(5)
    assert st["n_fixed"] > 0.97 * (B // C)
    assert st["n_spatial"] == 0
