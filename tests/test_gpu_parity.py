"""GPU <-> oracle parity through the C ABI (libckpt.so): bit-exact diffs, leaf digests,
leaf classification statistics, record sets and restores on the same seeded inputs.

Tolerance: none — every output is integer/byte data, so the bar is bit-exact.
"""
import numpy as np
import pytest

from tests._lineages import dup_lineage

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _dev(buf: np.ndarray):
    t = torch.empty(max(buf.size, 1), dtype=torch.uint8, device="cuda")
    t[: buf.size].copy_(torch.from_numpy(np.ascontiguousarray(buf)))
    return t


STAT_KEYS = ["n_first_regions", "n_shift_regions", "n_first", "n_fixed", "n_spatial", "n_temporal",
             "list_entries", "meta_bytes", "data_bytes", "bytes", "phase2_inserts", "phase3_inserts"]


def run_parity(oracle_mod, bufs, C, check_record=True, check_digests=True, check_restore=True, mode=0,
               variant=None):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    o = oracle_mod.Oracle(C, mode=mode)
    ck = Checkpointer(C, mode)
    if variant is not None:   # (flags, switch_permille): Tree-method variants, NEXT #4
        o.set_variant(*variant)
        ck.set_variant(*variant)
    B = bufs[0].size
    devs = []
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        t = _dev(b)
        devs.append(t)
        d = ck.checkpoint(t, nbytes=B)
        torch.cuda.synchronize()
        st = o.stats(k)
        for key in STAT_KEYS:
            assert d[key] == st[key], (k, key, d[key], st[key])
        assert d["record_size"] == o.record_size()
        g = ck.diff_to_host(k)
        w = o.diff(k)
        if g != w:
            pg, pw = oracle_mod.parse_diff(g), oracle_mod.parse_diff(w)
            assert pg.get("changed") == pw.get("changed"), k
            assert pg["first"] == pw["first"], k
            assert pg["shift"] == pw["shift"], k
            assert g[:64] == w[:64], k
            assert pg["data"] == pw["data"], k
            assert False, "diff bytes differ"
        if check_digests:
            n = o.n_leaves
            dd = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
            ck.leaf_digests(dd)
            assert np.array_equal(dd.cpu().numpy().reshape(n, 16), o.leaf_digests()), k
        if check_record:
            assert np.array_equal(ck.record_array(), o.record_array()), k
    if check_restore:
        out = torch.empty(max(B, 1), dtype=torch.uint8, device="cuda")
        for k, b in enumerate(bufs):
            ck.restore(k, out)
            assert torch.equal(out[:B], devs[k][:B]), k
    ck.close()
    return o


def test_fig2_on_gpu(oracle_mod):
    C = 32
    rng = np.random.default_rng(2)
    A = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(8)]
    I, J, K, L = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(4)]
    b0 = np.concatenate(A)
    b1 = np.concatenate([I, J, K, L, A[4], A[0], I, J])
    o = run_parity(oracle_mod, [b0, b1], C)
    d = oracle_mod.parse_diff(o.diff(1))
    assert d["first"] == [1] and d["shift"] == [(12, 7, 0), (6, 3, 1)]


def test_config1_full_lineage(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(1, 1 << 20, 128, 10))
    run_parity(oracle_mod, bufs, 128)


@pytest.mark.parametrize("C", [32, 64, 128, 256])
def test_config2_small(oracle_mod, C):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, (1 << 22) + 100, C, 5, p=0.05))
    run_parity(oracle_mod, bufs, C)


def test_config4_dup_heavy(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(4, 1 << 20, 128, 8))
    run_parity(oracle_mod, bufs, 128)


@pytest.mark.parametrize("seed", range(24))
def test_random_dup_lineages_odd_sizes(oracle_mod, seed):
    rng = np.random.default_rng(9000 + seed)
    C = int(rng.choice([32, 48, 64, 96, 128, 144, 256, 512, 4096]))
    n = int(rng.choice([1, 2, 3, 7, 255, 256, 257, 1000, 1023, 1025, 3000, 5000]))
    tail = int(rng.integers(0, C)) if rng.random() < 0.5 else 0
    nbytes = max(1, n * C - tail)
    bufs = dup_lineage(seed, nbytes, C, K=int(rng.integers(1, 5)), alphabet=int(rng.integers(2, 12)))
    run_parity(oracle_mod, bufs, C)


@pytest.mark.parametrize("C", [144, 160, 192, 240, 272, 400, 1040, 2064])
def test_partial_segment_chunk_sizes(oracle_mod, C):
    """C > 128 and not a multiple of 128 (K1 MODE3D 2: a 2-D map of C-byte rows read in 128-B
    boxes, the last one zero-filled past C and hashed over C mod 128 bytes only): many
    256-chunk tiles through the TMA pipeline, a ragged tail tile and a short last chunk."""
    rng = np.random.default_rng(C)
    n = 256 * (37 if C < 1024 else 9) + 101
    nbytes = n * C - int(rng.integers(1, C))
    bufs = dup_lineage(C, nbytes, C, K=4, alphabet=6)
    run_parity(oracle_mod, bufs, C)


@pytest.mark.parametrize("C", [160, 400])
def test_partial_segment_config2(oracle_mod, C):
    """The config-2 recipe (GDV-like, p = 1 %) at 32 MiB with a partial-segment chunk size."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, 1 << 25, C, 4))
    run_parity(oracle_mod, bufs, C)


def test_all_zero_and_unchanged(oracle_mod):
    C = 64
    z = np.zeros(1000 * C, dtype=np.uint8)
    o = run_parity(oracle_mod, [z, z.copy(), z.copy()], C)
    assert len(o.diff(1)) == 64


@pytest.mark.parametrize("C,nbytes", [(32, (1 << 26) + 100), (128, (1 << 27) + 48), (64, 1 << 27)])
def test_multi_stage_tree(oracle_mod, C, nbytes):
    """n > 2^20 leaves: three tree stages (tile, two upper), ragged tail, odd n."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(1, nbytes, C, 3, p=0.002))
    # add an aligned 2^12-chunk block copy so an upper-stage SHIFT region appears
    b2 = bufs[2].copy()
    blk = (1 << 12) * C
    b2[3 * blk:4 * blk] = bufs[0][blk:2 * blk]
    bufs.append(b2)
    run_parity(oracle_mod, bufs, C)


def test_fully_unique_checkpoint0_large(oracle_mod):
    """Whole buffer one FIRST region (root): exercises upper-stage emission + the data pass."""
    rng = np.random.default_rng(5)
    C = 128
    b = rng.integers(0, 256, (1 << 24) + 16, dtype=np.uint8)
    run_parity(oracle_mod, [b, b.copy()], C)


def test_determinism_two_runs():
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(4, 1 << 20, 128, 4))
    outs = []
    for _ in range(2):
        ck = Checkpointer(128)
        for b in bufs:
            ck.checkpoint(_dev(b), nbytes=b.size)
        outs.append([ck.diff_to_host(k) for k in range(len(bufs))])
        ck.close()
    assert outs[0] == outs[1]


@pytest.mark.parametrize("dbg", [256])
def test_alternate_engine_modes(oracle_mod, monkeypatch, dbg):
    """Engine variants selected by CKPT_DBG at ckpt_create must stay bit-exact:
    256 = record table sized to half the leaves (long probe chains, frequent growth)."""
    monkeypatch.setenv("CKPT_DBG", str(dbg))
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, (1 << 23) + 48, 128, 5, p=0.05))
    run_parity(oracle_mod, bufs, 128)
    bufs = dup_lineage(77, 5000 * 64 - 7, 64, K=4, alphabet=5)
    run_parity(oracle_mod, bufs, 64)


@pytest.mark.parametrize("nbytes", [1, 15, 16, 17, 31, 33, 47, 100])
@pytest.mark.parametrize("variant", [None, (3, 500)])
def test_tiny_buffers(oracle_mod, nbytes, variant):
    """Buffers below one chunk up to a few chunks, with partial last 16-byte units: diffs,
    digests, record and the chunk-major restore's partial-unit path (R4)."""
    rng = np.random.default_rng(nbytes)
    C = 32
    base = rng.integers(0, 256, nbytes, dtype=np.uint8)
    bufs = [base.copy()]
    for k in range(1, 5):
        b = bufs[-1].copy()
        if k % 2:
            b[int(rng.integers(0, nbytes))] ^= 0x5A
        bufs.append(b)
    run_parity(oracle_mod, bufs, C, variant=variant)
