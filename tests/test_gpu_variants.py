"""GPU <-> oracle parity of the Tree-method variants (readings R22,
R23): full first checkpoint and the full-change switch. Bit-exact
diffs, statistics, leaf digests, record sets and restores through the C ABI, plus a lineage
rebuilt with ckpt_import across full differences."""
import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_gpu_parity import run_parity
from tests.test_oracle_variants import changed_count

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

FULL_FIRST, FULL_SWITCH = 1, 2


def _mostly_rewritten(bufs, ks, seed):
    """Rewrite every chunk of checkpoints ks (so the switch fires at any threshold)."""
    rng = np.random.default_rng(seed)
    out = [bufs[0].copy()]
    for k in range(1, len(bufs)):
        b = bufs[k].copy()
        if k in ks:
            b = rng.integers(0, 256, b.size, dtype=np.uint8)
        out.append(b)
    return out


def test_fig2_full_first_on_gpu(oracle_mod):
    C = 32
    rng = np.random.default_rng(2)
    A = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(8)]
    I, J, K, L = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(4)]
    b0 = np.concatenate(A)
    b1 = np.concatenate([I, J, K, L, A[4], A[0], I, J])
    o = run_parity(oracle_mod, [b0, b1], C, variant=(FULL_FIRST, 1000))
    assert oracle_mod.parse_diff(o.diff(0))["flags"] == 3
    d = oracle_mod.parse_diff(o.diff(1))
    assert d["first"] == [1] and d["shift"] == [(12, 7, 0), (6, 3, 1)]


@pytest.mark.parametrize("flags", [FULL_FIRST, FULL_SWITCH, FULL_FIRST | FULL_SWITCH])
def test_config1_lineage_variants(oracle_mod, flags):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = _mostly_rewritten(list(W.lineage(1, 1 << 20, 128, 8)), {3, 4}, 5)
    o = run_parity(oracle_mod, bufs, 128, variant=(flags, 900))
    n = o.n_leaves
    for k in range(len(bufs)):
        # 3 and 4 are rewritten, and 5 (the original lineage again) differs from 4 everywhere
        switched = k >= 1 and 1000 * changed_count(bufs, k, 128) >= 900 * n
        assert switched == (k in (3, 4, 5))
        full = (k == 0 and flags & FULL_FIRST) or (switched and flags & FULL_SWITCH)
        assert (oracle_mod.parse_diff(o.diff(k))["flags"] == 3) == bool(full), k


@pytest.mark.parametrize("permille", [0, 10, 30, 60, 1000])
@pytest.mark.parametrize("C", [32, 128])
def test_config2_switch_thresholds(oracle_mod, permille, C):
    """Config-2 updates at p = 5 %: thresholds around the changed fraction switch some
    checkpoints and not others; permille = 0 stores every checkpoint k >= 1 in full."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, (1 << 22) + 100, C, 5, p=0.05))
    run_parity(oracle_mod, bufs, C, variant=(FULL_SWITCH, permille))


@pytest.mark.parametrize("seed", range(8))
def test_random_duplicate_lineages_variants(oracle_mod, seed):
    rng = np.random.default_rng(700 + seed)
    C = int(rng.choice([32, 48, 96, 128, 4096]))
    n = int(rng.choice([1, 2, 3, 7, 255, 1000, 3000]))
    nbytes = max(1, n * C - int(rng.integers(0, C)))
    bufs = dup_lineage(seed, nbytes, C, K=5, p_change=float(rng.choice([0.3, 0.8, 0.97])))
    flags = int(rng.choice([FULL_FIRST, FULL_SWITCH, FULL_FIRST | FULL_SWITCH]))
    permille = int(rng.choice([0, 200, 500, 900, 1000]))
    run_parity(oracle_mod, bufs, C, variant=(flags, permille))


def test_config4_variants(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(4, 1 << 20, 128, 6))
    run_parity(oracle_mod, bufs, 128, variant=(FULL_FIRST | FULL_SWITCH, 850))


def test_import_across_full_diffs(oracle_mod):
    """A restarted handle with the same variant rebuilds the lineage from host copies that
    include full differences, and continues it bit-exactly."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    C = 128
    bufs = _mostly_rewritten(list(W.lineage(2, (1 << 21) + 48, C, 7, p=0.05)), {2}, 9)
    var = (FULL_FIRST | FULL_SWITCH, 800)
    B = bufs[0].size
    a = Checkpointer(C)
    a.set_variant(*var)
    o = oracle_mod.Oracle(C)
    o.set_variant(*var)
    devs = [torch.from_numpy(np.ascontiguousarray(b)).cuda() for b in bufs]
    for k in range(4):
        a.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
    host = [a.diff_to_host(k) for k in range(4)]
    assert oracle_mod.parse_diff(host[0])["flags"] == 3 and oracle_mod.parse_diff(host[2])["flags"] == 3
    b = Checkpointer(C)
    b.set_variant(*var)
    for d in host:
        b.import_diff(d)
    for k in range(4, len(bufs)):
        a.checkpoint(devs[k], nbytes=B)
        b.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
        assert b.diff_to_host(k) == a.diff_to_host(k) == o.diff(k), k
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(len(bufs)):
        b.restore(k, out)
        assert torch.equal(out, devs[k]), k
    assert b.record() == o.record()
    # a handle without the variant rejects the full difference and stays usable
    from paper_conf_icpp_tanlmtmbctn23_b200 import CkptError
    c = Checkpointer(C)
    with pytest.raises(CkptError):
        c.import_diff(host[0])
    c.checkpoint(devs[0], nbytes=B)
    for h in (a, b, c):
        h.close()


def test_set_variant_rejections():
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, CkptError
    with pytest.raises(CkptError):
        Checkpointer(128, 1).set_variant(FULL_FIRST)          # List mode
    ck = Checkpointer(128)
    with pytest.raises(CkptError):
        ck.set_variant(FULL_SWITCH, 1001)
    with pytest.raises(CkptError):
        ck.set_variant(8)
    ck.checkpoint(torch.zeros(4096, dtype=torch.uint8, device="cuda"))
    with pytest.raises(CkptError):
        ck.set_variant(FULL_FIRST)                             # after the first checkpoint
    ck.close()
