"""GPU <-> oracle parity of the SHIFT-SHIFT-insert variant (
readings R24, R25; pinned in tests/test_oracle_shift_insert.py): bit-exact differences,
statistics (incl. the inserted shifted regions), leaf digests, record sets and restores
through the C ABI — restores whose sources are nodes with no first-occurrence data are
resolved chunk by chunk (R25) — plus a lineage rebuilt with ckpt_import."""
import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_gpu_parity import run_parity

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

SHIFT_INSERT, FULL_FIRST = 4, 1


@pytest.mark.parametrize("nchunks", [1, 2, 8, 1024, 1000, 4096 + 7])
def test_all_zero_buffers(oracle_mod, nchunks):
    """The zero-heavy first checkpoint the variant exists for: 2 log2(n) regions at n = 2^h
    (closed form pinned on the oracle), ragged n too; a later checkpoint with a shifted
    zero block references the nodes that found their own entries."""
    C = 64
    b0 = np.zeros(nchunks * C, dtype=np.uint8)
    b1 = b0.copy()
    b1[: min(len(b1), 3 * C)] = 7
    o = run_parity(oracle_mod, [b0, b1, b0.copy()], C, variant=(SHIFT_INSERT, 1000))
    if nchunks in (8, 1024):
        d = oracle_mod.parse_diff(o.diff(0))
        assert len(d["first"]) + len(d["shift"]) == 2 * int(np.log2(nchunks))


@pytest.mark.parametrize("seed", range(16))
def test_random_duplicate_lineages(oracle_mod, seed):
    rng = np.random.default_rng(1700 + seed)
    C = int(rng.choice([32, 48, 64, 128]))
    n = int(rng.choice([7, 64, 255, 256, 1000, 3000]))
    nbytes = n * C - int(rng.integers(0, C)) * int(rng.integers(0, 2))
    bufs = dup_lineage(1800 + seed, nbytes, C, K=int(rng.integers(2, 7)), alphabet=int(rng.integers(1, 5)),
                       p_change=float(rng.choice([0.2, 0.6, 0.95])))
    flags = SHIFT_INSERT | (FULL_FIRST if seed % 5 == 4 else 0)
    run_parity(oracle_mod, bufs, C, variant=(flags, 1000))


@pytest.mark.parametrize("cfg", [2, 4])
def test_configs(oracle_mod, cfg):
    """Config 2 (GDV-like, 4 MiB + 100 B: half the row blocks all-zero at checkpoint 0) and
    config 4 (duplicate-heavy, 1 MiB)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B = (1 << 22) + 100 if cfg == 2 else 1 << 20
    bufs = list(W.lineage(cfg, B, 128, 5, p=0.05))
    o = run_parity(oracle_mod, bufs, 128, variant=(SHIFT_INSERT, 1000))
    assert o.stats(0)["phase3_inserts"] > 0


def test_multi_stage_zero_heavy(oracle_mod):
    """n > 2^20 (three tree stages): zero blocks larger than a tile climb through the upper
    stages as potential shifted nodes."""
    C = 32
    n = (1 << 21) + 5
    rng = np.random.default_rng(3)
    b0 = np.zeros(n * C, dtype=np.uint8)
    b0[: 4096 * C] = rng.integers(0, 256, 4096 * C, dtype=np.uint8)
    b1 = b0.copy()
    b1[(1 << 20) * C:(1 << 20) * C + 64 * C] = 9
    run_parity(oracle_mod, [b0, b1], C, variant=(SHIFT_INSERT, 1000), check_record=True)


def test_import_continues_lineage(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    C = 64
    bufs = dup_lineage(77, 3000 * C - 9, C, K=6, alphabet=2, p_change=0.6)
    B = bufs[0].size
    var = (SHIFT_INSERT, 1000)
    a = Checkpointer(C)
    a.set_variant(*var)
    o = oracle_mod.Oracle(C)
    o.set_variant(*var)
    devs = [torch.from_numpy(np.ascontiguousarray(b)).cuda() for b in bufs]
    for k in range(3):
        a.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
    host = [a.diff_to_host(k) for k in range(3)]
    assert all(oracle_mod.parse_diff(h)["flags"] == 4 for h in host)
    b = Checkpointer(C)
    b.set_variant(*var)
    for d in host:
        b.import_diff(d)
    for k in range(3, len(bufs)):
        a.checkpoint(devs[k], nbytes=B)
        b.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
        assert b.diff_to_host(k) == a.diff_to_host(k) == o.diff(k), k
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(len(bufs)):
        b.restore(k, out)
        assert torch.equal(out, devs[k]), k
    assert b.record() == o.record()
    for h in (a, b):
        h.close()
