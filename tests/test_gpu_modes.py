"""GPU <-> oracle parity of the List and Basic methods:
bit-exact diffs, statistics, leaf digests, record sets and restores, through the C ABI.
Tree-mode parity lives in test_gpu_parity.py; the same harness is reused with `mode`."""
import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_gpu_parity import run_parity

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

LIST, BASIC = 1, 2


@pytest.mark.parametrize("mode", [LIST, BASIC])
def test_fig2_modes(oracle_mod, mode):
    C = 32
    rng = np.random.default_rng(2)
    A = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(8)]
    I, J, K, L = [rng.integers(0, 256, C, dtype=np.uint8) for _ in range(4)]
    b0 = np.concatenate(A)
    b1 = np.concatenate([I, J, K, L, A[4], A[0], I, J])
    o = run_parity(oracle_mod, [b0, b1], C, mode=mode)
    d = oracle_mod.parse_diff(o.diff(1))
    if mode == LIST:
        assert len(d["first"]) + len(d["shift"]) == 7
    else:
        assert d["changed"] == [0, 1, 2, 3, 5, 6, 7]           # chunk 4 unchanged


@pytest.mark.parametrize("mode", [LIST, BASIC])
def test_config1_lineage_modes(oracle_mod, mode):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(1, 1 << 20, 128, 10))
    run_parity(oracle_mod, bufs, 128, mode=mode)


@pytest.mark.parametrize("mode", [LIST, BASIC])
@pytest.mark.parametrize("C", [32, 64, 128, 256])
def test_config2_modes(oracle_mod, mode, C):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, (1 << 22) + 100, C, 4, p=0.05))
    run_parity(oracle_mod, bufs, C, mode=mode)


@pytest.mark.parametrize("mode", [LIST, BASIC])
@pytest.mark.parametrize("seed", range(10))
def test_random_duplicate_lineages_modes(oracle_mod, mode, seed):
    rng = np.random.default_rng(900 + seed)
    C = int(rng.choice([32, 48, 96, 128, 4096]))
    n = int(rng.choice([1, 2, 3, 7, 255, 1000, 3000]))
    nbytes = max(1, n * C - int(rng.integers(0, C)))
    bufs = dup_lineage(seed, nbytes, C, K=4)
    run_parity(oracle_mod, bufs, C, mode=mode)


@pytest.mark.parametrize("mode", [LIST, BASIC])
def test_config4_and_multistage_modes(oracle_mod, mode):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(4, 1 << 20, 128, 6))
    run_parity(oracle_mod, bufs, 128, mode=mode)
    # more than one tree stage (n > 2^20 leaves at C = 32) and a ragged tail
    bufs = list(W.lineage(2, (1 << 25) + 40, 32, 3, p=0.01))
    run_parity(oracle_mod, bufs, 32, check_record=False, mode=mode)


def test_modes_rejected_and_tree_equivalence(oracle_mod):
    import ctypes
    from paper_conf_icpp_tanlmtmbctn23_b200 import ckpt
    h = ctypes.c_void_p()
    assert ckpt.lib().ckpt_create_mode(128, 3, ctypes.byref(h)) == ckpt.CKPT_EINVAL
    # Tree, List and Basic handles on the same lineage: same leaf digests, List/Tree data
    # sections equal, Basic changed count = non-FIXED leaves
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, 1 << 22, 128, 4, p=0.02))
    cks = [Checkpointer(128, m) for m in (0, 1, 2)]
    for k, b in enumerate(bufs):
        t = torch.from_numpy(b).cuda()
        ds = [c.checkpoint(t) for c in cks]
        assert ds[2]["n_first"] == ds[0]["n_first"] + ds[0]["n_spatial"] + ds[0]["n_temporal"]
        assert ds[1]["list_entries"] == ds[0]["list_entries"]
        assert ds[0]["data_bytes"] == ds[1]["data_bytes"]
    for c in cks:
        c.close()
