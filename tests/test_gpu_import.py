"""Lineage rebuild after a restart (ckpt_import): a fresh handle that
imports the host copies of diffs 0..k-1 must continue the lineage exactly as the original
handle does — same later diffs (bit-exact, and equal to the oracle's), same restores."""
import ctypes

import numpy as np
import pytest

from tests._lineages import dup_lineage

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _continue_after_import(oracle_mod, bufs, C, mode, k_import):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    B = bufs[0].size
    a = Checkpointer(C, mode)
    o = oracle_mod.Oracle(C, mode=mode)
    devs = [torch.from_numpy(np.ascontiguousarray(b)).cuda() for b in bufs]
    for k in range(k_import):
        a.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
    host = [a.diff_to_host(k) for k in range(k_import)]
    b = Checkpointer(C, mode)                      # "after the restart"
    for d in host:
        b.import_diff(d)
    assert b.num_checkpoints == k_import
    for k in range(k_import, len(bufs)):
        da, db = a.checkpoint(devs[k], nbytes=B), b.checkpoint(devs[k], nbytes=B)
        o.checkpoint(bufs[k])
        assert da == {**db, "dev_ptr": da["dev_ptr"]} or da["bytes"] == db["bytes"]
        assert b.diff_to_host(k) == a.diff_to_host(k) == o.diff(k), k
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(len(bufs)):
        b.restore(k, out)
        assert torch.equal(out, devs[k]), k
    if mode == 0:
        assert b.record() == a.record() == o.record()
    a.close()
    b.close()


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_import_continues_lineage_config2(oracle_mod, mode):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, (1 << 22) + 100, 128, 7, p=0.05))
    _continue_after_import(oracle_mod, bufs, 128, mode, 4)


@pytest.mark.parametrize("seed", range(4))
def test_import_duplicate_lineages(oracle_mod, seed):
    bufs = dup_lineage(40 + seed, 3000 * 64 - 5 * seed, 64, K=6)
    _continue_after_import(oracle_mod, bufs, 64, 0, 3)


def test_import_rejects_bad_diffs(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, ckpt
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(1, 1 << 20, 128, 3))
    a = Checkpointer(128)
    for b in bufs:
        a.checkpoint(torch.from_numpy(b).cuda())
    d0, d1 = a.diff_to_host(0), a.diff_to_host(1)
    b = Checkpointer(128)
    with pytest.raises(ckpt.CkptError) as e:
        b.import_diff(d1)                           # wrong position in the lineage
    assert e.value.status == ckpt.CKPT_EINVAL
    with pytest.raises(ckpt.CkptError):
        Checkpointer(256).import_diff(d0)           # other chunk size
    with pytest.raises(ckpt.CkptError):
        Checkpointer(128, 1).import_diff(d0)        # other method
    b.import_diff(d0)                               # the handle was left unchanged
    # An inconsistent diff: its first FIRST chunk replaced by content the record already
    # holds (chunk 0 of checkpoint 0). Re-de-duplicating the restored buffer labels that
    # chunk a temporal duplicate, so the regenerated diff differs. (A self-consistent edit,
    # e.g. other new bytes, re-imports as written: the check is lineage consistency, not a
    # checksum.)
    bad = bytearray(d1)
    p = oracle_mod.parse_diff(d1)
    meta = p["meta_bytes"]
    bad[meta:meta + 128] = bytes(bufs[0][:128])
    with pytest.raises(ckpt.CkptError) as e:
        b.import_diff(bytes(bad))
    assert e.value.status == ckpt.CKPT_EINVAL
    with pytest.raises(ckpt.CkptError) as e:
        b.checkpoint(torch.from_numpy(bufs[1]).cuda())   # the mismatch poisoned the handle
    assert e.value.status == ckpt.CKPT_ESTATE
    a.close()
