"""Boundary contract on the GPU (include/ckpt.h):

- ckpt_checkpoint synchronises the host exactly once per call, also when the call grows the
  record table (stream-ordered growth, ckpt_host_syncs), and stays bit-exact with the oracle;
- ckpt_import validates the body of a diff on the host before any kernel reads it: corrupt
  node ids, source checkpoints, region sizes or Basic bitmaps are rejected with CKPT_EINVAL
  and leave the handle usable and unchanged;
- restores are ordered after the caller's earlier work: on torch's current stream
  (ckpt_restore_stream) and, for ckpt_restore, on the legacy default stream.
"""
import struct

import numpy as np
import pytest

from tests._lineages import dup_lineage

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def test_one_sync_per_checkpoint_including_growth(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    C, n = 128, 1 << 14
    rng = np.random.default_rng(7)
    bufs = [rng.integers(0, 256, n * C, dtype=np.uint8)]          # fully unique: record = 2n - 1
    for k in range(1, 5):
        b = bufs[-1].copy()
        sel = rng.random(n) < 0.6                                   # most chunks new each time
        b.reshape(n, C)[sel] = rng.integers(0, 256, (int(sel.sum()), C), dtype=np.uint8)
        bufs.append(b)
    o = oracle_mod.Oracle(C)
    ck = Checkpointer(C)
    caps = []
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        t = torch.from_numpy(b).cuda()
        torch.cuda.synchronize()
        s0 = ck.host_syncs
        d = ck.checkpoint(t)
        assert ck.host_syncs - s0 == 1, (k, ck.host_syncs - s0)
        caps.append(d["record_capacity"])
        assert d["record_size"] == o.record_size()
        assert ck.diff_to_host(k) == o.diff(k), k
    assert len(set(caps)) >= 2, caps                                 # the table grew inside a call
    assert np.array_equal(ck.record_array(), o.record_array())
    out = torch.empty(n * C, dtype=torch.uint8, device="cuda")
    ck.restore(len(bufs) - 1, out)
    assert np.array_equal(out.cpu().numpy(), bufs[-1])
    ck.close()


def _lineage_with_shifts(C=64):
    bufs = dup_lineage(3, 2000 * C - 7, C, K=3)
    return bufs


def _take(C, bufs, mode=0):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    a = Checkpointer(C, mode)
    for b in bufs:
        a.checkpoint(torch.from_numpy(np.ascontiguousarray(b)).cuda(), nbytes=b.size)
    out = [a.diff_to_host(k) for k in range(len(bufs))]
    a.close()
    return out


def _rejects(C, good_prefix, bad, mode=0):
    """Importing `bad` after `good_prefix` fails with EINVAL, and the handle still takes the
    next good diff."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, ckpt
    b = Checkpointer(C, mode)
    for d in good_prefix:
        b.import_diff(d)
    with pytest.raises(ckpt.CkptError) as e:
        b.import_diff(bytes(bad))
    assert e.value.status == ckpt.CKPT_EINVAL
    assert b.num_checkpoints == len(good_prefix)
    return b


def test_import_rejects_corrupt_tree_bodies(oracle_mod):
    C = 64
    bufs = _lineage_with_shifts(C)
    diffs = _take(C, bufs)
    k = next(i for i in range(1, len(diffs)) if len(oracle_mod.parse_diff(diffs[i])["shift"]) > 0)
    d = diffs[k]
    p = oracle_mod.parse_diff(d)
    nF, nS = len(p["first"]), len(p["shift"])
    n = p["n_leaves"]
    assert nF > 0 and nS > 0
    cases = []
    bad = bytearray(d); struct.pack_into("<I", bad, 64, 0xFFFFFFFF); cases.append(bad)        # FIRST node id
    bad = bytearray(d); struct.pack_into("<I", bad, 64, 2 * n - 1); cases.append(bad)         # one past the last node
    s0 = 64 + 4 * nF
    bad = bytearray(d); struct.pack_into("<I", bad, s0 + 8, k + 5); cases.append(bad)         # source checkpoint > id
    bad = bytearray(d); struct.pack_into("<I", bad, s0 + 4, 0xFFFFFFF0); cases.append(bad)     # source node id
    bad = bytearray(d); struct.pack_into("<I", bad, s0, 0); cases.append(bad)                  # SHIFT region = root: size
    node0 = struct.unpack_from("<I", d, 64)[0]
    if node0 > 0:
        bad = bytearray(d); struct.pack_into("<I", bad, 64, (node0 - 1) // 2); cases.append(bad)   # FIRST -> its parent
    for bad in cases:
        b = _rejects(C, diffs[:k], bad)
        b.import_diff(d)                                  # unchanged and not poisoned
        assert b.num_checkpoints == k + 1
        b.close()


def test_import_rejects_corrupt_basic_bitmap(oracle_mod):
    C = 64
    bufs = _lineage_with_shifts(C)
    diffs = _take(C, bufs, mode=2)
    d = diffs[1]
    p = oracle_mod.parse_diff(d)
    n = p["n_leaves"]
    words = (n + 31) // 32
    cases = []
    if n % 32:
        bad = bytearray(d)
        w = struct.unpack_from("<I", bad, 64 + 4 * (words - 1))[0] | (1 << 31)   # a bit past n
        struct.pack_into("<I", bad, 64 + 4 * (words - 1), w)
        cases.append(bad)
    bad = bytearray(d)
    for c in range(n):                                   # one more changed chunk than nF
        w = struct.unpack_from("<I", bad, 64 + 4 * (c // 32))[0]
        if not (w >> (c % 32)) & 1:
            struct.pack_into("<I", bad, 64 + 4 * (c // 32), w | (1 << (c % 32)))
            break
    cases.append(bad)
    for bad in cases:
        b = _rejects(C, diffs[:1], bad, mode=2)
        b.import_diff(d)
        b.close()


def test_restore_ordered_after_caller_stream_work():
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import ckpt
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B = 1 << 24
    bufs = list(W.lineage(2, B, 128, 3, p=0.05))
    ck = Checkpointer(128)
    devs = [torch.from_numpy(b).cuda() for b in bufs]
    for t in devs:
        ck.checkpoint(t)
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    side = torch.cuda.Stream()
    for k in range(3):
        # a delayed overwrite on the caller's (non-blocking) stream, then the restore on it:
        # the restore must land after the fill
        with torch.cuda.stream(side):
            torch.cuda._sleep(20_000_000)
            out.fill_(0xA5)
            ck.restore(k, out)
        side.synchronize()
        assert torch.equal(out, devs[k]), k
        # ckpt_restore (internal blocking stream) after work on the legacy default stream
        torch.cuda._sleep(20_000_000)
        out.fill_(0x5A)
        rc = ckpt.lib().ckpt_restore(ck._h, k, out.data_ptr())
        assert rc == 0
        assert torch.equal(out, devs[k]), k
    ck.close()


def test_calls_ordered_across_streams_after_early_return(oracle_mod):
    """ckpt_checkpoint returns once the statistics are final while its last kernel may still
    write the diff: consecutive checkpoints on different streams, the D2H copies and a restore
    issued right after each call must still see complete diffs (the library orders them after
    the call's completion event)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B, C = (1 << 22) + 48, 128
    bufs = list(W.lineage(2, B, C, 6, p=0.05))
    devs = [torch.from_numpy(b).cuda() for b in bufs]
    torch.cuda.synchronize()
    o = oracle_mod.Oracle(C)
    ck = Checkpointer(C)
    streams = [torch.cuda.Stream() for _ in range(3)]
    pinned = torch.empty(B + 64 + 12 * ((B + C - 1) // C) + 16, dtype=torch.uint8).pin_memory()
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k, t in enumerate(devs):
        o.checkpoint(bufs[k])
        s = streams[k % 3]
        d = ck.checkpoint(t, stream=s)
        side = streams[(k + 1) % 3]
        ck.diff_to_host_async(k, pinned, side, nbytes=d["bytes"])   # another stream, right away
        side.synchronize()
        assert bytes(pinned[: d["bytes"]].numpy()) == o.diff(k), k
        assert ck.diff_to_host(k) == o.diff(k), k
    for k in range(len(devs)):
        ck.restore(k, out)
        assert torch.equal(out, devs[k]), k
    ck.close()


def test_calls_from_another_host_thread():
    """Any host thread may drive a handle (the library binds the handle's device per call): a
    checkpoint and a restore issued from a fresh thread match the same lineage run inline."""
    import threading
    import numpy as np
    import torch
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    C = 128
    bufs = [torch.from_numpy(b).cuda() for b in W.lineage(2, 1 << 22, C, 3)]
    a, b = Checkpointer(C), Checkpointer(C)
    for x in bufs:
        a.checkpoint(x)
    out, err = {}, []

    def work():
        try:
            st = torch.cuda.Stream()
            for x in bufs:
                b.checkpoint(x, stream=st)
            r = torch.empty_like(bufs[-1])
            b.restore(2, r)
            torch.cuda.synchronize()
            out["r"] = r.cpu().numpy()
        except Exception as e:   # surfaced in the main thread
            err.append(e)
    t = threading.Thread(target=work)
    t.start()
    t.join()
    assert not err, err
    for k in range(3):
        assert a.diff_to_host(k) == b.diff_to_host(k), k
    assert np.array_equal(out["r"], bufs[-1].cpu().numpy())
