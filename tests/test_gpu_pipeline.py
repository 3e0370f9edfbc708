"""Pipelined checkpoints (include/ckpt.h ckpt_checkpoint_submit / ckpt_checkpoint_wait):
checkpoint k + 1's leaf pass runs while checkpoint k's record and tree phases do. The method
is unchanged, so every diff, statistic, record set, leaf digest and restore must equal the
CPU oracle's (bit-exact), exactly as for ckpt_checkpoint (pipelining).

The lineages keep every buffer alive (a submitted buffer is borrowed until its wait), and
re-change the same chunks in consecutive checkpoints, so a leaf pass that overwrote digests
the previous call's tree phases still read would show up as a wrong diff.
"""
import numpy as np
import pytest

from tests._lineages import dup_lineage
from tests.test_gpu_parity import STAT_KEYS

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _dev(b):
    t = torch.empty(max(b.size, 1), dtype=torch.uint8, device="cuda")
    t[: b.size].copy_(torch.from_numpy(np.ascontiguousarray(b)))
    return t


def pipelined(ck, devs, B, stream=None, depth=2, sync_every=0):
    """Submit every buffer, collecting call k - depth + 1 after submitting call k (depth 2: the
    bench's order); sync_every > 0 takes every sync_every-th checkpoint synchronously."""
    out = [None] * len(devs)
    pend = []
    for k, t in enumerate(devs):
        if sync_every and k % sync_every == sync_every - 1:
            for j in pend:
                out[j] = ck.wait(j, stream=stream)
            pend = []
            out[k] = ck.checkpoint(t, nbytes=B, stream=stream)
            continue
        cid = ck.submit(t, nbytes=B, stream=stream)
        assert cid == k
        pend.append(cid)
        while len(pend) >= depth:
            j = pend.pop(0)
            out[j] = ck.wait(j, stream=stream)
    for j in pend:
        out[j] = ck.wait(j, stream=stream)
    return out


def run_pipe_parity(oracle_mod, bufs, C, mode=0, variant=None, check_record=True, **kw):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    o = oracle_mod.Oracle(C, mode=mode)
    ck = Checkpointer(C, mode)
    if variant is not None:
        o.set_variant(*variant)
        ck.set_variant(*variant)
    B = bufs[0].size
    devs = [_dev(b) for b in bufs]
    torch.cuda.synchronize()
    ds = pipelined(ck, devs, B, **kw)
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        st = o.stats(k)
        for key in STAT_KEYS:
            assert ds[k][key] == st[key], (k, key, ds[k][key], st[key])
        assert ck.diff_to_host(k) == o.diff(k), k
    assert ds[-1]["record_size"] == o.record_size()
    n = o.n_leaves
    dd = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
    ck.leaf_digests(dd)
    assert np.array_equal(dd.cpu().numpy().reshape(n, 16), o.leaf_digests())
    if check_record and mode == 0:
        assert np.array_equal(ck.record_array(), o.record_array())
    out = torch.empty(max(B, 1), dtype=torch.uint8, device="cuda")
    for k in range(len(bufs)):
        ck.restore(k, out)
        assert torch.equal(out[:B], devs[k][:B]), k
    ck.close()
    return o


def test_config1_pipelined(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    run_pipe_parity(oracle_mod, list(W.lineage(1, 1 << 20, 128, 10)), 128)


@pytest.mark.parametrize("C", [32, 64, 128, 160, 256])
def test_config2_pipelined(oracle_mod, C):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    run_pipe_parity(oracle_mod, list(W.lineage(2, (1 << 22) + 100, C, 6, p=0.05)), C)


def test_config4_pipelined(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    run_pipe_parity(oracle_mod, list(W.lineage(4, 1 << 20, 128, 10)), 128)


@pytest.mark.parametrize("seed", range(16))
def test_dup_lineages_pipelined(oracle_mod, seed):
    """Duplicate-heavy lineages with most chunks rewritten every checkpoint (the same chunks
    are candidates in consecutive calls), odd sizes, one to five chunk sizes of tiles."""
    rng = np.random.default_rng(4000 + seed)
    C = int(rng.choice([32, 48, 64, 128, 144, 256, 4096]))
    n = int(rng.choice([1, 3, 255, 257, 1025, 3000, 9000]))
    nbytes = max(1, n * C - (int(rng.integers(0, C)) if rng.random() < 0.5 else 0))
    bufs = dup_lineage(seed, nbytes, C, K=int(rng.integers(3, 8)), alphabet=int(rng.integers(2, 8)),
                       p_change=float(rng.choice([0.3, 0.9])))
    run_pipe_parity(oracle_mod, bufs, C)


@pytest.mark.parametrize("mode", [1, 2])
def test_list_and_basic_pipelined(oracle_mod, mode):
    bufs = dup_lineage(77, 3000 * 64 + 17, 64, K=6, alphabet=5, p_change=0.6)
    run_pipe_parity(oracle_mod, bufs, 64, mode=mode)


@pytest.mark.parametrize("variant", [(1, 1000), (2, 250), (4, 1000), (5, 1000)])
def test_variants_pipelined(oracle_mod, variant):
    bufs = dup_lineage(91, 5000 * 64, 64, K=6, alphabet=4, p_change=0.9)
    run_pipe_parity(oracle_mod, bufs, 64, variant=variant)


def test_multi_stage_pipelined(oracle_mod):
    """n > 2^20 leaves (three tree stages), an upper-stage SHIFT region, pipelined."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    C, nbytes = 32, (1 << 26) + 100
    bufs = list(W.lineage(1, nbytes, C, 3, p=0.002))
    b2 = bufs[2].copy()
    blk = (1 << 12) * C
    b2[3 * blk:4 * blk] = bufs[0][blk:2 * blk]
    bufs.append(b2)
    run_pipe_parity(oracle_mod, bufs, C)


def test_mixed_sync_and_pipelined(oracle_mod):
    """Every third checkpoint synchronous, the others pipelined, on the caller's stream."""
    bufs = dup_lineage(5, 4000 * 128, 128, K=9, alphabet=6, p_change=0.7)
    run_pipe_parity(oracle_mod, bufs, 128, stream=torch.cuda.Stream(), sync_every=3)


def test_depth_one_and_other_streams(oracle_mod):
    """Collect each call before the next (no overlap), and submit on a different stream each
    call: the diffs are the oracle's either way."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    bufs = dup_lineage(6, 2000 * 64, 64, K=6, alphabet=6, p_change=0.8)
    o = oracle_mod.Oracle(64)
    for b in bufs:
        o.checkpoint(b)
    ck = Checkpointer(64)
    devs = [_dev(b) for b in bufs]
    torch.cuda.synchronize()
    pipelined(ck, devs, bufs[0].size, depth=1)
    for k in range(len(bufs)):
        assert ck.diff_to_host(k) == o.diff(k), k
    ck.close()
    ck = Checkpointer(64)
    streams = [torch.cuda.Stream() for _ in range(3)]
    ids = []
    for k, t in enumerate(devs):
        ids.append(ck.submit(t, stream=streams[k % 3]))
        if k:
            ck.wait(ids[k - 1], stream=streams[k % 3])
    ck.wait(ids[-1])
    for k in range(len(bufs)):
        assert ck.diff_to_host(k) == o.diff(k), k
    ck.close()


def test_one_host_wait_per_call_and_growth(oracle_mod):
    """Pipelined calls keep the one-wait-per-call contract, also across record-table growth
    (the rehash runs on the chain stream after the in-flight call's inserts)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    C, n = 128, 1 << 14
    rng = np.random.default_rng(8)
    bufs = [rng.integers(0, 256, n * C, dtype=np.uint8)]
    for k in range(1, 6):
        b = bufs[-1].copy()
        sel = rng.random(n) < 0.6
        b.reshape(n, C)[sel] = rng.integers(0, 256, (int(sel.sum()), C), dtype=np.uint8)
        bufs.append(b)
    o = oracle_mod.Oracle(C)
    for b in bufs:
        o.checkpoint(b)
    ck = Checkpointer(C)
    devs = [_dev(b) for b in bufs]
    torch.cuda.synchronize()
    s0 = ck.host_syncs
    ds = pipelined(ck, devs, n * C)
    assert ck.host_syncs - s0 == len(bufs)
    assert len({d["record_capacity"] for d in ds}) >= 2
    for k in range(len(bufs)):
        assert ck.diff_to_host(k) == o.diff(k), k
    assert np.array_equal(ck.record_array(), o.record_array())
    ck.close()


def test_pipelined_equals_synchronous_at_1gib():
    """The benchmarked configuration (config 2, 1 GiB, C = 128): a pipelined lineage gives
    byte-identical diffs and statistics to the synchronous calls (themselves oracle-checked
    at this size in test_gpu_parity.py), and restores the newest checkpoint exactly."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B, C, K = 1 << 30, 128, 6
    st = torch.cuda.Stream()
    seed = W.seed_of(2)
    bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
    with torch.cuda.stream(st):
        W.DeviceGen.initial(2, bufs[0], B, seed, st)
        for k in range(1, K):
            bufs[k].copy_(bufs[k - 1])
            W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, 0.01, st)
    st.synchronize()
    a, b = Checkpointer(C), Checkpointer(C)
    da = [a.checkpoint(x, stream=st) for x in bufs]
    db = pipelined(b, bufs, B, stream=st)
    for k in range(K):
        for key in STAT_KEYS:
            assert da[k][key] == db[k][key], (k, key)
        assert a.diff_to_host(k) == b.diff_to_host(k), k
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    b.restore(K - 1, out)
    assert torch.equal(out, bufs[-1])
    a.close()
    b.close()


def test_pipelined_stress_tiny_lineages(oracle_mod):
    """A 255-chunk lineage (one leaf-tail kernel, microsecond kernels) pipelined 150 times:
    with K1b launched programmatically after the previous call's gather, the next call's
    chain could start early and its gather zero the previous call's counters before that
    call's phase 3 had read them (1 failure in 200 runs before the fix)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    bufs = dup_lineage(13, 255 * 128 - 116, 128, K=5, alphabet=4, p_change=0.9)
    o = oracle_mod.Oracle(128)
    for b in bufs:
        o.checkpoint(b)
    want = [o.stats(k) for k in range(len(bufs))]
    devs = [_dev(b) for b in bufs]
    torch.cuda.synchronize()
    for it in range(150):
        ck = Checkpointer(128)
        ds = pipelined(ck, devs, bufs[0].size)
        for k in range(len(bufs)):
            for key in STAT_KEYS:
                assert ds[k][key] == want[k][key], (it, k, key)
        if it % 50 == 0:
            for k in range(len(bufs)):
                assert ck.diff_to_host(k) == o.diff(k), (it, k)
        ck.close()


def test_pipelined_with_profiling_events(oracle_mod):
    """Profiling level 2 (events between every kernel, on both streams) with pipelined calls:
    per-phase times are reported and the diffs are still the oracle's."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(2, 1 << 22, 128, 5, p=0.05))
    o = oracle_mod.Oracle(128)
    for b in bufs:
        o.checkpoint(b)
    for level in (1, 2):
        ck = Checkpointer(128)
        ck.set_profiling(level)
        pipelined(ck, [_dev(b) for b in bufs], bufs[0].size)
        for k in range(len(bufs)):
            assert ck.diff_to_host(k) == o.diff(k), (level, k)
            pt = ck.phase_times(k)
            assert pt["leaf_hash"] > 0 and pt["total"] >= pt["leaf_hash"], (level, k, pt)
            if level == 2:
                assert pt["insert"] > 0 and pt["phase2"] > 0 and pt["phase3"] > 0 and pt["compact"] > 0, pt
        ck.close()


def test_async_d2h_of_collected_diffs_keeps_pipelining(oracle_mod):
    """diff_to_host_async of a collected diff while the next pipelined call is in flight (no
    collection of that call): every host copy equals the oracle's diff, and the handle still
    has the newer call outstanding afterwards (one host wait per call in total)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    bufs = dup_lineage(21, 3000 * 128 - 9, 128, K=7, alphabet=5, p_change=0.7)
    o = oracle_mod.Oracle(128)
    for b in bufs:
        o.checkpoint(b)
    ck = Checkpointer(128)
    devs = [_dev(b) for b in bufs]
    torch.cuda.synchronize()
    d2h = torch.cuda.Stream()
    cap = 64 + 12 * 3000 + 16 + bufs[0].size
    hosts = [torch.empty(cap, dtype=torch.uint8).pin_memory() for _ in bufs]
    sizes = {}
    s0 = ck.host_syncs
    pend = None
    for k, t in enumerate(devs):
        cid = ck.submit(t)
        if pend is not None:
            d = ck.wait(pend)
            sizes[pend] = d["bytes"]
            ck.diff_to_host_async(pend, hosts[pend], d2h, nbytes=cap)
        pend = cid
    assert ck.host_syncs - s0 == len(bufs) - 1          # the newest call is still outstanding
    d = ck.wait(pend)
    sizes[pend] = d["bytes"]
    ck.diff_to_host_async(pend, hosts[pend], d2h, nbytes=cap)
    d2h.synchronize()
    for k in range(len(bufs)):
        assert bytes(hosts[k][:sizes[k]].numpy()) == o.diff(k), k
    ck.close()


def _alternating_lineage(nbytes, C, K, seed=5):
    """Checkpoints alternate between rewriting every chunk and changing ~1 % of them, so the
    SM partition a pipelined call picks from the previous call's candidate count (DESIGN.md
    §1a: none above 40 x 2 300 candidates, 16 chain SMs below 16 x 2 300) switches at every
    call, and the chain stream changes from call to call."""
    rng = np.random.default_rng(seed)
    buf = rng.integers(0, 256, nbytes, dtype=np.uint8)
    out = [buf.copy()]
    for k in range(1, K):
        if k % 2:
            buf = rng.integers(0, 256, nbytes, dtype=np.uint8)
        else:
            n = nbytes // C
            for c in rng.choice(n, size=max(1, n // 100), replace=False):
                buf[c * C] ^= 0x5A
        out.append(buf.copy())
    return out


@pytest.mark.parametrize("green", ["1", "0"])
def test_partition_switching_pipelined(oracle_mod, monkeypatch, green):
    # 16 MiB at C = 128: 131 072 leaves; a full rewrite is above the largest partition's
    # threshold, a 1 % change below the smallest. green = "0": the unpartitioned form.
    if green == "0":
        monkeypatch.setenv("CKPT_GREEN", "0")
    else:
        monkeypatch.delenv("CKPT_GREEN", raising=False)
    run_pipe_parity(oracle_mod, _alternating_lineage((16 << 20) + 48, 128, 8), 128)


@pytest.mark.parametrize("seed", [3, 11])
def test_full_depth_in_flight(oracle_mod, seed):
    # CKPT_PIPELINE_DEPTH calls in flight, submitted through the generic depth loop of bench.py
    # (K1(k) reuses the buffers of call k - depth while the calls between are in their tree
    # phases; a depth-3 build, CKPT_PIPE_DEPTH=3, passed the same tests)
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    from paper_conf_icpp_tanlmtmbctn23_b200.ckpt import PIPELINE_DEPTH
    rng = np.random.default_rng(seed)
    bufs = dup_lineage(seed, int(rng.integers(40_000, 400_000)), 128, K=9, alphabet=4, p_change=0.5)
    run_pipe_parity(oracle_mod, bufs, 128, depth=PIPELINE_DEPTH)
    run_pipe_parity(oracle_mod, list(W.lineage(2, (1 << 22) + 100, 128, 8, p=0.05)), 128, depth=PIPELINE_DEPTH)
