"""C-ABI behaviour on the GPU: error contract (include/ckpt.h), host-memory path (one H2D,
one D2H), device generators == host generators, and full-size (1 GiB,
config 2) properties in the launch configuration bench.py times."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def test_error_contract():
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, CkptError
    from paper_conf_icpp_tanlmtmbctn23_b200.ckpt import CKPT_EINVAL, CKPT_ERANGE
    with pytest.raises(CkptError) as e:
        Checkpointer(40)                       # not a multiple of 16
    assert e.value.status == CKPT_EINVAL
    with pytest.raises(CkptError):
        Checkpointer(16)                       # below 32 B
    ck = Checkpointer(64)
    buf = torch.zeros(4096 + 16, dtype=torch.uint8, device="cuda")
    with pytest.raises(CkptError) as e:
        ck.checkpoint(buf[1:], nbytes=4096)    # misaligned
    assert e.value.status == CKPT_EINVAL
    host = np.zeros(4096, dtype=np.uint8)
    with pytest.raises(CkptError) as e:
        ck.checkpoint(host.ctypes.data, nbytes=4096)   # host pointer to the device entry point
    assert e.value.status == CKPT_EINVAL
    ck.checkpoint(buf, nbytes=4096)
    with pytest.raises(CkptError) as e:
        ck.checkpoint(buf, nbytes=2048)        # size change (R17)
    assert e.value.status == CKPT_EINVAL
    with pytest.raises(CkptError) as e:
        ck.restore(5, buf)
    assert e.value.status == CKPT_ERANGE
    assert ck.num_checkpoints == 1
    ck.close()


def test_host_path_and_d2h(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    bufs = list(W.lineage(1, 1 << 20, 128, 4))
    o = oracle_mod.Oracle(128)
    ck = Checkpointer(128)
    out = torch.empty(2 << 20, dtype=torch.uint8).pin_memory()
    for k, b in enumerate(bufs):
        o.checkpoint(b)
        hb = torch.from_numpy(b).pin_memory()
        d = ck.checkpoint_host(hb, host_diff=out)
        assert bytes(out[: d["bytes"]].numpy()) == o.diff(k)
    ck.close()


@pytest.mark.parametrize("cfg,nbytes,C,p", [(1, (1 << 20) + 5, 128, 0.01), (2, (1 << 22) + 100, 128, 0.05),
                                            (2, 3 * 292 + 7, 64, 0.5)])
def test_device_generators_match_host(cfg, nbytes, C, p):
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    assert list(W.DeviceGen.freq_orbits()) == list(W.FREQ_ORBITS)
    seed = W.seed_of(cfg)
    t = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    W.DeviceGen.initial(cfg, t, nbytes, seed)
    for k, hb in enumerate(W.lineage(cfg, nbytes, C, 4, p=p)):
        if k:
            W.DeviceGen.mutate(cfg, t, nbytes, k, C, seed, p)
        torch.cuda.synchronize()
        assert np.array_equal(t.cpu().numpy(), hb), k


def test_full_size_config2_properties(oracle_mod):
    """BASELINE configs[1] at full size (1 GiB, C = 128) in bench.py's launch configuration:
    restore(k) == input_k on the device; sampled leaf digests == the oracle's Murmur3;
    diff header/size identities; sampled FIRST data equals the input chunks."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B, C, K = 1 << 30, 128, 4
    seed = W.seed_of(2)
    ck = Checkpointer(C)
    bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
    W.DeviceGen.initial(2, bufs[0], B, seed)
    for k in range(1, K):
        bufs[k].copy_(bufs[k - 1])
        W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, 0.01)
    n = B // C
    rng = np.random.default_rng(0)
    sample = np.sort(rng.choice(n, 2000, replace=False))
    dd = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
    for k in range(K):
        d = ck.checkpoint(bufs[k])
        assert d["bytes"] == d["meta_bytes"] + d["data_bytes"]
        assert d["meta_bytes"] == (64 + 4 * d["n_first_regions"] + 12 * d["n_shift_regions"] + 15) // 16 * 16
        assert d["n_first"] + d["n_fixed"] + d["n_spatial"] + d["n_temporal"] == n
        if k:
            assert d["n_fixed"] > 0.95 * n
        ck.leaf_digests(dd)
        dig = dd.view(n, 16)[torch.from_numpy(sample).cuda()].cpu().numpy()
        host = bufs[k].view(n, C)[torch.from_numpy(sample).cuda()].cpu().numpy()
        for i in range(len(sample)):
            assert oracle_mod.mmh3(host[i].tobytes()) == dig[i].tobytes()
        raw = ck.diff_to_host(k)
        p = oracle_mod.parse_diff(raw)
        assert p["id"] == k and p["n_leaves"] == n and len(p["data"]) == d["data_bytes"]
        # first FIRST regions' bytes equal the input at their position
        off = 0
        hb = None
        for u in p["first"][:50]:
            depth = (u + 1).bit_length() - 1
            L = 30 - 7 - depth          # h = 23 for n = 2^23
            lo = (u + 1 - (1 << depth)) << L
            ln = (1 << L) * C
            seg = bufs[k][lo * C: lo * C + ln].cpu().numpy().tobytes()
            assert p["data"][off:off + ln] == seg
            off += ln
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(K):
        ck.restore(k, out)
        assert torch.equal(out, bufs[k]), k
    ck.close()


def test_phase_times_ring():
    """ckpt_phase_times_of: per-checkpoint device phase times (CUDA events), queried after
    the calls; the per-phase times add up to at most the whole-call time."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, CkptError
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    ck = Checkpointer(128)
    ck.set_profiling(True)
    bufs = list(W.lineage(2, 1 << 24, 128, 4, p=0.01))
    for b in bufs:
        ck.checkpoint(torch.from_numpy(b).cuda(), nbytes=b.size)
    for k in range(len(bufs)):
        t = ck.phase_times(k)
        parts = sum(t[x] for x in ("leaf_hash", "insert", "phase2", "phase3", "compact"))
        assert all(t[x] >= 0 for x in t)
        assert 0 < parts <= t["total"] * 1.001 + 1e-3, (k, t)
    with pytest.raises(CkptError):
        ck.phase_times(len(bufs))
    ck.set_profiling(1)                # K1 + whole call only
    b = W.cfg2_mutate(bufs[-1].copy(), len(bufs), W.seed_of(2), 0.01)
    ck.checkpoint(torch.from_numpy(b).cuda(), nbytes=b.size)
    t = ck.phase_times()
    assert 0 < t["leaf_hash"] <= t["total"] and t["insert"] == t["phase2"] == t["phase3"] == t["compact"] == 0
    with pytest.raises(CkptError):
        ck.set_profiling(3)
    ck.close()


def test_kernel_launch_counter():
    """ckpt_kernel_launches counts what the library enqueues: a steady checkpoint of a
    2^23-chunk buffer is K1, K1b, phase 2, phase 3, gather = 5 kernels
    (plus K1t only when B is not a multiple of 256 C)."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    ck = Checkpointer(128)
    buf = torch.zeros(1 << 30, dtype=torch.uint8, device="cuda")
    assert ck.kernel_launches == 0
    ck.checkpoint(buf)
    a = ck.kernel_launches
    ck.checkpoint(buf)
    assert ck.kernel_launches - a == 5
    out = torch.empty_like(buf)
    b = ck.kernel_launches
    ck.restore(1, out)
    assert ck.kernel_launches > b and torch.equal(out, buf)
    ck.close()


def test_diff_to_host_async_overlaps_next_checkpoint(oracle_mod):
    """NEXT #1: the one D2H of diff k (ckpt_diff_to_host_async on a side stream) may run
    while checkpoint k+1 de-duplicates; every copy equals the oracle's diff."""
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer, CkptError
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    C = 128
    bufs = list(W.lineage(2, (1 << 22) + 100, C, 6, p=0.05))
    B = bufs[0].size
    o = oracle_mod.Oracle(C)
    ck = Checkpointer(C)
    side = torch.cuda.Stream()
    main = torch.cuda.Stream()
    devs = [torch.from_numpy(np.ascontiguousarray(b)).cuda() for b in bufs]
    hosts = []
    for k, b in enumerate(bufs):
        d = ck.checkpoint(devs[k], nbytes=B, stream=main)
        o.checkpoint(b)
        h = torch.empty(d["bytes"], dtype=torch.uint8).pin_memory()
        ck.diff_to_host_async(k, h, side)
        hosts.append(h)
    side.synchronize()
    for k in range(len(bufs)):
        assert bytes(hosts[k].numpy()) == o.diff(k), k
    with pytest.raises(CkptError):
        ck.diff_to_host_async(0, torch.empty(8, dtype=torch.uint8).pin_memory(), side)   # too small
    with pytest.raises(CkptError):
        ck.diff_to_host_async(len(bufs), hosts[0], side)                                 # no such diff
    ck.close()
