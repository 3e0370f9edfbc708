"""GPU <-> oracle parity at the sizes SURVEY §8(c)/(d) name for the oracle, element by
element (bit-exact):

- config 4 (duplicate-heavy, spatial + temporal de-dup) at 2^26 bytes x 20 checkpoints;
- config 2 (GDV-like) at the benchmarked 1 GiB, C = 128 B, p = 1 %, 4 checkpoints, in the
  launch configuration bench.py times (the device generator writes the buffers, the oracle
  de-duplicates host copies of the same bytes).

Each checkpoint compares the whole diff bytes, the per-checkpoint statistics, every leaf
digest and the record as a set; every checkpoint is restored on the device and compared
with its input.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

STAT_KEYS = ["n_first_regions", "n_shift_regions", "n_first", "n_fixed", "n_spatial", "n_temporal",
             "list_entries", "meta_bytes", "data_bytes", "bytes", "phase2_inserts"]


def _check_step(ck, o, k, d):
    st = o.stats(k)
    for key in STAT_KEYS:
        assert d[key] == st[key], (k, key, d[key], st[key])
    assert d["record_size"] == o.record_size(), k
    assert ck.diff_to_host(k) == o.diff(k), k
    n = o.n_leaves
    dd = torch.empty(16 * n, dtype=torch.uint8, device="cuda")
    ck.leaf_digests(dd)
    assert np.array_equal(dd.cpu().numpy().reshape(n, 16), o.leaf_digests()), k
    assert np.array_equal(ck.record_array(), o.record_array()), k


def test_config4_64mib_20_checkpoints(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B, C, K = 1 << 26, 128, 20
    o = oracle_mod.Oracle(C)
    ck = Checkpointer(C)
    devs = []
    for k, b in enumerate(W.lineage(4, B, C, K)):
        o.checkpoint(b)
        t = torch.from_numpy(b).cuda()
        devs.append(t)
        d = ck.checkpoint(t)
        _check_step(ck, o, k, d)
        if k:
            assert d["n_spatial"] + d["n_temporal"] > 0, k   # the workload de-duplicates
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(K):
        ck.restore(k, out)
        assert torch.equal(out, devs[k]), k
    ck.close()


def test_config2_1gib_benchmarked(oracle_mod):
    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    from paper_conf_icpp_tanlmtmbctn23_b200 import workloads as W
    B, C, K, p = 1 << 30, 128, 4, 0.01
    seed = W.seed_of(2)
    st = torch.cuda.Stream()          # bench.py times the calls on a side stream
    bufs = [torch.empty(B, dtype=torch.uint8, device="cuda") for _ in range(K)]
    with torch.cuda.stream(st):
        W.DeviceGen.initial(2, bufs[0], B, seed, st)
        for k in range(1, K):
            bufs[k].copy_(bufs[k - 1])
            W.DeviceGen.mutate(2, bufs[k], B, k, C, seed, p, st)
    st.synchronize()
    o = oracle_mod.Oracle(C)
    ck = Checkpointer(C)
    ck.set_profiling(1)               # bench.py's timed profiling level
    for k in range(K):
        o.checkpoint(bufs[k].cpu().numpy())
        d = ck.checkpoint(bufs[k], stream=st)
        _check_step(ck, o, k, d)
    out = torch.empty(B, dtype=torch.uint8, device="cuda")
    for k in range(K):
        ck.restore(k, out)
        assert torch.equal(out, bufs[k]), k
    ck.close()
