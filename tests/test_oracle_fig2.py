"""Figure 2 worked example, reproduced exactly by the oracle."""
import json
import os

import numpy as np

GOLD = os.path.join(os.path.dirname(__file__), "golden", "fig2.json")
NAMES = {"FIRST": 1, "FIXED": 2, "SHIFT": 3}


def _content(name, C):
    rng = np.random.default_rng(int.from_bytes(name.encode(), "little"))
    return rng.integers(0, 256, C, dtype=np.uint8).tobytes()


def test_fig2(oracle_mod):
    g = json.load(open(GOLD))
    C = g["chunk_bytes"]
    cont = {nm: _content(nm, C) for nm in set(g["ckpt0"] + g["ckpt1"])}
    assert len(set(cont.values())) == len(cont)  # all named chunks distinct
    o = oracle_mod.Oracle(C)
    b0 = b"".join(cont[x] for x in g["ckpt0"])
    b1 = b"".join(cont[x] for x in g["ckpt1"])
    o.checkpoint(b0)
    assert o.record_size() == g["ckpt0_record_size"]
    d0 = oracle_mod.parse_diff(o.diff(0))
    assert d0["first"] == g["ckpt0_first_regions"] and d0["shift"] == []
    rec0 = o.record()
    o.checkpoint(b1)
    lab, sn, sc = o.leaf_labels(1)
    assert [int(x) for x in lab] == [NAMES[x] for x in g["ckpt1_leaf_labels"]]
    for i, s in enumerate(g["ckpt1_leaf_src"]):
        if s is not None:
            assert (int(sn[i]), int(sc[i])) == tuple(s)
    new = {(node, ck) for (_, node, ck) in o.record() - rec0}
    # four leaf inserts I,J,K,L (nodes 7-10) plus phase-2 nodes 3, 4, 1
    assert new == {(u, 1) for u in [7, 8, 9, 10] + g["ckpt1_phase2_record_inserts"]}
    d1 = oracle_mod.parse_diff(o.diff(1))
    assert d1["first"] == g["ckpt1_first_regions"]
    assert [tuple(x) for x in d1["shift"]] == [tuple(x) for x in g["ckpt1_shift_regions"]]
    st = o.stats(1)
    assert st["list_entries"] == g["ckpt1_list_entries"]
    assert st["n_first_regions"] + st["n_shift_regions"] == g["ckpt1_tree_entries"]
    assert o.restore(0) == b0 and o.restore(1) == b1


def test_fig2_internal_node_keys(oracle_mod):
    """R2 ("hashing the left child's hash with the right child's hash"): the record
    keys of Figure 2's phase-2 nodes are MMH3 over the 32-byte concatenation T[l] || T[r],
    seed 0. The expected keys are composed here from the SMHasher-pinned leaf hash
    (tests/test_oracle_murmur.py), not from the oracle's tree code, so an oracle that hashed
    r || l, used another seed or a domain separator would fail."""
    g = json.load(open(GOLD))
    C = g["chunk_bytes"]
    cont = {nm: _content(nm, C) for nm in set(g["ckpt0"] + g["ckpt1"])}
    o = oracle_mod.Oracle(C)
    o.checkpoint(b"".join(cont[x] for x in g["ckpt0"]))
    o.checkpoint(b"".join(cont[x] for x in g["ckpt1"]))
    h = oracle_mod.mmh3
    T = {7: h(cont["I"]), 8: h(cont["J"]), 9: h(cont["K"]), 10: h(cont["L"])}
    T[3] = h(T[7] + T[8])
    T[4] = h(T[9] + T[10])
    T[1] = h(T[3] + T[4])
    rec = {(key, node, ck) for (key, node, ck) in o.record()}
    for u in (7, 8, 9, 10, 3, 4, 1):
        assert (T[u], u, 1) in rec, u
    keys = {key for (key, _, _) in rec}
    assert h(T[8] + T[7]) not in keys          # not r || l
    assert h(T[7] + T[8], 1) not in keys       # not another seed
    # checkpoint 0 taken whole: the root key is the Merkle root of A0..A7
    L = [h(cont[f"A{i}"]) for i in range(8)]
    while len(L) > 1:
        L = [h(L[2 * i] + L[2 * i + 1]) for i in range(len(L) // 2)]
    assert (L[0], 0, 0) in rec
