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
