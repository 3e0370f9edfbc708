"""CPU oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, single-threaded C++17 implementation of Algorithm 1 of Tan et al.
(ICPP'23), its serialisation and restore
(P:158), loaded through ctypes. Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this module.
The product package ``paper_conf_icpp_tanlmtmbctn23_b200`` never imports it and
shares no code with it.

Parity unpinned: optimality of the region set (P:87 calls the method a heuristic);
every other function is pinned by tests/test_oracle_*.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SOURCES = ["murmur3_ref.cpp", "oracle.cpp"]

LABEL_NONE, FIRST, FIXED, SHIFT, DONE = 0, 1, 2, 3, 4

STAT_NAMES = [
    "id", "bytes", "meta_bytes", "data_bytes", "n_first_regions", "n_shift_regions",
    "n_first", "n_fixed", "n_spatial", "n_temporal", "list_entries", "record_growth",
    "phase2_inserts", "n_leaves", "phase3_inserts",
]


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (plain -O2, single-threaded)."""
    srcs = [os.path.join(_HERE, s) for s in _SOURCES]
    if not force and os.path.exists(_LIB_PATH):
        lib_m = os.path.getmtime(_LIB_PATH)
        if all(os.path.getmtime(s) <= lib_m for s in srcs):
            return _LIB_PATH
    cmd = ["g++", "-std=c++17", "-O2", "-fPIC", "-shared", "-o", _LIB_PATH] + srcs
    subprocess.check_call(cmd)
    return _LIB_PATH


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        u8p = ctypes.POINTER(ctypes.c_uint8)
        L.orc_mmh3.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p]
        L.orc_mmh3.restype = None
        L.orc_create.argtypes = [ctypes.c_uint32, ctypes.c_int]
        L.orc_create.restype = ctypes.c_void_p
        L.orc_create_mode.argtypes = [ctypes.c_uint32, ctypes.c_int, ctypes.c_int]
        L.orc_create_mode.restype = ctypes.c_void_p
        L.orc_set_variant.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint32]
        L.orc_set_variant.restype = ctypes.c_int
        L.orc_destroy.argtypes = [ctypes.c_void_p]
        L.orc_destroy.restype = None
        L.orc_checkpoint.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64]
        L.orc_checkpoint.restype = ctypes.c_int
        for name in ("orc_num_checkpoints",):
            getattr(L, name).argtypes = [ctypes.c_void_p]
            getattr(L, name).restype = ctypes.c_uint32
        for name in ("orc_num_leaves", "orc_record_size"):
            getattr(L, name).argtypes = [ctypes.c_void_p]
            getattr(L, name).restype = ctypes.c_uint64
        L.orc_diff_size.argtypes = [ctypes.c_void_p, ctypes.c_uint32]
        L.orc_diff_size.restype = ctypes.c_uint64
        L.orc_diff_copy.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
        L.orc_diff_copy.restype = ctypes.c_int
        L.orc_stats.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
        L.orc_stats.restype = ctypes.c_int
        L.orc_leaf_digests.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        L.orc_leaf_digests.restype = ctypes.c_int
        L.orc_leaf_labels.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                      ctypes.c_void_p, ctypes.c_void_p]
        L.orc_leaf_labels.restype = ctypes.c_int
        L.orc_record_dump.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        L.orc_record_dump.restype = ctypes.c_int
        L.orc_restore.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
        L.orc_restore.restype = ctypes.c_int
        for name in ("orc_node_of_chunk", "orc_lo", "orc_hi"):
            getattr(L, name).argtypes = [ctypes.c_void_p, ctypes.c_uint64]
            getattr(L, name).restype = ctypes.c_uint64
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> ctypes.c_void_p:
    return ctypes.c_void_p(a.ctypes.data)


def mmh3(data: bytes, seed: int = 0) -> bytes:
    """MurmurHash3_x64_128 digest, 16 bytes = h1 LE || h2 LE (reading R1)."""
    buf = np.frombuffer(bytes(data) + b"\0", dtype=np.uint8)  # +1 keeps the pointer valid for len 0
    out = np.zeros(16, dtype=np.uint8)
    lib().orc_mmh3(_ptr(buf), len(data), seed, _ptr(out))
    return out.tobytes()


MODE_TREE, MODE_LIST, MODE_BASIC = 0, 1, 2   # the methods compared in P:194 (Tree = ours)
VAR_FULL_FIRST, VAR_FULL_SWITCH = 1, 2       # Tree-method variants (NEXT #4)
VAR_SHIFT_INSERT = 4                         # NEXT #4(c): the SHIFT-SHIFT-insert reading of P:89 (R24)
FLAGS_FULL = 3                               # header flags of a difference stored in full
FLAGS_SHIFT_INSERT = 4                       # header flags of a Tree difference under VAR_SHIFT_INSERT


class Oracle:
    """One de-duplication lineage (one process / GPU in the paper).
    mode: MODE_TREE (Algorithm 1), MODE_LIST or MODE_BASIC."""

    def __init__(self, chunk_bytes: int, ideal: bool = False, mode: int = MODE_TREE):
        self._h = lib().orc_create_mode(chunk_bytes, 1 if ideal else 0, mode)
        if not self._h:
            raise ValueError("bad chunk size or mode")
        self.chunk_bytes = chunk_bytes
        self.ideal = ideal
        self.mode = mode
        self.buf_bytes = None

    def set_variant(self, flags: int, switch_permille: int = 1000) -> None:
        """VAR_FULL_FIRST / VAR_FULL_SWITCH (Tree mode, before the first checkpoint)."""
        if lib().orc_set_variant(self._h, flags, switch_permille) != 0:
            raise ValueError("variant rejected")

    def close(self):
        if self._h:
            lib().orc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def checkpoint(self, buf) -> int:
        a = np.ascontiguousarray(np.frombuffer(memoryview(buf).cast("B"), dtype=np.uint8))
        rc = lib().orc_checkpoint(self._h, _ptr(a), a.size)
        if rc != 0:
            raise RuntimeError(f"oracle checkpoint failed rc={rc}")
        self.buf_bytes = a.size
        return self.num_checkpoints - 1

    @property
    def num_checkpoints(self) -> int:
        return lib().orc_num_checkpoints(self._h)

    @property
    def n_leaves(self) -> int:
        return lib().orc_num_leaves(self._h)

    def diff(self, cid: int) -> bytes:
        size = lib().orc_diff_size(self._h, cid)
        out = np.zeros(max(size, 1), dtype=np.uint8)
        if lib().orc_diff_copy(self._h, cid, _ptr(out)) != 0:
            raise IndexError(cid)
        return out[:size].tobytes()

    def stats(self, cid: int) -> dict:
        out = np.zeros(16, dtype=np.uint64)
        if lib().orc_stats(self._h, cid, _ptr(out)) != 0:
            raise IndexError(cid)
        return {name: int(out[i]) for i, name in enumerate(STAT_NAMES)}

    def leaf_digests(self) -> np.ndarray:
        out = np.zeros((self.n_leaves, 16), dtype=np.uint8)
        if lib().orc_leaf_digests(self._h, _ptr(out)) != 0:
            raise RuntimeError("digests unavailable in ideal mode")
        return out

    def leaf_labels(self, cid: int):
        n = self.n_leaves
        lab = np.zeros(n, dtype=np.uint8)
        sn = np.zeros(n, dtype=np.uint32)
        sc = np.zeros(n, dtype=np.uint32)
        if lib().orc_leaf_labels(self._h, cid, _ptr(lab), _ptr(sn), _ptr(sc)) != 0:
            raise IndexError(cid)
        return lab, sn, sc

    def record_size(self) -> int:
        return lib().orc_record_size(self._h)

    def record(self):
        """Set of (digest bytes, node, ckpt)."""
        m = self.record_size()
        keys = np.zeros((max(m, 1), 16), dtype=np.uint8)
        nodes = np.zeros(max(m, 1), dtype=np.uint32)
        ckpts = np.zeros(max(m, 1), dtype=np.uint32)
        if lib().orc_record_dump(self._h, _ptr(keys), _ptr(nodes), _ptr(ckpts)) != 0:
            raise RuntimeError("record dump unavailable in ideal mode")
        return {(keys[i].tobytes(), int(nodes[i]), int(ckpts[i])) for i in range(m)}

    def record_array(self) -> np.ndarray:
        """The record as a sorted array of rows (key lo, key hi, ckpt << 32 | node), u64 each
        (the same content as record(), for fast comparison at millions of entries)."""
        m = self.record_size()
        keys = np.zeros((max(m, 1), 16), dtype=np.uint8)
        nodes = np.zeros(max(m, 1), dtype=np.uint32)
        ckpts = np.zeros(max(m, 1), dtype=np.uint32)
        if lib().orc_record_dump(self._h, _ptr(keys), _ptr(nodes), _ptr(ckpts)) != 0:
            raise RuntimeError("record dump unavailable in ideal mode")
        rows = np.empty((m, 3), dtype=np.uint64)
        rows[:, :2] = keys[:m].view(np.uint64)
        rows[:, 2] = (ckpts[:m].astype(np.uint64) << np.uint64(32)) | nodes[:m]
        return rows[np.lexsort((rows[:, 2], rows[:, 1], rows[:, 0]))]

    def restore(self, cid: int) -> bytes:
        out = np.zeros(max(self.buf_bytes or 1, 1), dtype=np.uint8)
        rc = lib().orc_restore(self._h, cid, _ptr(out))
        if rc != 0:
            raise RuntimeError(f"oracle restore failed rc={rc}")
        return out[: self.buf_bytes].tobytes()

    # geometry (reading R3)
    def node_of_chunk(self, i: int) -> int:
        return lib().orc_node_of_chunk(self._h, i)

    def lo(self, u: int) -> int:
        return lib().orc_lo(self._h, u)

    def hi(self, u: int) -> int:
        return lib().orc_hi(self._h, u)


def parse_diff(d: bytes) -> dict:
    """Decode the consolidated-difference byte format (reading R13).
    Basic diffs (flags == 2) carry a changed-chunk bitmap instead of entry lists."""
    import struct
    magic, ver, flags, cid, C, B, n, nF, nS, data_bytes, seed, _res = struct.unpack_from("<IHHIIQQQQQII", d, 0)
    if flags == MODE_BASIC:
        words = (n + 31) // 32
        bits = list(struct.unpack_from(f"<{words}I", d, 64)) if words else []
        changed = [i for i in range(n) if (bits[i // 32] >> (i % 32)) & 1]
        meta = (64 + 4 * words + 15) // 16 * 16
        return dict(magic=magic, version=ver, flags=flags, id=cid, chunk_bytes=C, buf_bytes=B, n_leaves=n,
                    changed=changed, n_changed=nF, data_bytes=data_bytes, seed=seed, meta_bytes=meta,
                    data=d[meta:], first=[], shift=[])
    F = list(struct.unpack_from(f"<{nF}I", d, 64)) if nF else []
    S = []
    off = 64 + 4 * nF
    for e in range(nS):
        S.append(struct.unpack_from("<III", d, off + 12 * e))
    meta = 64 + 4 * nF + 12 * nS
    meta = (meta + 15) // 16 * 16
    return dict(magic=magic, version=ver, flags=flags, id=cid, chunk_bytes=C, buf_bytes=B,
                n_leaves=n, first=F, shift=S, data_bytes=data_bytes, seed=seed,
                meta_bytes=meta, data=d[meta:])
