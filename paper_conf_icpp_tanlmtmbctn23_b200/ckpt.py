"""Thin Python binding of libckpt.so (include/ckpt.h) — argument marshalling only.

Every step of the de-duplication path runs in the library's sm_100a kernels; this module
only converts torch tensors / integers into the C ABI's pointers and sizes. There is no
CPU fallback: if the extension is missing or no B200 is visible, calls raise.

    from paper_conf_icpp_tanlmtmbctn23_b200 import Checkpointer
    ck = Checkpointer(chunk_bytes=128)
    d = ck.checkpoint(buf)            # buf: torch.uint8 CUDA tensor (16-B aligned)
    ck.restore(d["id"], out)          # out: torch.uint8 CUDA tensor of the same size
"""
from __future__ import annotations

import ctypes
import os

from . import _build

CKPT_OK, CKPT_EINVAL, CKPT_ENOMEM, CKPT_ECUDA, CKPT_ERANGE, CKPT_ESTATE, CKPT_ECOLLIDE = range(7)

CKPT_MODE_TREE, CKPT_MODE_LIST, CKPT_MODE_BASIC = 0, 1, 2   # methods of P:194 (include/ckpt.h)
CKPT_VARIANT_FULL_FIRST, CKPT_VARIANT_FULL_SWITCH = 1, 2      # Tree variants
CKPT_VARIANT_SHIFT_INSERT = 4                                 # Tree variant: P:89's insert reading (R24)
CKPT_FLAGS_FULL = 3                                           # header flags of a full difference
CKPT_FLAGS_SHIFT_INSERT = 4                                   # header flags under the SHIFT-insert variant

ABI_FUNCTIONS = [
    "ckpt_create", "ckpt_create_mode", "ckpt_set_variant", "ckpt_checkpoint", "ckpt_checkpoint_submit",
    "ckpt_checkpoint_wait", "ckpt_restore",
    "ckpt_restore_stream", "ckpt_diff_info", "ckpt_diff_to_host", "ckpt_diff_to_host_async",
    "ckpt_checkpoint_host", "ckpt_import", "ckpt_num_checkpoints", "ckpt_leaf_digests", "ckpt_record_dump",
    "ckpt_set_profiling", "ckpt_phase_times", "ckpt_phase_times_of", "ckpt_kernel_launches",
    "ckpt_host_syncs", "ckpt_destroy", "ckpt_strerror",
]


PIPELINE_DEPTH = 2   # include/ckpt.h CKPT_PIPELINE_DEPTH: pipelined calls in flight at most


class CkptDiff(ctypes.Structure):
    _fields_ = [
        ("id", ctypes.c_uint32),
        ("chunk_bytes", ctypes.c_uint32),
        ("dev_ptr", ctypes.c_void_p),
        ("bytes", ctypes.c_uint64),
        ("meta_bytes", ctypes.c_uint64),
        ("data_bytes", ctypes.c_uint64),
        ("buf_bytes", ctypes.c_uint64),
        ("n_leaves", ctypes.c_uint64),
        ("n_first_regions", ctypes.c_uint64),
        ("n_shift_regions", ctypes.c_uint64),
        ("n_first", ctypes.c_uint64),
        ("n_fixed", ctypes.c_uint64),
        ("n_spatial", ctypes.c_uint64),
        ("n_temporal", ctypes.c_uint64),
        ("list_entries", ctypes.c_uint64),
        ("record_size", ctypes.c_uint64),
        ("record_capacity", ctypes.c_uint64),
        ("phase2_inserts", ctypes.c_uint64),
        ("phase3_inserts", ctypes.c_uint64),
    ]

    def as_dict(self) -> dict:
        return {name: getattr(self, name) for name, _ in self._fields_}


class CkptError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: {strerror(status)} (status {status})")
        self.status = status


_lib = None


def lib() -> ctypes.CDLL:
    """Load the in-tree libckpt.so (fails loudly if it is missing)."""
    global _lib
    if _lib is None:
        # CKPT_LIB: an alternative in-tree build of the same library (A/B experiments)
        path = os.environ.get("CKPT_LIB") or _build.lib_path("libckpt.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(path)
        vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        P = ctypes.POINTER
        sig = {
            "ckpt_create": ([u32, P(vp)], i32),
            "ckpt_create_mode": ([u32, i32, P(vp)], i32),
            "ckpt_set_variant": ([vp, u32, u32], i32),
            "ckpt_checkpoint": ([vp, vp, u64, vp, P(CkptDiff)], i32),
            "ckpt_checkpoint_submit": ([vp, vp, u64, vp, P(u32)], i32),
            "ckpt_checkpoint_wait": ([vp, u32, vp, P(CkptDiff)], i32),
            "ckpt_restore": ([vp, u32, vp], i32),
            "ckpt_restore_stream": ([vp, u32, vp, vp], i32),
            "ckpt_diff_info": ([vp, u32, P(CkptDiff)], i32),
            "ckpt_diff_to_host": ([vp, u32, vp, u64], i32),
            "ckpt_diff_to_host_async": ([vp, u32, vp, u64, vp], i32),
            "ckpt_checkpoint_host": ([vp, vp, u64, vp, vp, u64, P(CkptDiff)], i32),
            "ckpt_num_checkpoints": ([vp, P(u32)], i32),
            "ckpt_import": ([vp, vp, u64, vp], i32),
            "ckpt_leaf_digests": ([vp, vp], i32),
            "ckpt_record_dump": ([vp, vp, vp, vp, u64, P(u64)], i32),
            "ckpt_set_profiling": ([vp, i32], i32),
            "ckpt_phase_times": ([vp, P(ctypes.c_float), i32], i32),
            "ckpt_phase_times_of": ([vp, u32, P(ctypes.c_float), i32], i32),
            "ckpt_kernel_launches": ([vp, P(ctypes.c_uint64)], i32),
            "ckpt_host_syncs": ([vp, P(ctypes.c_uint64)], i32),
            "ckpt_destroy": ([vp], i32),
            "ckpt_strerror": ([i32], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def strerror(status: int) -> str:
    return lib().ckpt_strerror(status).decode()


def _ptr(x) -> int:
    """Device/host pointer of a torch tensor, numpy array or raw integer."""
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(type(x))


def _nbytes(x) -> int:
    if hasattr(x, "element_size"):
        return x.numel() * x.element_size()
    if hasattr(x, "nbytes"):
        return int(x.nbytes)
    raise TypeError("pass nbytes explicitly")


def _stream_handle(stream) -> int:
    if stream is None:
        try:
            import torch
            return torch.cuda.current_stream().cuda_stream
        except Exception:
            return 0
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


class Checkpointer:
    """One de-duplication lineage on the current CUDA device (one per process / GPU)."""

    def __init__(self, chunk_bytes: int, mode: int = CKPT_MODE_TREE):
        h = ctypes.c_void_p()
        rc = lib().ckpt_create_mode(chunk_bytes, mode, ctypes.byref(h))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_create_mode")
        self._h = h
        self.chunk_bytes = chunk_bytes
        self.mode = mode
        self._ckpt_fn = lib().ckpt_checkpoint   # bound once: the per-call path is marshalling only
        self._submit_fn = lib().ckpt_checkpoint_submit
        self._wait_fn = lib().ckpt_checkpoint_wait

    def set_variant(self, flags: int, switch_permille: int = 1000) -> None:
        """CKPT_VARIANT_FULL_FIRST / CKPT_VARIANT_FULL_SWITCH (Tree mode, before the first
        checkpoint; include/ckpt.h)."""
        rc = lib().ckpt_set_variant(self._h, flags, switch_permille)
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_set_variant")

    # ------------------------------------------------------------------ core calls
    def checkpoint(self, buf, nbytes: int | None = None, stream=None, raw: bool = False):
        d = CkptDiff()
        n = _nbytes(buf) if nbytes is None else nbytes
        rc = self._ckpt_fn(self._h, _ptr(buf), n, _stream_handle(stream), ctypes.byref(d))
        if rc != CKPT_OK:
            if rc == CKPT_ECOLLIDE:   # committed with a warning (include/ckpt.h, R14)
                return self._collided(d, raw)
            raise CkptError(rc, "ckpt_checkpoint")
        return d if raw else d.as_dict()

    def submit(self, buf, nbytes: int | None = None, stream=None) -> int:
        """Pipelined checkpoint (include/ckpt.h ckpt_checkpoint_submit): enqueue and return the
        id; collect it with wait(). The buffer stays borrowed until wait(id) returns."""
        cid = ctypes.c_uint32()
        n = _nbytes(buf) if nbytes is None else nbytes
        rc = self._submit_fn(self._h, _ptr(buf), n, _stream_handle(stream), ctypes.byref(cid))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_checkpoint_submit")
        return cid.value

    def wait(self, cid: int, stream=None, raw: bool = False):
        """Statistics of submitted checkpoint `cid` (ckpt_checkpoint_wait); `stream` (default:
        torch's current stream) is ordered after the rest of that call's work."""
        d = CkptDiff()
        rc = self._wait_fn(self._h, cid, _stream_handle(stream), ctypes.byref(d))
        if rc != CKPT_OK:
            if rc == CKPT_ECOLLIDE:
                return self._collided(d, raw)
            raise CkptError(rc, "ckpt_checkpoint_wait")
        return d if raw else d.as_dict()

    @staticmethod
    def _collided(d, raw):
        import warnings
        warnings.warn(f"ckpt_checkpoint: 128-bit digest collision in checkpoint {d.id} (R14); "
                      "the checkpoint is committed, its colliding record insert was skipped",
                      RuntimeWarning, stacklevel=3)
        if raw:
            return d
        out = d.as_dict()
        out["collision"] = True
        return out

    def checkpoint_host(self, host_buf, host_diff=None, nbytes: int | None = None, stream=None):
        d = CkptDiff()
        n = _nbytes(host_buf) if nbytes is None else nbytes
        cap = _nbytes(host_diff) if host_diff is not None else 0
        rc = lib().ckpt_checkpoint_host(self._h, _ptr(host_buf), n, _stream_handle(stream),
                                        _ptr(host_diff) if host_diff is not None else None, cap, ctypes.byref(d))
        if rc != CKPT_OK:
            if rc == CKPT_ECOLLIDE:
                return self._collided(d, False)
            raise CkptError(rc, "ckpt_checkpoint_host")
        return d.as_dict()

    def import_diff(self, host_diff, stream=None) -> None:
        """Append diff number num_checkpoints from host memory (bytes, numpy array or a host
        tensor) after a restart, rebuilding the record and leaf digests (ckpt_import)."""
        if isinstance(host_diff, (bytes, bytearray)):
            buf = ctypes.create_string_buffer(bytes(host_diff), len(host_diff))
            ptr, n = ctypes.addressof(buf), len(host_diff)
        else:
            ptr, n = _ptr(host_diff), _nbytes(host_diff)
        rc = lib().ckpt_import(self._h, ptr, n, _stream_handle(stream))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_import")

    def restore(self, cid: int, out, stream=None) -> None:
        """Rebuild checkpoint cid into device tensor `out`, ordered after the work already
        enqueued on `stream` (default: torch's current stream); synchronous."""
        rc = lib().ckpt_restore_stream(self._h, cid, _ptr(out), _stream_handle(stream))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_restore_stream")

    def diff_info(self, cid: int) -> dict:
        d = CkptDiff()
        rc = lib().ckpt_diff_info(self._h, cid, ctypes.byref(d))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_diff_info")
        return d.as_dict()

    def diff_to_host(self, cid: int, out=None) -> bytes:
        """One D2H of the consolidated diff. Returns bytes (or fills `out`)."""
        info = self.diff_info(cid)
        if out is None:
            buf = ctypes.create_string_buffer(max(info["bytes"], 1))
            rc = lib().ckpt_diff_to_host(self._h, cid, ctypes.addressof(buf), info["bytes"])
            if rc != CKPT_OK:
                raise CkptError(rc, "ckpt_diff_to_host")
            return buf.raw[: info["bytes"]]
        rc = lib().ckpt_diff_to_host(self._h, cid, _ptr(out), _nbytes(out))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_diff_to_host")
        return None

    def diff_to_host_async(self, cid: int, out, stream, nbytes: int | None = None) -> None:
        """Enqueue the one D2H of diff `cid` into pinned host memory `out` on `stream` and
        return (NEXT #1: overlap with the next checkpoint); sync `stream` before reading."""
        cap = _nbytes(out) if nbytes is None else nbytes
        rc = lib().ckpt_diff_to_host_async(self._h, cid, _ptr(out), cap, _stream_handle(stream))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_diff_to_host_async")

    @property
    def num_checkpoints(self) -> int:
        c = ctypes.c_uint32()
        rc = lib().ckpt_num_checkpoints(self._h, ctypes.byref(c))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_num_checkpoints")
        return c.value

    # ------------------------------------------------------------------ introspection
    def leaf_digests(self, out) -> None:
        rc = lib().ckpt_leaf_digests(self._h, _ptr(out))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_leaf_digests")

    def record(self):
        """Historical record as a set of (digest bytes, node, ckpt)."""
        import numpy as np
        cnt = ctypes.c_uint64()
        rc = lib().ckpt_record_dump(self._h, None, None, None, 0, ctypes.byref(cnt))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_record_dump")
        m = cnt.value + 16
        keys = np.zeros((m, 16), dtype=np.uint8)
        nodes = np.zeros(m, dtype=np.uint32)
        ckpts = np.zeros(m, dtype=np.uint32)
        rc = lib().ckpt_record_dump(self._h, keys.ctypes.data, nodes.ctypes.data, ckpts.ctypes.data, m,
                                    ctypes.byref(cnt))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_record_dump")
        k = cnt.value
        return {(keys[i].tobytes(), int(nodes[i]), int(ckpts[i])) for i in range(k)}

    def record_array(self):
        """Historical record as a sorted numpy array of rows (key lo, key hi, ckpt << 32 | node),
        u64 each: the same content as record(), comparable with np.array_equal at millions of
        entries."""
        import numpy as np
        cnt = ctypes.c_uint64()
        rc = lib().ckpt_record_dump(self._h, None, None, None, 0, ctypes.byref(cnt))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_record_dump")
        m = cnt.value + 16
        keys = np.zeros((m, 16), dtype=np.uint8)
        nodes = np.zeros(m, dtype=np.uint32)
        ckpts = np.zeros(m, dtype=np.uint32)
        rc = lib().ckpt_record_dump(self._h, keys.ctypes.data, nodes.ctypes.data, ckpts.ctypes.data, m,
                                    ctypes.byref(cnt))
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_record_dump")
        k = cnt.value
        rows = np.empty((k, 3), dtype=np.uint64)
        rows[:, :2] = keys[:k].view(np.uint64)
        rows[:, 2] = (ckpts[:k].astype(np.uint64) << np.uint64(32)) | nodes[:k]
        return rows[np.lexsort((rows[:, 2], rows[:, 1], rows[:, 0]))]

    def set_profiling(self, level: int | bool = 2) -> None:
        """0/False off; 1 = CUDA events around K1 and the whole call only (keeps the
        kernels' programmatic early launch, so this is the level to time under); 2/True =
        events around every phase."""
        level = 2 if level is True else (0 if level is False else int(level))
        rc = lib().ckpt_set_profiling(self._h, level)
        if rc != CKPT_OK:
            raise CkptError(rc, "ckpt_set_profiling")

    PHASES = ["leaf_hash", "insert", "phase2", "phase3", "compact", "total",
              "host_pre", "host_enqueue", "host_sync_wait", "host_post", "host_table_growth", "host_arena_growth"]

    def phase_times(self, cid: int | None = None) -> dict:
        """Per-phase device times (ms) of checkpoint cid (default: the latest), measured with
        CUDA events on the caller's stream when profiling is on; host times for the latest."""
        t = (ctypes.c_float * 12)()
        if cid is None:
            lib().ckpt_phase_times(self._h, t, 12)
        else:
            rc = lib().ckpt_phase_times_of(self._h, cid, t, 12)
            if rc != CKPT_OK:
                raise CkptError(rc, "ckpt_phase_times_of")
        return {self.PHASES[i]: t[i] for i in range(12)}

    @property
    def host_syncs(self) -> int:
        """Host waits on the device this handle has performed so far (ckpt_host_syncs)."""
        c = ctypes.c_uint64()
        lib().ckpt_host_syncs(self._h, ctypes.byref(c))
        return c.value

    @property
    def kernel_launches(self) -> int:
        """Kernels this handle has enqueued so far (counted at the library's launch sites)."""
        c = ctypes.c_uint64()
        lib().ckpt_kernel_launches(self._h, ctypes.byref(c))
        return c.value

    def close(self) -> None:
        if getattr(self, "_h", None):
            lib().ckpt_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
