"""B200-native GPU Merkle-tree checkpoint de-duplication (Tan et al., ICPP'23).

The hot path lives in libckpt.so (hand-written sm_100a CUDA behind the C ABI of
include/ckpt.h); ``Checkpointer`` is its thin ctypes binding. ``workloads`` holds the
seeded synthetic input generators (harness code).
"""
from .ckpt import Checkpointer, CkptError, strerror  # noqa: F401  (library loads lazily)

__all__ = ["Checkpointer", "CkptError", "strerror"]
