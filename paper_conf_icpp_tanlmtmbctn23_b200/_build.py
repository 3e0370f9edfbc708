"""In-tree build of the sm_100a shared libraries (nvcc; no JIT cache, no pip install).

libckpt.so    — the product: csrc/*.cu behind include/ckpt.h (C ABI)
libckptgen.so — harness: device twins of the seeded workload generators
"""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden",
                "-shared", "-cudart", "static", "-I", os.path.join(ROOT, "include")]

LIBS = {
    "libckpt.so": sorted(glob.glob(os.path.join(PKG, "csrc", "*.cu"))),
    "libckptgen.so": [os.path.join(PKG, "workloads", "gen.cu")],
}
DEPS = {
    "libckpt.so": sorted(glob.glob(os.path.join(PKG, "csrc", "*.cu*")) + glob.glob(os.path.join(PKG, "csrc", "*.h"))
                         + [os.path.join(ROOT, "include", "ckpt.h")]),
    "libckptgen.so": [os.path.join(PKG, "workloads", "gen.cu")],
}


def lib_path(name: str) -> str:
    return os.path.join(PKG, name)


def build(force: bool = False, verbose: bool = False) -> list[str]:
    out = []
    for name, srcs in LIBS.items():
        path = lib_path(name)
        fresh = os.path.exists(path) and all(os.path.getmtime(d) <= os.path.getmtime(path) for d in DEPS[name])
        if force or not fresh:
            cmd = [NVCC] + FLAGS + (["-Xptxas", "-v"] if verbose else []) + ["-o", path] + srcs
            subprocess.check_call(cmd)
        out.append(path)
    return out


def build_variant(name: str, defines: list[str]) -> str:
    """An experiment build of libckpt.so with extra -D flags (selected with CKPT_LIB)."""
    path = lib_path(name)
    cmd = [NVCC] + FLAGS + [f"-D{d}" for d in defines] + ["-o", path] + LIBS["libckpt.so"]
    subprocess.check_call(cmd)
    return path


if __name__ == "__main__":
    import sys
    for p in build(force="-f" in sys.argv, verbose="-v" in sys.argv):
        print(p)
