"""The C-ABI library builds for sm_100a, loads on a machine without a GPU and exports
exactly the functions include/ckpt.h declares (no compute calls here)."""
import ctypes
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared():
    src = open(os.path.join(ROOT, "include", "ckpt.h")).read()
    return sorted(set(re.findall(r"CKPT_API\s+(?:const\s+)?\w+\*?\s+\*?(ckpt_\w+)\s*\(", src)))


def test_library_exports_header_symbols():
    from paper_conf_icpp_tanlmtmbctn23_b200 import _build, ckpt
    _build.build()
    path = _build.lib_path("libckpt.so")
    L = ctypes.CDLL(path)          # loads without libcuda / libcudart (static runtime)
    names = declared()
    assert len(names) >= 13
    for nm in names:
        assert hasattr(L, nm), nm
    assert sorted(ckpt.ABI_FUNCTIONS) == names
    out = subprocess.check_output(["nm", "-D", "--defined-only", path], text=True)
    exported = sorted(ln.split()[-1] for ln in out.splitlines() if " T " in ln)
    assert exported == names       # nothing else leaks out of the shared object


def test_strerror_and_create_without_gpu():
    from paper_conf_icpp_tanlmtmbctn23_b200 import ckpt
    assert ckpt.strerror(0) == "ok"
    assert "collision" in ckpt.strerror(6)
    h = ctypes.c_void_p()
    assert ckpt.lib().ckpt_create(40, ctypes.byref(h)) == ckpt.CKPT_EINVAL   # argument check first
    assert ckpt.lib().ckpt_create_mode(128, 3, ctypes.byref(h)) == ckpt.CKPT_EINVAL   # unknown method


def test_kernels_are_sm100a_with_tma_and_128bit_cas():
    from paper_conf_icpp_tanlmtmbctn23_b200 import _build
    path = _build.lib_path("libckpt.so")
    sass = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-sass", path], text=True)
    assert "sm_100a" in subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-lelf", path], text=True)
    assert "UTMALDG.3D" in sass and "UTMALDG.2D" in sass       # TMA tensor loads (K1)
    assert "UBLKCP" in sass                                     # bulk copy of prev digests
    assert "ATOMG.E.CAS.128" in sass                            # 128-bit key claim (record)
