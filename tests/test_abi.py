"""CPU-only checks of the boundary: libfd.so loads, exports every symbol include/fd.h
declares, the host-only plan matches the oracle's, host-side validation errors (no compute)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_icpp_orofsmh12_b200 as fd

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    txt = open(os.path.join(ROOT, "include", "fd.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(fd_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    L = fd.lib()
    syms = declared_symbols()
    assert len(syms) >= 12
    for s in syms:
        assert hasattr(L, s), s
    assert L.fd_abi_version() == 3


def test_detection_struct_layout_matches_oracle():
    assert fd.DET_DTYPE.itemsize == 40
    assert fd.DET_DTYPE == oracle.DET_DTYPE


@pytest.mark.parametrize("W,H,s,step", [(320, 240, 1.25, 1), (640, 480, 1.2, 1), (1920, 1080, 1.1, 1),
                                        (1920, 1080, 1.1, 2), (3840, 2160, 1.1, 1), (100, 31, 1.07, 3),
                                        (24, 24, 1.5, 1), (25, 700, 1.01, 4)])
def test_plan_matches_oracle(W, H, s, step):
    a = fd.fd_pyramid_plan(W, H, 24, s, step)
    b = oracle.plan(W, H, 24, s, step)
    assert a == b


def test_plan_min_size():
    assert fd.fd_pyramid_plan(640, 480, 48, 1.2, 1) == oracle.plan(640, 480, 48, 1.2, 1)


@pytest.mark.parametrize("args", [(23, 240, 24, 1.1, 1), (320, 240, 23, 1.1, 1), (320, 240, 24, 1.0, 1),
                                  (320, 240, 24, 1.1, 0), (320, 240, 24, float("nan"), 1)])
def test_plan_invalid(args):
    with pytest.raises(fd.FDError) as e:
        fd.fd_pyramid_plan(*args)
    assert e.value.status == fd.FD_EINVAL


def test_too_many_levels():
    with pytest.raises(fd.FDError):
        fd.fd_pyramid_plan(60000, 60000, 24, 1.0001, 1)


def test_group_rejects_bad_args_without_gpu():
    L = fd.lib()
    cnt = C.c_int64()
    assert L.fd_group(None, 0, 0.5, 1, None, 0, C.byref(cnt), None) == fd.FD_OK and cnt.value == 0
    assert L.fd_group(None, 5, 0.5, 1, None, 0, C.byref(cnt), None) == fd.FD_EINVAL
    assert L.fd_group(None, 0, -1.0, 1, None, 0, C.byref(cnt), None) == fd.FD_EINVAL


def test_detect_rejects_null_cascade():
    L = fd.lib()
    cnt = C.c_int64()
    buf = np.zeros(16, np.uint8)
    st = L.fd_detect(None, buf.ctypes.data_as(C.c_void_p), 1, 24, 24, 24, 24, 1.1, 1, None, 0, C.byref(cnt), None)
    assert st == fd.FD_EINVAL
    assert b"cascade" in L.fd_last_error()


@pytest.mark.parametrize("name", ["c1.fdc", "c3.fdc"])
def test_specialised_k2_compiles_without_gpu(name):
    """The step-1 K2 specialised for a cascade (fd_jit.cpp) is generated and NVRTC-compiled for
    sm_100a; no device is touched."""
    L = fd.lib()
    L.fd_debug_jit_compile.argtypes = [C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]
    text = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "cascades", name), "rb").read()
    n = C.c_size_t(0)
    rc = L.fd_debug_jit_compile(text, len(text), C.byref(n))
    assert rc == 0, fd.last_error() if hasattr(fd, "last_error") else rc
    assert n.value > 100000
