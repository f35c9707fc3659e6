"""Seeded synthetic input generators (frames with planted faces, the face template, the
Table I Haar feature space).  Input generation only: no pyramid, integral-image, feature or
cascade arithmetic lives here.  Serves both the CPU oracle and the CUDA path.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libfdgen.so")
_SRC = os.path.join(_HERE, "fdgen.c")
_lock = threading.Lock()
_lib = None

MAX_FACES = 32


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", _SRC,
                               "-o", _SO + ".tmp"])
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(_SO)
            P = C.c_void_p
            L.fdgen_splitmix64.restype = C.c_uint64
            L.fdgen_splitmix64.argtypes = [C.c_uint64]
            L.fdgen_frame_seed.restype = C.c_uint64
            L.fdgen_frame_seed.argtypes = [C.c_uint32, C.c_uint64]
            L.fdgen_template.argtypes = [P]
            L.fdgen_background.restype = C.c_int
            L.fdgen_background.argtypes = [C.c_uint32, C.c_uint64, C.c_int, C.c_int, C.c_int, P]
            L.fdgen_render_face.argtypes = [P, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int]
            L.fdgen_frames.restype = C.c_int
            L.fdgen_frames.argtypes = [C.c_uint32, C.c_uint64, C.c_int, C.c_int, C.c_int, C.c_int, P,
                                       C.c_int, P, P, P, C.c_int, C.c_int, C.c_double, P, P, C.c_int,
                                       C.c_int]
            _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def splitmix64(x: int) -> int:
    return int(_load().fdgen_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def template() -> np.ndarray:
    """The 24x24 face-like template (values 20 / 235)."""
    t = np.zeros((24, 24), np.uint8)
    _load().fdgen_template(_p(t))
    return t


def background(cfg: int, frame_index: int, W: int, H: int) -> np.ndarray:
    out = np.zeros((H, W), np.uint8)
    if _load().fdgen_background(cfg, frame_index, W, H, W, _p(out)) != 0:
        raise MemoryError("fdgen: background")
    return out


def render_face(frame: np.ndarray, X: int, Y: int, S: int) -> None:
    assert frame.dtype == np.uint8 and frame.flags.c_contiguous
    H, W = frame.shape
    _load().fdgen_render_face(_p(frame), W, H, W, X, Y, S)


def frames(cfg: int, first: int, n: int, W: int, H: int, levels=None, *, faces: str = "none",
           face_param: float = 0.0, max_face_level: int = 1000, nthreads: int | None = None,
           out: np.ndarray | None = None):
    """n frames with global indices first..first+n-1.

    levels: list of (f_k, W_k, H_k[, ...]) from the caller's pyramid plan, used only to put
    planted faces on a level's window grid.  faces: "none" | "fixed" (face_param faces) |
    "poisson" (Poisson(face_param) faces).  Returns (frames u8[n,H,W], faces list per frame of
    (level, wx, wy, X, Y, S) tuples).
    """
    L = _load()
    if out is None:
        out = np.empty((n, H, W), np.uint8)
    assert out.shape == (n, H, W) and out.dtype == np.uint8 and out.flags.c_contiguous
    mode = {"none": 0, "fixed": 1, "poisson": 2}[faces]
    if levels is None or mode == 0:
        levels = []
        mode = 0
    nl = len(levels)
    f = np.array([lv[0] for lv in levels] or [1.0], np.float64)
    wk = np.array([lv[1] for lv in levels] or [0], np.int32)
    hk = np.array([lv[2] for lv in levels] or [0], np.int32)
    fb = np.zeros((n, MAX_FACES, 6), np.int32)
    nfb = np.zeros(n, np.int32)
    nth = nthreads or min(32, os.cpu_count() or 1)
    rc = L.fdgen_frames(cfg, first, n, W, H, W, _p(out), nl, _p(f), _p(wk), _p(hk), max_face_level, mode,
                        float(face_param), _p(fb), _p(nfb), MAX_FACES, nth)
    if rc != 0:
        raise MemoryError("fdgen: frames")
    planted = [[tuple(int(v) for v in fb[i, j]) for j in range(nfb[i])] for i in range(n)]
    return out, planted


# ---- Table I feature space: positions 1.., cells >= 2 px ----

def _spans(ncell: int):
    """(start, cell) pairs along one axis of the 24-px window for an ncell-cell pattern."""
    out = []
    for a in range(2, 24):
        size = ncell * a
        for x in range(1, 24 - size + 1):
            out.append((x, a))
    return out


def _spans1():
    return [(x, s) for s in range(2, 24) for x in range(1, 24 - s + 1)]


def table1_counts():
    """Counts of the four Haar families enumerated by table1_features()."""
    s2, s3, s1 = len(_spans(2)), len(_spans(3)), len(_spans1())
    return {"edge": 2 * s2 * s1, "line": 2 * s3 * s1, "center": s3 * s3, "diagonal": s2 * s2}


def table1_feature(family: str, index: int):
    """The index-th feature of a family as a list of (x, y, w, h, wt) rects (Lienhart form:
    -1 x whole + k x part so every family sums to 0 on a constant window; Fig. 4)."""
    s2, s3, s1 = _spans(2), _spans(3), _spans1()
    if family == "edge":
        o, i = divmod(index, len(s2) * len(s1))
        (x, a), (y, h) = s2[i // len(s1)], s1[i % len(s1)]
        if o == 0:   # two cells side by side along x
            return [(x, y, 2 * a, h, -1), (x, y, a, h, 2)]
        return [(y, x, h, 2 * a, -1), (y, x, h, a, 2)]       # transposed: cells along y
    if family == "line":
        o, i = divmod(index, len(s3) * len(s1))
        (x, a), (y, h) = s3[i // len(s1)], s1[i % len(s1)]
        if o == 0:
            return [(x, y, 3 * a, h, -1), (x + a, y, a, h, 3)]
        return [(y, x, h, 3 * a, -1), (y, x + a, h, a, 3)]
    if family == "center":
        (x, a), (y, b) = s3[index // len(s3)], s3[index % len(s3)]
        return [(x, y, 3 * a, 3 * b, -1), (x + a, y + b, a, b, 9)]
    if family == "diagonal":
        (x, a), (y, b) = s2[index // len(s2)], s2[index % len(s2)]
        return [(x, y, 2 * a, 2 * b, -1), (x, y, a, b, 2), (x + a, y + b, a, b, 2)]
    raise ValueError(family)
