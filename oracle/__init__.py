"""CPU oracle for the boosted-cascade face-detection hot path (Oro et al., ICPP 2012).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It wraps the plain C
oracle in ``fd_oracle.c`` (see its header for the paper citations) with numpy marshalling and
shares no code with the CUDA path in ``paper_conf_icpp_orofsmh12_b200``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "fd_oracle.c")
_lock = threading.Lock()
_lib = None

# oracle compile flags: no FMA contraction, IEEE sqrtf
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-pthread"]

DET_DTYPE = np.dtype([("frame", "<i4"), ("level", "<i4"), ("wx", "<i4"), ("wy", "<i4"),
                      ("x", "<i4"), ("y", "<i4"), ("w", "<i4"), ("h", "<i4"),
                      ("score", "<f4"), ("aux", "<i4")])
RECT_DTYPE = np.dtype([("x", "<i4"), ("y", "<i4"), ("w", "<i4"), ("h", "<i4"), ("wt", "<i4")])


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (the checker; building it is not using it)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", _SO + ".tmp", "-lm"])
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(_SO)
            P = C.c_void_p
            i32, i64, dbl, f32 = C.c_int, C.c_int64, C.c_double, C.c_float
            L.fdo_cascade_parse.restype = P
            L.fdo_cascade_parse.argtypes = [C.c_char_p, C.c_size_t, C.c_char_p, i32]
            L.fdo_cascade_free.argtypes = [P]
            L.fdo_plan.restype = i32
            L.fdo_plan.argtypes = [i32, i32, i32, dbl, i32, i32, P, P, P, P]
            L.fdo_resample.argtypes = [P, i32, i32, i32, dbl, i32, i32, P]
            L.fdo_integral.argtypes = [P, i32, i32, i32, P, P]
            L.fdo_filter_binomial.argtypes = [P, i32, i32]
            L.fdo_rect_sum.restype = C.c_uint32
            L.fdo_rect_sum.argtypes = [P, i32, i32, i32, i32, i32]
            L.fdo_window_nf.restype = f32
            L.fdo_window_nf.argtypes = [P, P, i32, i32, i32]
            L.fdo_feature.restype = C.c_int32
            L.fdo_feature.argtypes = [P, i32, i32, i32, P, i32]
            L.fdo_feature_values.argtypes = [P, i32, P, i64, P, i32, P]
            L.fdo_window_nf_values.argtypes = [P, P, i32, P, i64, P]
            L.fdo_eval_window.restype = i32
            L.fdo_eval_window.argtypes = [P, P, P, i32, i32, i32, P, P]
            L.fdo_eval_level.argtypes = [P, P, P, i32, i32, i32, P, P, P]
            L.fdo_detect.restype = i64
            L.fdo_detect.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, i32, P, i64, P]
            L.fdo_detect_depth.restype = i32
            L.fdo_detect_depth.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, i32, P, P, P]
            L.fdo_group.restype = i64
            L.fdo_group.argtypes = [P, i64, dbl, i32, P, i64]
            L.fdo_s_eyes.restype = dbl
            L.fdo_s_eyes.argtypes = [dbl] * 8
            L.fdo_half_bits.restype = C.c_int32
            L.fdo_half_bits.argtypes = [f32]
            L.fdo_half_value.restype = f32
            L.fdo_half_value.argtypes = [C.c_uint16]
            L.fdo_pack16.restype = i32
            L.fdo_pack16.argtypes = [P, P]
            L.fdo_unpack16.restype = i32
            L.fdo_unpack16.argtypes = [P, i32, P]
            L.fdo_cascade_words.restype = i64
            L.fdo_cascade_words.argtypes = [P, P, i64]
            _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


class _CascadeC(C.Structure):
    _fields_ = [("win_w", C.c_int32), ("win_h", C.c_int32), ("n_stages", C.c_int32),
                ("n_stumps", C.c_int32), ("filter", C.c_int32), ("soft", C.c_int32),
                ("packed", C.c_int32), ("words", C.c_void_p), ("n_words", C.c_int64),
                ("stages", C.c_void_p), ("stumps", C.c_void_p)]


class Cascade:
    """A parsed .fdc cascade (the oracle's own parser)."""

    def __init__(self, text: str | bytes):
        L = _load()
        b = text.encode() if isinstance(text, str) else bytes(text)
        err = C.create_string_buffer(512)
        h = L.fdo_cascade_parse(b, len(b), err, 512)
        if not h:
            raise ValueError("oracle: bad cascade: " + err.value.decode())
        self._h = h
        s = C.cast(h, C.POINTER(_CascadeC)).contents
        self.n_stages = int(s.n_stages)
        self.n_stumps = int(s.n_stumps)

    @classmethod
    def from_file(cls, path: str) -> "Cascade":
        with open(path, "rb") as fh:
            return cls(fh.read())

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.fdo_cascade_free(h)
            self._h = None


def plan(W: int, H: int, min_size: int = 24, scale: float = 1.1, step: int = 1):
    """c1: list of (f_k, W_k, H_k, windows_k)."""
    L = _load()
    f = np.zeros(128, np.float64)
    wk = np.zeros(128, np.int32)
    hk = np.zeros(128, np.int32)
    nw = np.zeros(128, np.int64)
    n = L.fdo_plan(W, H, min_size, float(scale), step, 128, _p(f), _p(wk), _p(hk), _p(nw))
    if n < 0:
        raise ValueError("oracle: bad plan arguments")
    return [(float(f[k]), int(wk[k]), int(hk[k]), int(nw[k])) for k in range(n)]


def resample(frame: np.ndarray, f: float, Wk: int, Hk: int) -> np.ndarray:
    """c2: level image sampled from the frame."""
    frame = np.ascontiguousarray(frame, dtype=np.uint8)
    H, W = frame.shape
    out = np.zeros((Hk, Wk), np.uint8)
    _load().fdo_resample(_p(frame), W, H, W, float(f), Wk, Hk, _p(out))
    return out


def filter_binomial(img: np.ndarray) -> np.ndarray:
    """f2 filtering stage (reading R3b): 3x3 binomial / 16, round half up, clamp-to-edge."""
    out = np.array(img, dtype=np.uint8, order="C", copy=True)
    H, W = out.shape
    _load().fdo_filter_binomial(_p(out), W, H)
    return out


def integral(img: np.ndarray):
    """c3: (ii uint32 (H+1, W+1), sqii uint64 (H+1, W+1))."""
    img = np.ascontiguousarray(img, dtype=np.uint8)
    H, W = img.shape
    ii = np.zeros((H + 1, W + 1), np.uint32)
    sq = np.zeros((H + 1, W + 1), np.uint64)
    _load().fdo_integral(_p(img), W, H, W, _p(ii), _p(sq))
    return ii, sq


def rect_sum(ii: np.ndarray, x: int, y: int, w: int, h: int) -> int:
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    return int(_load().fdo_rect_sum(_p(ii), ii.shape[1], x, y, w, h))


def window_nf(ii, sq, wx: int, wy: int) -> float:
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    sq = np.ascontiguousarray(sq, dtype=np.uint64)
    return float(np.float32(_load().fdo_window_nf(_p(ii), _p(sq), ii.shape[1], wx, wy)))


def _rects(rects) -> np.ndarray:
    return np.array([tuple(int(v) for v in r) for r in rects], dtype=RECT_DTYPE)


def feature(ii, wx: int, wy: int, rects) -> int:
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    r = _rects(rects)
    return int(_load().fdo_feature(_p(ii), ii.shape[1], wx, wy, _p(r), len(r)))


def feature_values(ii, wins: np.ndarray, rects) -> np.ndarray:
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    wins = np.ascontiguousarray(wins, dtype=np.int32).reshape(-1, 2)
    r = _rects(rects)
    out = np.zeros(len(wins), np.int32)
    _load().fdo_feature_values(_p(ii), ii.shape[1], _p(wins), len(wins), _p(r), len(r), _p(out))
    return out


def window_nf_values(ii, sq, wins: np.ndarray) -> np.ndarray:
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    sq = np.ascontiguousarray(sq, dtype=np.uint64)
    wins = np.ascontiguousarray(wins, dtype=np.int32).reshape(-1, 2)
    out = np.zeros(len(wins), np.float32)
    _load().fdo_window_nf_values(_p(ii), _p(sq), ii.shape[1], _p(wins), len(wins), _p(out))
    return out


def eval_window(casc: Cascade, ii, sq, wx: int, wy: int):
    """c7/c8: (depth, score, near_flags) of one window."""
    ii = np.ascontiguousarray(ii, dtype=np.uint32)
    sq = np.ascontiguousarray(sq, dtype=np.uint64)
    sc = C.c_float()
    nr = C.c_int()
    d = _load().fdo_eval_window(casc._h, _p(ii), _p(sq), ii.shape[1], wx, wy, C.byref(sc), C.byref(nr))
    return int(d), float(np.float32(sc.value)), int(nr.value)


def _frames(frames: np.ndarray) -> np.ndarray:
    frames = np.ascontiguousarray(frames, dtype=np.uint8)
    if frames.ndim == 2:
        frames = frames[None]
    return frames


def detect(casc: Cascade, frames: np.ndarray, min_size: int = 24, scale: float = 1.1, step: int = 1,
           nthreads: int = 1):
    """c1..c9 over frames u8[n, H, W]; returns (detections sorted (frame, level, wy, wx), n_near)."""
    L = _load()
    frames = _frames(frames)
    n, H, W = frames.shape
    nn = C.c_int64()
    cnt = L.fdo_detect(casc._h, _p(frames), n, W, H, W, min_size, float(scale), step, nthreads, None, 0,
                       C.byref(nn))
    if cnt < 0:
        raise ValueError("oracle: detect failed")
    out = np.zeros(cnt, DET_DTYPE)
    if cnt:
        cnt2 = L.fdo_detect(casc._h, _p(frames), n, W, H, W, min_size, float(scale), step, nthreads,
                            _p(out), cnt, C.byref(nn))
        assert cnt2 == cnt
    return out, int(nn.value)


def detect_depth(casc: Cascade, frames: np.ndarray, min_size: int = 24, scale: float = 1.1, step: int = 1,
                 nthreads: int = 1):
    """Per-window (depth u8, score f32, near u8), flat over [frame][level][wy][wx]."""
    frames = _frames(frames)
    n, H, W = frames.shape
    tot = sum(p[3] for p in plan(W, H, min_size, scale, step)) * n
    depth = np.zeros(tot, np.uint8)
    score = np.zeros(tot, np.float32)
    near = np.zeros(tot, np.uint8)
    rc = _load().fdo_detect_depth(casc._h, _p(frames), n, W, H, W, min_size, float(scale), step, nthreads,
                                  _p(depth), _p(score), _p(near))
    if rc != 0:
        raise ValueError("oracle: detect_depth failed")
    return depth, score, near


def depth_histogram(depth: np.ndarray, n_frames: int, W: int, H: int, n_stages: int, min_size: int = 24,
                    scale: float = 1.1, step: int = 1) -> np.ndarray:
    """Fig. 7: for every scale k, how many windows (over all frames)
    reached depth d -- "the distribution of the deepest stage reached ... for each considered
    scale".  Plain definition: split each frame's depth map at the level window counts and count
    each depth value (np.bincount).  int64 [levels, n_stages + 1]; depths above n_stages count
    into the last bin."""
    counts = [p[3] for p in plan(W, H, min_size, scale, step)]
    per = sum(counts)
    d = np.minimum(np.asarray(depth, np.int64).reshape(n_frames, per), n_stages)
    out = np.zeros((len(counts), n_stages + 1), np.int64)
    off = 0
    for k, c in enumerate(counts):
        for f in range(n_frames):
            out[k] += np.bincount(d[f, off:off + c], minlength=n_stages + 1)
        off += c
    return out


def group(dets: np.ndarray, eyes_thresh: float = 0.5, min_neighbors: int = 1) -> np.ndarray:
    """c10: greedy S_eyes grouping per frame (input sorted by frame)."""
    L = _load()
    dets = np.ascontiguousarray(dets, dtype=DET_DTYPE)
    cnt = L.fdo_group(_p(dets), len(dets), float(eyes_thresh), min_neighbors, None, 0)
    out = np.zeros(max(cnt, 0), DET_DTYPE)
    if cnt > 0:
        L.fdo_group(_p(dets), len(dets), float(eyes_thresh), min_neighbors, _p(out), cnt)
    return out


class _RectC(C.Structure):
    _fields_ = [("x", C.c_int32), ("y", C.c_int32), ("w", C.c_int32), ("h", C.c_int32), ("wt", C.c_int32)]


class _StumpC(C.Structure):
    _fields_ = [("nrect", C.c_int32), ("r", _RectC * 3), ("theta", C.c_float), ("left", C.c_float),
                ("right", C.c_float)]


def half_bits(v: float) -> int:
    """f3 (R13): IEEE binary16 bits of v, or -1 if v is not exactly a finite binary16 value."""
    return int(_load().fdo_half_bits(float(v)))


def half_value(h: int) -> float:
    return float(np.float32(_load().fdo_half_value(int(h))))


def pack16(rects, theta, left, right):
    """f3 (R13): a stump -> its compressed words (list of uint16), or None."""
    s = _StumpC()
    s.nrect = len(rects)
    for i, (x, y, w, h, wt) in enumerate(rects):
        s.r[i] = _RectC(x, y, w, h, wt)
    s.theta, s.left, s.right = float(theta), float(left), float(right)
    out = (C.c_uint16 * 9)()
    n = _load().fdo_pack16(C.byref(s), out)
    return None if n < 0 else [int(v) for v in out[:n]]


def unpack16(words, nrect):
    """f3: compressed words -> (rects, theta, left, right)."""
    arr = (C.c_uint16 * len(words))(*words)
    s = _StumpC()
    _load().fdo_unpack16(arr, nrect, C.byref(s))
    rects = [(s.r[i].x, s.r[i].y, s.r[i].w, s.r[i].h, s.r[i].wt) for i in range(nrect)]
    return rects, float(np.float32(s.theta)), float(np.float32(s.left)), float(np.float32(s.right))


def cascade_words(casc: "Cascade") -> np.ndarray:
    """The compressed word stream of a 'compress packed16' cascade (empty otherwise)."""
    L = _load()
    n = L.fdo_cascade_words(casc._h, None, 0)
    out = np.zeros(max(n, 0), np.uint16)
    if n > 0:
        L.fdo_cascade_words(casc._h, _p(out), n)
    return out


def s_eyes(a, b) -> float:
    """eq. 6 between rects a=(x,y,w,h), b=(x,y,w,h)."""
    return float(_load().fdo_s_eyes(*[float(v) for v in a], *[float(v) for v in b]))
