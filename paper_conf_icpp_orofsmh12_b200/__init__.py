"""B200-native boosted-cascade face detection (Oro et al., ICPP 2012) -- Python binding.

A thin ctypes layer over the C ABI in ``include/fd.h`` (libfd.so, built in-tree for sm_100a).
Argument marshalling only: every step of the hot path runs in the CUDA kernels behind the
ABI.  torch is used for device memory and streams.  There is no CPU fallback: if libfd.so is
missing or cannot be loaded, importing the binding's functions raises.

Detections are returned as int32 tensors of shape [n, 10] laid out like ``fd_detection``
(frame, level, wx, wy, x, y, w, h, score-as-float-bits, aux); ``to_numpy`` turns them into a
structured numpy array with a float ``score`` field.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# FD_LIB_VARIANT=timing loads the diagnostic build libfd_timing.so (same ABI + K2 phase counters)
_SO = os.path.join(_PKG, f"libfd_{os.environ['FD_LIB_VARIANT']}.so" if os.environ.get("FD_LIB_VARIANT") else "libfd.so")
_lock = threading.Lock()
_lib = None

FD_OK, FD_EINVAL, FD_EFORMAT, FD_ECAPACITY, FD_ECUDA, FD_ENOMEM = range(6)
FD_MAX_LEVELS = 128
DET_DTYPE = np.dtype([("frame", "<i4"), ("level", "<i4"), ("wx", "<i4"), ("wy", "<i4"),
                      ("x", "<i4"), ("y", "<i4"), ("w", "<i4"), ("h", "<i4"),
                      ("score", "<f4"), ("aux", "<i4")])


class FDError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"fd status {status}: {msg}")
        self.status = status


class FDCapacityError(FDError):
    def __init__(self, status: int, msg: str, required: int):
        super().__init__(status, msg)
        self.required = required


class _Plan(C.Structure):
    _fields_ = [("n_levels", C.c_int32), ("f", C.c_double * FD_MAX_LEVELS),
                ("w", C.c_int32 * FD_MAX_LEVELS), ("h", C.c_int32 * FD_MAX_LEVELS),
                ("windows", C.c_int64 * FD_MAX_LEVELS), ("total_windows", C.c_int64)]


K_NAMES = ["colsum", "carry", "band", "cascade", "sort", "dets", "group", "pyramid", "tail", "deep", "depth_hist",
           "level"]


class _Profile(C.Structure):
    _fields_ = [("launches", C.c_int64 * len(K_NAMES)), ("ms", C.c_double * len(K_NAMES))]


def library_path() -> str:
    return _SO


def lib():
    """Load libfd.so (raises if it was not built: no fallback path exists)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(_SO):
                raise ImportError(f"{_SO} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
            L = C.CDLL(_SO)
            P, i32, i64, dbl, sz = C.c_void_p, C.c_int, C.c_int64, C.c_double, C.c_size_t
            L.fd_last_error.restype = C.c_char_p
            L.fd_abi_version.restype = i32
            L.fd_load_cascade.argtypes = [C.c_char_p, sz, C.POINTER(P)]
            L.fd_free_cascade.argtypes = [P]
            L.fd_cascade_info.argtypes = [P, C.POINTER(C.c_int32), C.POINTER(C.c_int32)]
            L.fd_pyramid_plan.argtypes = [i32, i32, i32, dbl, i32, C.POINTER(_Plan)]
            L.fd_build_pyramid.argtypes = [P, i32, i32, i32, i32, i32, dbl, P, P]
            L.fd_integral.argtypes = [P, i32, i32, i32, i32, P, P, i32, P]
            L.fd_detect.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, P, i64, C.POINTER(i64), P]
            L.fd_detect_ex.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, P, i64, C.POINTER(i64), P, P]
            L.fd_detect_depth.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, P, P, P]
            L.fd_detect_host.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, P, i64, C.POINTER(i64), P]
            L.fd_group.argtypes = [P, i64, dbl, i32, P, i64, C.POINTER(i64), P]
            L.fd_release_workspaces.argtypes = []
            L.fd_detect_group_host.argtypes = [P, P, i32, i32, i32, i32, i32, dbl, i32, dbl, i32, P, i64,
                                               C.POINTER(i64), C.POINTER(i64), P]
            L.fd_depth_histogram.argtypes = [P, i32, i32, i32, i32, dbl, i32, i32, P, P]
            L.fd_profile_reset.argtypes = [i32]
            L.fd_profile_read.argtypes = [C.POINTER(_Profile)]
            for fn in ("fd_load_cascade", "fd_free_cascade", "fd_cascade_info", "fd_pyramid_plan",
                       "fd_build_pyramid", "fd_integral", "fd_detect", "fd_detect_ex", "fd_detect_depth",
                       "fd_detect_host", "fd_group", "fd_release_workspaces", "fd_detect_group_host",
                       "fd_profile_reset", "fd_profile_read", "fd_depth_histogram"):
                getattr(L, fn).restype = i32
            _lib = L
    return _lib


def _check(st: int, required: int | None = None):
    if st == FD_OK:
        return
    msg = lib().fd_last_error().decode(errors="replace")
    if st == FD_ECAPACITY:
        raise FDCapacityError(st, msg, required if required is not None else -1)
    raise FDError(st, msg)


def _torch():
    import torch
    return torch


def _stream(stream):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


def _ptr(t) -> C.c_void_p:
    return C.c_void_p(t.data_ptr())


def _frames_arg(frames):
    """frames: uint8 CUDA tensor [n, H, W] (row stride = pitch) or [H, W]."""
    torch = _torch()
    if frames.dim() == 2:
        frames = frames.unsqueeze(0)
    if frames.dtype != torch.uint8 or not frames.is_cuda:
        raise TypeError("frames must be a uint8 CUDA tensor [n, H, W]")
    n, H, W = frames.shape
    if frames.stride(2) != 1 or frames.stride(0) != H * frames.stride(1):
        frames = frames.contiguous()
    return frames, int(n), int(H), int(W), int(frames.stride(1))


class Cascade:
    """An fd_cascade handle (parsed .fdc, uploaded to the current device)."""

    def __init__(self, text: str | bytes):
        b = text.encode() if isinstance(text, str) else bytes(text)
        h = C.c_void_p()
        _check(lib().fd_load_cascade(b, len(b), C.byref(h)))
        self._h = h
        ns, nst = C.c_int32(), C.c_int32()
        _check(lib().fd_cascade_info(h, C.byref(ns), C.byref(nst)))
        self.n_stages, self.n_stumps = int(ns.value), int(nst.value)
        self.stage_sizes = _stage_sizes(b)

    @classmethod
    def from_file(cls, path: str) -> "Cascade":
        with open(path, "rb") as fh:
            return cls(fh.read())

    @property
    def handle(self):
        return self._h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.fd_free_cascade(h)
            self._h = None


def _stage_sizes(b: bytes):
    out = []
    for line in b.decode().splitlines():
        t = line.split()
        if t and t[0] == "stage":
            out.append(int(t[1]))
    return out


def fd_load_cascade(text) -> Cascade:
    return Cascade(text)


def fd_pyramid_plan(W: int, H: int, min_size: int = 24, scale_factor: float = 1.1, step: int = 1):
    """List of (f_k, W_k, H_k, windows_k)."""
    p = _Plan()
    _check(lib().fd_pyramid_plan(W, H, min_size, float(scale_factor), step, C.byref(p)))
    return [(p.f[k], p.w[k], p.h[k], p.windows[k]) for k in range(p.n_levels)]


def fd_build_pyramid(frames, min_size: int = 24, scale_factor: float = 1.1, stream=None):
    """All pyramid levels of each frame: uint8 [n, sum_k W_k*H_k] (level-major, tight)."""
    torch = _torch()
    frames, n, H, W, pitch = _frames_arg(frames)
    plan = fd_pyramid_plan(W, H, min_size, scale_factor, 1)
    tot = sum(w * h for (_, w, h, _) in plan)
    out = torch.empty((n, max(tot, 1)), dtype=torch.uint8, device=frames.device)
    _check(lib().fd_build_pyramid(_ptr(frames), n, W, H, pitch, min_size, float(scale_factor), _ptr(out),
                                  _stream(stream)))
    return out[:, :tot]


def fd_integral(img, stream=None):
    """(ii uint32-as-int32 [n, H+1, P], sqii uint64-as-int64 [n, H+1, P]) with P = round_up(W+1, 4);
    columns >= W+1 hold the row total.  Values are bit patterns of the unsigned results."""
    torch = _torch()
    img, n, H, W, pitch = _frames_arg(img)
    P = (W + 1 + 3) & ~3
    ii = torch.empty((n, H + 1, P), dtype=torch.int32, device=img.device)
    sq = torch.empty((n, H + 1, P), dtype=torch.int64, device=img.device)
    _check(lib().fd_integral(_ptr(img), n, W, H, pitch, _ptr(ii), _ptr(sq), P, _stream(stream)))
    return ii, sq


def fd_detect(casc: Cascade, frames, min_size: int = 24, scale_factor: float = 1.1, step: int = 1,
              capacity: int | None = None, stage_counts=None, stream=None):
    """Detections [n_det, 10] int32 on the frames' device, sorted (frame, level, wy, wx).
    stage_counts: optional int64 CUDA tensor [n_stages+1] that is ADDED to."""
    torch = _torch()
    frames, n, H, W, pitch = _frames_arg(frames)
    cap = int(capacity) if capacity is not None else max(4096, 64 * n)
    while True:
        out = torch.empty((max(cap, 1), 10), dtype=torch.int32, device=frames.device)
        cnt = C.c_int64()
        sc = _ptr(stage_counts) if stage_counts is not None else C.c_void_p(0)
        st = lib().fd_detect_ex(casc.handle, _ptr(frames), n, W, H, pitch, min_size, float(scale_factor), step,
                                _ptr(out), cap, C.byref(cnt), sc, _stream(stream))
        if st == FD_ECAPACITY and capacity is None:
            cap = int(cnt.value)
            if stage_counts is not None:
                raise FDError(st, "capacity retry would double-count stage_counts; pass capacity")
            continue
        _check(st, int(cnt.value))
        return out[: cnt.value]


def fd_detect_depth(casc: Cascade, frames, min_size: int = 24, scale_factor: float = 1.1, step: int = 1,
                    stream=None):
    """Per-window (depth uint8, score float32), flat [n * windows_per_frame], layout
    [frame][level][wy/step][wx/step]."""
    torch = _torch()
    frames, n, H, W, pitch = _frames_arg(frames)
    tot = sum(p[3] for p in fd_pyramid_plan(W, H, min_size, scale_factor, step)) * n
    depth = torch.empty(max(tot, 1), dtype=torch.uint8, device=frames.device)
    score = torch.empty(max(tot, 1), dtype=torch.float32, device=frames.device)
    _check(lib().fd_detect_depth(casc.handle, _ptr(frames), n, W, H, pitch, min_size, float(scale_factor), step,
                                 _ptr(depth), _ptr(score), _stream(stream)))
    return depth[:tot], score[:tot]


def fd_depth_histogram(depth, n_frames: int, W: int, H: int, n_stages: int, min_size: int = 24,
                       scale_factor: float = 1.1, step: int = 1, stream=None):
    """Fig. 7 analytics of an fd_detect_depth map: int64 [n_levels, n_stages + 1], entry [k, d] =
    windows of level k (over the n_frames) whose depth is d."""
    torch = _torch()
    assert depth.dtype == torch.uint8 and depth.is_cuda and depth.is_contiguous()
    levels = len(fd_pyramid_plan(W, H, min_size, scale_factor, step))
    hist = torch.zeros((max(levels, 1), n_stages + 1), dtype=torch.int64, device=depth.device)
    _check(lib().fd_depth_histogram(_ptr(depth), n_frames, W, H, min_size, float(scale_factor), step, n_stages,
                                    _ptr(hist), _stream(stream)))
    return hist[:levels]


def fd_detect_host(casc: Cascade, frames, min_size: int = 24, scale_factor: float = 1.1, step: int = 1,
                   capacity: int = 1 << 16, out=None, stream=None):
    """End-to-end call with HOST buffers (numpy array or CPU tensor, pinned is faster):
    returns a structured numpy array of detections."""
    torch = _torch()
    if isinstance(frames, np.ndarray):
        frames = torch.from_numpy(np.ascontiguousarray(frames))
    if frames.dim() == 2:
        frames = frames.unsqueeze(0)
    assert frames.dtype == torch.uint8 and not frames.is_cuda and frames.is_contiguous()
    n, H, W = frames.shape
    if out is None:
        out = np.empty(capacity, DET_DTYPE)
    cnt = C.c_int64()
    st = lib().fd_detect_host(casc.handle, _ptr(frames), int(n), int(W), int(H), int(W), min_size,
                              float(scale_factor), step, out.ctypes.data_as(C.c_void_p), len(out), C.byref(cnt),
                              _stream(stream))
    _check(st, int(cnt.value))
    return out[: cnt.value]


def fd_group(dets, eyes_thresh: float = 0.5, min_neighbors: int = 1, capacity: int | None = None, stream=None):
    """Grouped detections [m, 10] int32 (frame-sorted input as produced by fd_detect)."""
    torch = _torch()
    assert dets.dtype == torch.int32 and dets.is_cuda and dets.dim() == 2 and dets.shape[1] == 10
    dets = dets.contiguous()
    n = dets.shape[0]
    cap = int(capacity) if capacity is not None else max(n, 1)
    out = torch.empty((max(cap, 1), 10), dtype=torch.int32, device=dets.device)
    cnt = C.c_int64()
    _check(lib().fd_group(_ptr(dets), n, float(eyes_thresh), min_neighbors, _ptr(out), cap, C.byref(cnt),
                          _stream(stream)), None)
    return out[: cnt.value]


def fd_detect_group_host(casc: Cascade, frames, min_size: int = 24, scale_factor: float = 1.1, step: int = 1,
                         eyes_thresh: float = 0.5, min_neighbors: int = 1, capacity: int = 1 << 16, out=None,
                         stream=None):
    """End-to-end detect + group with HOST buffers.  Returns (grouped structured array, n_raw)."""
    torch = _torch()
    if isinstance(frames, np.ndarray):
        frames = torch.from_numpy(np.ascontiguousarray(frames))
    if frames.dim() == 2:
        frames = frames.unsqueeze(0)
    assert frames.dtype == torch.uint8 and not frames.is_cuda and frames.is_contiguous()
    n, H, W = frames.shape
    if out is None:
        out = np.empty(capacity, DET_DTYPE)
    cnt, raw = C.c_int64(), C.c_int64()
    st = lib().fd_detect_group_host(casc.handle, _ptr(frames), int(n), int(W), int(H), int(W), min_size,
                                    float(scale_factor), step, float(eyes_thresh), int(min_neighbors),
                                    out.ctypes.data_as(C.c_void_p), len(out), C.byref(cnt), C.byref(raw),
                                    _stream(stream))
    _check(st, int(cnt.value))
    return out[: cnt.value], int(raw.value)


def fd_profile_reset(time_kernels: bool = False):
    _check(lib().fd_profile_reset(1 if time_kernels else 0))


def fd_profile_read() -> dict:
    """{kernel: (launches, ms)} since the last fd_profile_reset."""
    p = _Profile()
    _check(lib().fd_profile_read(C.byref(p)))
    return {K_NAMES[k]: (int(p.launches[k]), float(p.ms[k])) for k in range(len(K_NAMES))}


def fd_release_workspaces():
    _check(lib().fd_release_workspaces())


def to_numpy(dets) -> np.ndarray:
    """[n, 10] int32 tensor -> structured numpy array (DET_DTYPE)."""
    a = np.ascontiguousarray(dets.detach().cpu().numpy().astype(np.int32, copy=False))
    return a.view(DET_DTYPE).reshape(-1)
