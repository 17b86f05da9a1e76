"""fp64 CPU oracle for spatial-domain NCC (template matching) and PIV.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this package.
The product path (``paper_conf_ipps_moorelk13_b200``) never imports it, and the two
share no code: the oracle is ``oracle/ncc_oracle.c`` (plain C, fp64, two-pass centred
``corr2`` per window, OpenMP over offsets/windows) plus the independent FFT route in
``oracle/ncc_fft.py`` (numpy), which is used only to cross-check full surfaces.

Citations: ``/root/reference/PAPER.md`` lines ("P:a-b") -- Fig 5.1 caption P:132-137
(A-bar, B-bar matrix averages), Listing 5.1 caption P:250-251 and Tab 5.1 caption
P:190-191 (``corr2`` per shift), PIV Figs 5.8-5.12 captions P:164-171.  Where the paper
text is lost the readings of SURVEY.md section 8(c) apply (listed in DESIGN.md).

Pins: tests/test_oracle.py (closed-form hand cases, numpy.corrcoef, invariants,
brute force vs FFT, planted shifts, sub-pixel closed forms).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ncc_oracle.c")
_LIB = os.path.join(_HERE, "libncc_oracle.so")

# flag bits (interface values, see include/ncc.h)
FLAT_TEMPLATE = 1
EDGE_Y = 2
EDGE_X = 4
PARABOLA_Y = 8
PARABOLA_X = 16
INVALID = 32


def build(force: bool = False) -> str:
    """Compile the oracle shared library (gcc, -O2 -fopenmp -ffp-contract=off)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared",
             "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _PivVec(ctypes.Structure):
    _fields_ = [("iy", ctypes.c_int32), ("ix", ctypes.c_int32),
                ("dy", ctypes.c_double), ("dx", ctypes.c_double),
                ("score", ctypes.c_double), ("flags", ctypes.c_uint32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i32, i64 = ctypes.c_int, ctypes.c_int64
        _lib.oracle_ncc_surface.argtypes = [P, i32, i32, i64, P, i32, i32, i64, i32, i32, P]
        _lib.oracle_ncc_at.argtypes = [P, i32, i32, i64, P, i32, i32, i64, P, P, i32, P]
        _lib.oracle_argmax.argtypes = [P, i64]
        _lib.oracle_argmax.restype = i64
        _lib.oracle_template_is_flat.argtypes = [P, i64, i32, i32]
        _lib.oracle_subpixel3.argtypes = [ctypes.c_double] * 3 + [ctypes.POINTER(ctypes.c_int)]
        _lib.oracle_subpixel3.restype = ctypes.c_double
        _lib.oracle_subpixel3_min.argtypes = [ctypes.c_double] * 3
        _lib.oracle_subpixel3_min.restype = ctypes.c_double
        _lib.oracle_piv_grid.argtypes = [i32] * 8 + [ctypes.POINTER(ctypes.c_int)] * 2
        _lib.oracle_piv_pair.argtypes = [P, P, i32, i32, i64] + [i32] * 6 + [P, P]
        _lib.oracle_piv_windows.argtypes = [P, P, i32, i32, i64] + [i32] * 6 + [P, P, i32, P, P]
        _lib.oracle_piv_window_scores.argtypes = [P, P, i32, i32, i64] + [i32] * 8 + [P]
        _lib.oracle_num_threads.restype = i32
        _lib.oracle_set_num_threads.argtypes = [i32]
        _lib.oracle_ssd_surface.argtypes = [P, i32, i32, i64, P, i32, i32, i64, i32, i32, P]
        _lib.oracle_argmin.argtypes = [P, i64]
        _lib.oracle_argmin.restype = i64
        _lib.oracle_piv_windows_ssd.argtypes = [P, P, i32, i32, i64] + [i32] * 6 + [P, P, i32, P, P]
        _lib.oracle_sad_surface.argtypes = [P, i32, i32, i64, P, i32, i32, i64, i32, i32, P]
        _lib.oracle_piv_windows_sad.argtypes = [P, P, i32, i32, i64] + [i32] * 6 + [P, P, i32, P, P]
    return _lib


def _f32(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def set_num_threads(n: int) -> None:
    """OpenMP threads for later oracle calls (bench.py times a 1-thread rate beside the full one)."""
    lib().oracle_set_num_threads(int(n))


def ncc_surface(img: np.ndarray, tmpl: np.ndarray, u_begin: int = 0, u_end: int | None = None) -> np.ndarray:
    """corr2 at every valid offset (rows [u_begin, u_end)) -> float64 (rows, V)."""
    img, tmpl = _f32(img), _f32(tmpl)
    H, W = img.shape
    h, w = tmpl.shape
    U, V = H - h + 1, W - w + 1
    if u_end is None:
        u_end = U
    out = np.empty((u_end - u_begin, V), dtype=np.float64)
    rc = lib().oracle_ncc_surface(_ptr(img), H, W, W, _ptr(tmpl), h, w, w, u_begin, u_end, _ptr(out))
    if rc:
        raise ValueError("oracle_ncc_surface: invalid arguments")
    return out


def ncc_at(img: np.ndarray, tmpl: np.ndarray, us, vs) -> np.ndarray:
    """corr2 at the listed offsets -> float64 (count,)."""
    img, tmpl = _f32(img), _f32(tmpl)
    us = np.ascontiguousarray(us, dtype=np.int32)
    vs = np.ascontiguousarray(vs, dtype=np.int32)
    H, W = img.shape
    h, w = tmpl.shape
    out = np.empty(len(us), dtype=np.float64)
    rc = lib().oracle_ncc_at(_ptr(img), H, W, W, _ptr(tmpl), h, w, w, _ptr(us), _ptr(vs), len(us), _ptr(out))
    if rc:
        raise ValueError("oracle_ncc_at: invalid arguments")
    return out


def argmax(scores: np.ndarray) -> int:
    s = np.ascontiguousarray(scores, dtype=np.float64).ravel()
    return int(lib().oracle_argmax(_ptr(s), s.size))


def template_is_flat(tmpl: np.ndarray) -> bool:
    t = _f32(tmpl)
    return bool(lib().oracle_template_is_flat(_ptr(t), t.shape[1], t.shape[0], t.shape[1]))


@dataclass
class Peak:
    score: float
    u: int
    v: int
    valid: bool


def ncc_match(img: np.ndarray, tmpl: np.ndarray) -> tuple[np.ndarray, Peak]:
    """Full surface + peak (argmax, tie -> smallest u*V+v; invalid if template flat)."""
    s = ncc_surface(img, tmpl)
    k = argmax(s)
    V = s.shape[1]
    return s, Peak(float(s.ravel()[k]), k // V, k % V, not template_is_flat(tmpl))


def subpixel3(cm: float, c0: float, cp: float) -> tuple[float, bool]:
    par = ctypes.c_int(0)
    d = lib().oracle_subpixel3(float(cm), float(c0), float(cp), ctypes.byref(par))
    return float(d), bool(par.value)


def subpixel3_min(cm: float, c0: float, cp: float) -> float:
    """3-point parabolic fit of a minimum (SSD sub-pixel, Fig 5.10): 0 if not a minimum."""
    return float(lib().oracle_subpixel3_min(float(cm), float(c0), float(cp)))


def piv_grid(H, W, h, w, my, mx, sy, sx) -> tuple[int, int]:
    ky, kx = ctypes.c_int(), ctypes.c_int()
    if lib().oracle_piv_grid(H, W, h, w, my, mx, sy, sx, ctypes.byref(ky), ctypes.byref(kx)):
        raise ValueError("no window fits")
    return ky.value, kx.value


_PIV_DTYPE = np.dtype([("iy", np.int32), ("ix", np.int32), ("dy", np.float64), ("dx", np.float64),
                       ("score", np.float64), ("flags", np.uint32)], align=True)
assert _PIV_DTYPE.itemsize == ctypes.sizeof(_PivVec)


def piv_pair(A, B, h, w, my, mx, sy, sx) -> np.ndarray:
    """All interior windows of one pair -> structured array (Ky, Kx) of vectors."""
    A, B = _f32(A), _f32(B)
    H, W = A.shape
    Ky, Kx = piv_grid(H, W, h, w, my, mx, sy, sx)
    scratch = np.empty(Ky * Kx * (2 * my + 1) * (2 * mx + 1), dtype=np.float64)
    out = np.zeros(Ky * Kx, dtype=_PIV_DTYPE)
    rc = lib().oracle_piv_pair(_ptr(A), _ptr(B), H, W, W, h, w, my, mx, sy, sx, _ptr(scratch), _ptr(out))
    if rc:
        raise ValueError("oracle_piv_pair: invalid arguments")
    return out.reshape(Ky, Kx)


def piv_windows(A, B, h, w, my, mx, sy, sx, kys, kxs) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    H, W = A.shape
    kys = np.ascontiguousarray(kys, dtype=np.int32)
    kxs = np.ascontiguousarray(kxs, dtype=np.int32)
    n = len(kys)
    scratch = np.empty(n * (2 * my + 1) * (2 * mx + 1), dtype=np.float64)
    out = np.zeros(n, dtype=_PIV_DTYPE)
    rc = lib().oracle_piv_windows(_ptr(A), _ptr(B), H, W, W, h, w, my, mx, sy, sx,
                                  _ptr(kys), _ptr(kxs), n, _ptr(scratch), _ptr(out))
    if rc:
        raise ValueError("oracle_piv_windows: invalid arguments")
    return out


def piv_window_scores(A, B, h, w, my, mx, sy, sx, ky, kx) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    H, W = A.shape
    out = np.empty((2 * my + 1, 2 * mx + 1), dtype=np.float64)
    rc = lib().oracle_piv_window_scores(_ptr(A), _ptr(B), H, W, W, h, w, my, mx, sy, sx, ky, kx, _ptr(out))
    if rc:
        raise ValueError("oracle_piv_window_scores: invalid arguments")
    return out


# ---------------------------------------------------------------- SSD (paper's PIV metric, Fig 5.10)
def ssd_surface(img: np.ndarray, tmpl: np.ndarray, u_begin: int = 0, u_end: int | None = None) -> np.ndarray:
    img, tmpl = _f32(img), _f32(tmpl)
    H, W = img.shape
    h, w = tmpl.shape
    U, V = H - h + 1, W - w + 1
    if u_end is None:
        u_end = U
    out = np.empty((u_end - u_begin, V), dtype=np.float64)
    if lib().oracle_ssd_surface(_ptr(img), H, W, W, _ptr(tmpl), h, w, w, u_begin, u_end, _ptr(out)):
        raise ValueError("oracle_ssd_surface: invalid arguments")
    return out


def argmin(scores: np.ndarray) -> int:
    s = np.ascontiguousarray(scores, dtype=np.float64).ravel()
    return int(lib().oracle_argmin(_ptr(s), s.size))


def ssd_match(img, tmpl):
    s = ssd_surface(img, tmpl)
    k = argmin(s)
    V = s.shape[1]
    return s, Peak(float(s.ravel()[k]), k // V, k % V, True)


def piv_windows_ssd(A, B, h, w, my, mx, sy, sx, kys, kxs) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    H, W = A.shape
    kys = np.ascontiguousarray(kys, dtype=np.int32)
    kxs = np.ascontiguousarray(kxs, dtype=np.int32)
    n = len(kys)
    scratch = np.empty(n * (2 * my + 1) * (2 * mx + 1), dtype=np.float64)
    out = np.zeros(n, dtype=_PIV_DTYPE)
    if lib().oracle_piv_windows_ssd(_ptr(A), _ptr(B), H, W, W, h, w, my, mx, sy, sx,
                                    _ptr(kys), _ptr(kxs), n, _ptr(scratch), _ptr(out)):
        raise ValueError("oracle_piv_windows_ssd: invalid arguments")
    return out


# ---------------------------------------------------------------- SAD (Ch. 4 specialisation example)
def sad_surface(img: np.ndarray, tmpl: np.ndarray, u_begin: int = 0, u_end: int | None = None) -> np.ndarray:
    img, tmpl = _f32(img), _f32(tmpl)
    H, W = img.shape
    h, w = tmpl.shape
    U, V = H - h + 1, W - w + 1
    if u_end is None:
        u_end = U
    out = np.empty((u_end - u_begin, V), dtype=np.float64)
    if lib().oracle_sad_surface(_ptr(img), H, W, W, _ptr(tmpl), h, w, w, u_begin, u_end, _ptr(out)):
        raise ValueError("oracle_sad_surface: invalid arguments")
    return out


def sad_match(img, tmpl):
    s = sad_surface(img, tmpl)
    k = argmin(s)
    V = s.shape[1]
    return s, Peak(float(s.ravel()[k]), k // V, k % V, True)


def piv_windows_sad(A, B, h, w, my, mx, sy, sx, kys, kxs) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    H, W = A.shape
    kys = np.ascontiguousarray(kys, dtype=np.int32)
    kxs = np.ascontiguousarray(kxs, dtype=np.int32)
    n = len(kys)
    scratch = np.empty(n * (2 * my + 1) * (2 * mx + 1), dtype=np.float64)
    out = np.zeros(n, dtype=_PIV_DTYPE)
    if lib().oracle_piv_windows_sad(_ptr(A), _ptr(B), H, W, W, h, w, my, mx, sy, sx,
                                    _ptr(kys), _ptr(kxs), n, _ptr(scratch), _ptr(out)):
        raise ValueError("oracle_piv_windows_sad: invalid arguments")
    return out
