"""ctypes binding of the PCIAM oracle (liboracle.so, built from oracle.c with gcc).

TEST INFRASTRUCTURE ONLY: only tests/, ``__graft_entry__.smoke()`` and
``bench.py``'s cpu_baseline / ``--impl reference`` leg may import this package.
The CUDA product path (``paper_conf_icpp_blattnerkcsbz14_b200``) never does.

See oracle.c's header for the paper passages each function follows and the
readings (C1-C10) it takes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

PAIR_DTYPE = np.dtype([
    ("dx", np.int32), ("dy", np.int32), ("ccf", np.float64), ("candidate", np.int32),
    ("peak_x", np.int32), ("peak_y", np.int32), ("peak", np.float64),
    ("runner_up", np.float64), ("ccf_k", np.float64, (4,)), ("max_imag_ratio", np.float64),
], align=True)


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain C11, -O2, no fast-math, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-shared", "-fPIC", "-pthread",
                               "-fno-fast-math", _SRC, "-o", _LIB, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    lib = ctypes.CDLL(_LIB)
    vp, ci = ctypes.c_void_p, ctypes.c_int
    lib.oracle_dft.argtypes = [vp, vp, ci, ci]
    lib.oracle_dft.restype = None
    lib.oracle_dft2.argtypes = [vp, vp, ci, ci, ci]
    lib.oracle_dft2.restype = None
    lib.oracle_fft2_u16.argtypes = [vp, ci, ci, vp]
    lib.oracle_fft2_u16.restype = None
    lib.oracle_ccf.argtypes = [vp, vp, ci, ci, ci, ci, ctypes.POINTER(ci)]
    lib.oracle_ccf.restype = ctypes.c_double
    lib.oracle_ccf_moments.argtypes = [vp, vp, ci, ci, ci, ci, vp, ctypes.POINTER(ci)]
    lib.oracle_ccf_moments.restype = ctypes.c_double
    lib.oracle_eval_peak.argtypes = [vp, vp, ci, ci, ci, ci, vp]
    lib.oracle_eval_peak.restype = None
    lib.oracle_pciam.argtypes = [vp, vp, ci, ci, vp]
    lib.oracle_pciam.restype = None
    lib.oracle_surface.argtypes = [vp, vp, ci, ci, vp]
    lib.oracle_surface.restype = None
    lib.oracle_grid.argtypes = [vp, ci, ci, ci, ci, ci, vp, vp]
    lib.oracle_grid.restype = ci
    lib.oracle_pair_size.restype = ci
    if lib.oracle_pair_size() != PAIR_DTYPE.itemsize:
        raise RuntimeError("oracle_pair layout mismatch")
    _lib = lib
    return lib


def _c(a: np.ndarray, dtype) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=dtype)


def dft(x: np.ndarray, inverse: bool = False) -> np.ndarray:
    """1-D DFT (forward e^{-i}, inverse e^{+i} unnormalised) by the oracle's mixed-radix code."""
    x = _c(np.asarray(x, np.complex128), np.complex128)
    out = np.empty_like(x)
    _load().oracle_dft(x.ctypes.data, out.ctypes.data, x.size, -1 if inverse else 1)
    return out


def dft2(x: np.ndarray, inverse: bool = False) -> np.ndarray:
    x = _c(np.asarray(x, np.complex128), np.complex128)
    out = np.empty_like(x)
    H, W = x.shape
    _load().oracle_dft2(x.ctypes.data, out.ctypes.data, H, W, -1 if inverse else 1)
    return out


def fft2_u16(img: np.ndarray) -> np.ndarray:
    """Step 2: full C2C forward transform of a uint16 tile, complex128 [H][W]."""
    img = _c(img, np.uint16)
    H, W = img.shape
    out = np.empty((H, W), np.complex128)
    _load().oracle_fft2_u16(img.ctypes.data, H, W, out.ctypes.data)
    return out


def ccf(A: np.ndarray, B: np.ndarray, dx: int, dy: int):
    """Fig. 3 CCF of region A[dy:H, dx:W] vs B[0:H-dy, 0:W-dx]; returns (value, valid)."""
    A = _c(A, np.uint16); B = _c(B, np.uint16)
    H, W = A.shape
    v = ctypes.c_int(0)
    c = _load().oracle_ccf(A.ctypes.data, B.ctypes.data, H, W, int(dx), int(dy), ctypes.byref(v))
    return c, bool(v.value)


def ccf_moments(A: np.ndarray, B: np.ndarray, dx: int, dy: int):
    """Integer-moment CCF (cross-check); returns (value, valid, moments[6])."""
    A = _c(A, np.uint16); B = _c(B, np.uint16)
    H, W = A.shape
    v = ctypes.c_int(0)
    mom = np.zeros(6, np.uint64)
    c = _load().oracle_ccf_moments(A.ctypes.data, B.ctypes.data, H, W, int(dx), int(dy),
                                   mom.ctypes.data, ctypes.byref(v))
    return c, bool(v.value), mom


def eval_peak(A: np.ndarray, B: np.ndarray, x: int, y: int) -> np.void:
    """Steps 6-7 (Fig. 2 l.8-12) from a given peak (x, y)."""
    A = _c(A, np.uint16); B = _c(B, np.uint16)
    H, W = A.shape
    out = np.zeros(1, PAIR_DTYPE)
    _load().oracle_eval_peak(A.ctypes.data, B.ctypes.data, H, W, int(x), int(y), out.ctypes.data)
    return out[0]


def pciam(A: np.ndarray, B: np.ndarray) -> np.void:
    """Fig. 2 pciam(A, B), steps 2-7, A = west/north neighbour, B = tile (reading C1)."""
    A = _c(A, np.uint16); B = _c(B, np.uint16)
    H, W = A.shape
    out = np.zeros(1, PAIR_DTYPE)
    _load().oracle_pciam(A.ctypes.data, B.ctypes.data, H, W, out.ctypes.data)
    return out[0]


def surface(A: np.ndarray, B: np.ndarray) -> np.ndarray:
    """|Re iFFT2(NCC)| / (HW), the normalised correlation surface (test helper)."""
    A = _c(A, np.uint16); B = _c(B, np.uint16)
    H, W = A.shape
    out = np.empty((H, W), np.float64)
    _load().oracle_surface(A.ctypes.data, B.ctypes.data, H, W, out.ctypes.data)
    return out


def grid(tiles: np.ndarray, threads: int | None = None):
    """Fig. 4: (west, north) result arrays [n, m] of PAIR_DTYPE for a uint16 [n, m, H, W] grid."""
    tiles = _c(tiles, np.uint16)
    n, m, H, W = tiles.shape
    west = np.zeros(n * m, PAIR_DTYPE)
    north = np.zeros(n * m, PAIR_DTYPE)
    if threads is None:
        threads = os.cpu_count() or 1
    rc = _load().oracle_grid(tiles.ctypes.data, n, m, H, W, threads, west.ctypes.data,
                             north.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_grid rejected its arguments")
    return west.reshape(n, m), north.reshape(n, m)
