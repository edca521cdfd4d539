"""Seeded synthetic tile grids shaped like the paper's workloads (input generator only).

This module is the one piece shared by the oracle side and the CUDA side: it
renders uint16 tiles cropped from one stateless procedural scene with known,
non-negative neighbour offsets, and holds none of the method's arithmetic.

Workloads (BASELINE.json ``configs``):
  config 1: 3x3 grid of 256x192 tiles (oracle runs in seconds)
  config 2: 18x22 grid of 1392x1040 tiles
  config 3: 42x59 grid of 1392x1040 tiles (headline)
  config 4: 161 scans x 2 channels x 18x22 (streamed: bench.py --config 4, stream.py)
  config 5: 100x100 grid of 1392x1040 tiles

Geometry: with step
``sx = W - round(ov*W)``, ``sy = H - round(ov*H)`` and jitter ``u, v in [0, delta]``,
tile (r, c) has origin ``ox = c*sx + r*delta + u(r,c)``, ``oy = r*sy + c*delta + v(r,c)``.
So a west pair (r, c-1)->(r, c) has dx in [sx-delta, sx+delta], dy in [0, 2*delta]
and a north pair (r-1, c)->(r, c) has dy in [sy-delta, sy+delta], dx in [0, 2*delta]:
all offsets are non-negative (reading C9).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

SEED = 20140909
_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_LIB = os.path.join(_HERE, "libsynth.so")
_lib = None

CONFIGS = {
    1: dict(name="3x3@256x192", n=3, m=3, H=192, W=256, overlap=0.10, delta=4),
    2: dict(name="18x22@1392x1040", n=18, m=22, H=1040, W=1392, overlap=0.10, delta=12),
    3: dict(name="42x59@1392x1040", n=42, m=59, H=1040, W=1392, overlap=0.10, delta=12),
    4: dict(name="161x2x(18x22)@1392x1040", n=18, m=22, H=1040, W=1392, overlap=0.10, delta=12,
            scans=161, channels=2),
    5: dict(name="100x100@1392x1040", n=100, m=100, H=1040, W=1392, overlap=0.10, delta=12),
}


def build(force: bool = False) -> str:
    """Compile libsynth.so with gcc (plain C, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-std=c11", "-pthread",
                               _SRC, "-o", _LIB])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.synth_tiles.restype = ctypes.c_int
        lib.synth_tiles.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                    ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_void_p]
        lib.synth_tiles_tex.restype = ctypes.c_int
        lib.synth_tiles_tex.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_uint32, ctypes.c_void_p]
        lib.synth_jitter.restype = ctypes.c_int64
        lib.synth_jitter.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                     ctypes.c_int64]
        _lib = lib
    return _lib


def _round_half_up(x: float) -> int:
    return int(np.floor(x + 0.5))


@dataclass
class Grid:
    tiles: np.ndarray      # uint16 [n, m, H, W], row-major, W contiguous
    origins: np.ndarray    # int64 [n, m, 2] = (ox, oy) of each tile in the scene
    n: int
    m: int
    H: int
    W: int
    seed: int
    overlap: float
    delta: int

    def true_west(self):
        """(dx, dy) [n, m] of tile (r, c) in the frame of its west neighbour; row c=0 invalid."""
        o = self.origins
        d = np.zeros((self.n, self.m, 2), np.int64)
        d[:, 1:] = o[:, 1:] - o[:, :-1]
        return d[..., 0], d[..., 1]

    def true_north(self):
        """(dx, dy) [n, m] of tile (r, c) in the frame of its north neighbour; row r=0 invalid."""
        o = self.origins
        d = np.zeros((self.n, self.m, 2), np.int64)
        d[1:] = o[1:] - o[:-1]
        return d[..., 0], d[..., 1]


def origins(n: int, m: int, H: int, W: int, overlap: float = 0.10, delta: int | None = None,
            seed: int = SEED, scan: int = 0, channel: int = 0) -> np.ndarray:
    lib = _load()
    if delta is None:
        delta = 4 if W <= 512 else 12
    sx = W - _round_half_up(overlap * W)
    sy = H - _round_half_up(overlap * H)
    if not (0 < sx <= W and 0 < sy <= H):
        raise ValueError("overlap must leave a positive step")
    base = ((scan * 2 + channel) << 48)
    o = np.zeros((n, m, 2), np.int64)
    for r in range(n):
        for c in range(m):
            key = base | (r << 24) | c
            u = lib.synth_jitter(seed, key, 0x75, delta)
            v = lib.synth_jitter(seed, key, 0x76, delta)
            o[r, c, 0] = c * sx + r * delta + u
            o[r, c, 1] = r * sy + c * delta + v
    return o


def make_grid(n: int, m: int, H: int, W: int, overlap: float = 0.10, delta: int | None = None,
              seed: int = SEED, scan: int = 0, channel: int = 0, threads: int | None = None,
              out: np.ndarray | None = None, rows: tuple[int, int] | None = None,
              texture: str = "default", density: float = 0.02) -> Grid:
    """Render an n x m grid of H x W uint16 tiles (optionally only tile rows [r0, r1)).

    ``out`` may be a caller-owned (e.g. pinned) uint16 array of the right shape.
    ``texture``: "default" (value noise + per-pixel scene detail) or "cells" (the low-texture
    scene: flat background + sparse bright cells, ``density`` = occupancy per 64 px lattice
    cell, the paper's sparse early colonies).
    """
    lib = _load()
    if delta is None:
        delta = 4 if W <= 512 else 12
    o = origins(n, m, H, W, overlap, delta, seed, scan, channel)
    r0, r1 = rows if rows is not None else (0, n)
    nr = r1 - r0
    if out is None:
        out = np.empty((nr, m, H, W), np.uint16)
    if out.shape != (nr, m, H, W) or out.dtype != np.uint16 or not out.flags.c_contiguous:
        raise ValueError("out has the wrong shape/dtype/layout")
    sub = np.ascontiguousarray(o[r0:r1].reshape(-1, 2))
    base = ((scan * 2 + channel) << 48)
    keys = np.array([base | (r << 24) | c for r in range(r0, r1) for c in range(m)], np.uint64)
    tex_seed = seed + 0x9E37 * channel
    if threads is None:
        threads = os.cpu_count() or 1
    if texture not in ("default", "cells"):
        raise ValueError("texture must be 'default' or 'cells'")
    dens = int(round(density * 65536))
    if not 0 <= dens <= 65536:
        raise ValueError("density must be in [0, 1]")
    rc = lib.synth_tiles_tex(tex_seed, sub.ctypes.data, keys.ctypes.data, nr * m, H, W, threads,
                             0 if texture == "default" else 1, dens, out.ctypes.data)
    if rc != 0:
        raise RuntimeError("synth_tiles failed")
    return Grid(out, o[r0:r1], nr, m, H, W, seed, overlap, delta)


def make_config(cfg: int, **kw) -> Grid:
    c = CONFIGS[cfg]
    return make_grid(c["n"], c["m"], c["H"], c["W"], overlap=kw.pop("overlap", c["overlap"]),
                     delta=kw.pop("delta", c["delta"]), **kw)
