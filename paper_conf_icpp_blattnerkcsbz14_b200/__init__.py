"""B200-native PCIAM tile-pair translation engine (Blattner et al., ICPP 2014, phase 1).

Thin Python binding of the C ABI in ``include/stitch.h`` (``libstitch_b200.so``):
argument marshalling only -- every step of the path runs in the library's
sm_100a kernels.  PyTorch is used for plumbing only (device workspace, the
current CUDA stream, torch.distributed in ``parallel.py``).

    from paper_conf_icpp_blattnerkcsbz14_b200 import PciamGrid
    g = PciamGrid(n, m, H, W)
    g.load_grid(tiles)                      # uint16 [n, m, H, W], host or CUDA
    west, north = g.compute_translations()  # PAIR_DTYPE [n, m] each (Fig. 4 output)

There is no CPU fallback: if the CUDA library is missing this import fails.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libstitch_b200.so")

STATUS = {0: "STITCH_OK", 1: "STITCH_ERR_INVALID_ARG", 2: "STITCH_ERR_UNSUPPORTED",
          3: "STITCH_ERR_OUT_OF_MEMORY", 4: "STITCH_ERR_CUDA", 5: "STITCH_ERR_NCCL",
          6: "STITCH_ERR_STATE"}
FLAG_NO_GRAPH = 1   # STITCH_FLAG_NO_GRAPH: direct launches instead of a replayed CUDA graph
FLAG_SERIAL = 2     # STITCH_FLAG_SERIAL: one stream for every kernel

# stitch_pair (include/stitch.h), 64 bytes
PAIR_DTYPE = np.dtype([
    ("dx", np.int32), ("dy", np.int32), ("ccf", np.float64), ("candidate", np.int32),
    ("peak_x", np.int32), ("peak_y", np.int32), ("peak", np.float32), ("ccf_k", np.float64, (4,)),
], align=True)
assert PAIR_DTYPE.itemsize == 64

# Tile sizes with a compiled FFT plan (stitch_api.cu plan table)
SUPPORTED_TILES = {(1392, 1040), (256, 192), (48, 40), (58, 26)}


class StitchError(RuntimeError):
    def __init__(self, status: int, msg: str = ""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {msg}")


class Config(ctypes.Structure):
    _fields_ = [("tile_width", ctypes.c_int32), ("tile_height", ctypes.c_int32),
                ("grid_rows", ctypes.c_int32), ("grid_cols", ctypes.c_int32),
                ("device", ctypes.c_int32), ("tile_begin", ctypes.c_int32),
                ("tile_end", ctypes.c_int32), ("chunk_pairs", ctypes.c_int32),
                ("chunk_tiles", ctypes.c_int32), ("precision", ctypes.c_int32),
                ("stream", ctypes.c_void_p), ("workspace", ctypes.c_void_p),
                ("workspace_bytes", ctypes.c_size_t), ("pool_tiles", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("world_size", ctypes.c_int32),
                ("nccl_id", ctypes.c_void_p), ("flags", ctypes.c_uint32)]


EXPORTS = ["stitch_status_string", "stitch_workspace_size", "stitch_pair_count", "stitch_init",
           "stitch_load_grid", "stitch_load_grid_device", "stitch_compute_translations_async",
           "stitch_compute_translations", "stitch_get_translations", "stitch_forward_async",
           "stitch_debug_spectrum", "stitch_synchronize", "stitch_last_counts",
           "stitch_last_timings", "stitch_set_timing", "stitch_last_error", "stitch_destroy",
           "stitch_load_tiles", "stitch_resident_range", "stitch_kernel_timings",
           "stitch_forward_range_async", "stitch_spectra_range", "stitch_pairs_async",
           "stitch_global_positions", "stitch_compose_overlay", "stitch_debug_spectrum_f64",
           "stitch_compute_translations_from_host_async", "stitch_timeline",
           "stitch_nccl_unique_id", "stitch_pairs_part_async", "stitch_debug_surface",
           "stitch_compose_overlay_async"]

_lib = None


def load_library():
    """Load libstitch_b200.so (raises if it has not been built: no fallback path)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                          "(python -m paper_conf_icpp_blattnerkcsbz14_b200.build)")
    lib = ctypes.CDLL(LIB_PATH)
    P, vp, i32, i64 = ctypes.POINTER, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    C = P(Config)
    sig = {
        "stitch_status_string": (ctypes.c_char_p, [ctypes.c_int]),
        "stitch_nccl_unique_id": (ctypes.c_int, [vp]),
        "stitch_pairs_part_async": (ctypes.c_int, [vp, i32]),
        "stitch_debug_surface": (ctypes.c_int, [vp, i32, i32, vp]),
        "stitch_workspace_size": (ctypes.c_int, [C, P(ctypes.c_size_t)]),
        "stitch_pair_count": (ctypes.c_int, [C, P(i64)]),
        "stitch_init": (ctypes.c_int, [C, P(vp)]),
        "stitch_load_grid": (ctypes.c_int, [vp, vp, ctypes.c_size_t]),
        "stitch_load_grid_device": (ctypes.c_int, [vp, vp, ctypes.c_size_t]),
        "stitch_compute_translations_async": (ctypes.c_int, [vp]),
        "stitch_compute_translations": (ctypes.c_int, [vp, vp, vp]),
        "stitch_get_translations": (ctypes.c_int, [vp, vp, vp]),
        "stitch_forward_async": (ctypes.c_int, [vp]),
        "stitch_debug_spectrum": (ctypes.c_int, [vp, i32, vp]),
        "stitch_debug_spectrum_f64": (ctypes.c_int, [vp, i32, vp]),
        "stitch_compute_translations_from_host_async": (ctypes.c_int, [vp, vp, i32, i32]),
        "stitch_timeline": (ctypes.c_int, [vp, vp, vp, vp, vp, i64, P(i64)]),
        "stitch_synchronize": (ctypes.c_int, [vp]),
        "stitch_last_counts": (ctypes.c_int, [vp, P(i64), P(i64), P(i64)]),
        "stitch_last_timings": (ctypes.c_int, [vp, P(ctypes.c_float)]),
        "stitch_set_timing": (ctypes.c_int, [vp, ctypes.c_int]),
        "stitch_last_error": (ctypes.c_char_p, [vp]),
        "stitch_destroy": (None, [vp]),
        "stitch_load_tiles": (ctypes.c_int, [vp, vp, i32, i32, i32]),
        "stitch_resident_range": (ctypes.c_int, [vp, P(i32), P(i32), P(i32)]),
        "stitch_kernel_timings": (ctypes.c_int, [vp, P(ctypes.c_float), P(i64)]),
        "stitch_forward_range_async": (ctypes.c_int, [vp, i32, i32]),
        "stitch_spectra_range": (ctypes.c_int, [vp, i32, i32, P(vp), P(ctypes.c_size_t)]),
        "stitch_pairs_async": (ctypes.c_int, [vp]),
        "stitch_global_positions": (ctypes.c_int, [i32, i32, vp, vp, vp, vp]),
        "stitch_compose_overlay": (ctypes.c_int, [vp, i32, i32, i32, i32, vp, i64, i64, vp, vp]),
        "stitch_compose_overlay_async": (ctypes.c_int,
                                         [vp, i32, i32, i32, i32, vp, i64, i64, vp, vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def make_config(n, m, H, W, device=0, tile_begin=0, tile_end=0, chunk_pairs=0, chunk_tiles=0,
                stream=None, workspace=None, workspace_bytes=0, precision=0, pool_tiles=0,
                rank=0, world_size=1, nccl_id=None, flags=0) -> Config:
    """precision: 0 = fp32 transforms (default), 1 = fp64; pool_tiles > 0: the
    bounded mode (row f1); nccl_id: 128 bytes from nccl_unique_id() (in-library halo exchange)."""
    return Config(W, H, n, m, device, tile_begin, tile_end, chunk_pairs, chunk_tiles, precision,
                  stream, workspace, workspace_bytes, pool_tiles, rank, world_size, nccl_id, flags)


def nccl_unique_id() -> bytes:
    """A fresh 128-byte NCCL unique id (rank 0; broadcast it to the other ranks)."""
    buf = ctypes.create_string_buffer(128)
    st = load_library().stitch_nccl_unique_id(buf)
    if st:
        raise StitchError(st, "stitch_nccl_unique_id")
    return buf.raw


def workspace_size(cfg: Config) -> int:
    b = ctypes.c_size_t(0)
    st = load_library().stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b))
    if st:
        raise StitchError(st, "stitch_workspace_size")
    return b.value


def pair_count(cfg: Config) -> int:
    c = ctypes.c_int64(0)
    st = load_library().stitch_pair_count(ctypes.byref(cfg), ctypes.byref(c))
    if st:
        raise StitchError(st, "stitch_pair_count")
    return c.value


def global_positions(west: np.ndarray, north: np.ndarray):
    """Phase 2 (f3): absolute tile origins [n, m, 2] (x, y) from the translations, and the
    maximum-spanning-tree parent of each tile (-1 at a root).  Host-only C code."""
    n, m = west.shape
    w = np.ascontiguousarray(west.reshape(-1), dtype=PAIR_DTYPE)
    nn = np.ascontiguousarray(north.reshape(-1), dtype=PAIR_DTYPE)
    pos = np.zeros((n * m, 2), np.int64)
    parent = np.zeros(n * m, np.int32)
    st = load_library().stitch_global_positions(n, m, w.ctypes.data, nn.ctypes.data,
                                                pos.ctypes.data, parent.ctypes.data)
    if st:
        raise StitchError(st, "stitch_global_positions")
    return pos.reshape(n, m, 2), parent.reshape(n, m)


def compose_overlay(tiles, pos_xy: np.ndarray, canvas=None, sync: bool = True):
    """Phase 3 (f4): overlay-blend composite of a device tile grid (torch CUDA uint16
    [n, m, H, W]) at integer origins pos_xy [n, m, 2]; returns the torch canvas.
    sync=False: stream-ordered on torch's current stream (stitch_compose_overlay_async)."""
    import torch
    n, m, H, W = tiles.shape
    p = np.ascontiguousarray(pos_xy.reshape(-1, 2), dtype=np.int64)
    p = p - p.min(axis=0)
    cw, ch = int(p[:, 0].max()) + W, int(p[:, 1].max()) + H
    if canvas is None:
        canvas = torch.zeros((ch, cw), dtype=torch.uint16, device=tiles.device)
    name = "stitch_compose_overlay" if sync else "stitch_compose_overlay_async"
    st = getattr(load_library(), name)(
        tiles.data_ptr(), n, m, H, W, p.ctypes.data, cw, ch, canvas.data_ptr(),
        torch.cuda.current_stream(tiles.device).cuda_stream)
    if st:
        raise StitchError(st, name)
    return canvas


class PciamGrid:
    """One context over an n x m grid of H x W uint16 tiles (or the row band
    [tile_begin, tile_end) of it, for multi-GPU row-band partitioning).

    pool_tiles > 0 selects the bounded mode: a fixed pool of tile slots recycled
    by reference count; tiles then arrive through compute_from_host_async.  rank / world_size /
    nccl_id: the in-library NCCL halo exchange (the library derives the rank's band)."""

    def __init__(self, n: int, m: int, H: int, W: int, device: int = 0, tile_begin: int = 0,
                 tile_end: int = 0, chunk_pairs: int = 0, chunk_tiles: int = 0,
                 use_torch: bool = True, precision: int = 0, pool_tiles: int = 0,
                 rank: int = 0, world_size: int = 1, nccl_id: bytes | None = None,
                 flags: int = 0):
        self.lib = load_library()
        self.n, self.m, self.H, self.W = n, m, H, W
        self.device = device
        self._ctx = ctypes.c_void_p(None)
        self._ws = None
        self.precision = precision
        self._nccl_id = ctypes.create_string_buffer(nccl_id, 128) if nccl_id is not None else None
        cfg = make_config(n, m, H, W, device, tile_begin, tile_end, chunk_pairs, chunk_tiles,
                          precision=precision, pool_tiles=pool_tiles, rank=rank,
                          world_size=world_size,
                          nccl_id=ctypes.cast(self._nccl_id, ctypes.c_void_p) if nccl_id else None,
                          flags=flags)
        self.stream = None
        if use_torch:
            import torch
            dev = torch.device("cuda", device)
            cur = torch.cuda.current_stream(dev)
            # The context enqueues on a real torch stream: the caller's current one, or --
            # if that is the legacy default stream -- a dedicated one.  Record timing events
            # and order other torch work against `self.stream`.
            self.stream = cur if cur.cuda_stream != 0 else torch.cuda.Stream(dev)
            nbytes = workspace_size(cfg)
            self._ws = torch.empty(nbytes, dtype=torch.uint8, device=dev)
            cfg.stream = self.stream.cuda_stream
            cfg.workspace = self._ws.data_ptr()
            cfg.workspace_bytes = nbytes
            # the workspace was allocated on the current stream: order the context after it
            self._after_torch()
        self.cfg = cfg
        self.npairs = pair_count(cfg)
        self._check(self.lib.stitch_init(ctypes.byref(cfg), ctypes.byref(self._ctx)), "init")
        hb, tb, te = self.resident_range()
        self.halo_begin, self.tile_begin, self.tile_end = hb, tb, te

    def _check(self, st: int, what: str):
        if st:
            msg = self.lib.stitch_last_error(self._ctx).decode() if self._ctx else ""
            raise StitchError(st, f"{what}: {msg}")

    def _after_torch(self, tensor=None) -> None:
        """Order the context stream after torch's current stream (where `tensor` was written)
        and tell torch's allocator the context stream uses `tensor`."""
        import torch
        cur = torch.cuda.current_stream(torch.device("cuda", self.device))
        if self.stream is not None and cur.cuda_stream != self.stream.cuda_stream:
            self.stream.wait_stream(cur)
        if tensor is not None and tensor.is_cuda and self.stream is not None:
            tensor.record_stream(self.stream)

    # -- step 1: load --------------------------------------------------------
    def load_grid(self, tiles) -> None:
        """tiles: uint16 [n, m, H, W] numpy array (host) or torch tensor (host or CUDA)."""
        nbytes = self.n * self.m * self.H * self.W * 2
        if isinstance(tiles, np.ndarray):
            if tiles.dtype != np.uint16 or not tiles.flags.c_contiguous or tiles.nbytes != nbytes:
                raise ValueError("tiles must be a C-contiguous uint16 [n, m, H, W] array")
            self._check(self.lib.stitch_load_grid(self._ctx, tiles.ctypes.data, nbytes), "load")
            return
        import torch
        if tiles.dtype != torch.uint16 or not tiles.is_contiguous() or \
                tiles.numel() * 2 != nbytes:
            raise ValueError("tiles must be a contiguous torch.uint16 [n, m, H, W] tensor")
        if tiles.is_cuda:
            self._after_torch(tiles)
            self._keep = tiles
            self._check(self.lib.stitch_load_grid_device(self._ctx, tiles.data_ptr(), nbytes),
                        "load")
        else:
            self._check(self.lib.stitch_load_grid(self._ctx, tiles.data_ptr(), nbytes), "load")

    def resident_range(self) -> tuple[int, int, int]:
        """(halo_begin, tile_begin, tile_end): tiles this context keeps in HBM."""
        a, b, c = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        self._check(self.lib.stitch_resident_range(self._ctx, ctypes.byref(a), ctypes.byref(b),
                                                   ctypes.byref(c)), "range")
        return a.value, b.value, c.value

    def load_tiles(self, tiles, first_tile: int) -> None:
        """Load a run of consecutive tiles starting at `first_tile` (numpy or torch, [k, H, W]
        or [rows, m, H, W]) covering resident_range()."""
        count = (tiles.size if isinstance(tiles, np.ndarray) else tiles.numel()) // (self.H * self.W)
        if isinstance(tiles, np.ndarray):
            if tiles.dtype != np.uint16 or not tiles.flags.c_contiguous:
                raise ValueError("tiles must be C-contiguous uint16")
            ptr, dev = tiles.ctypes.data, 0
        else:
            import torch
            if tiles.dtype != torch.uint16 or not tiles.is_contiguous():
                raise ValueError("tiles must be a contiguous torch.uint16 tensor")
            ptr, dev = tiles.data_ptr(), int(tiles.is_cuda)
            if dev:
                self._after_torch(tiles)
                self._keep = tiles
        self._check(self.lib.stitch_load_tiles(self._ctx, ptr, first_tile, count, dev), "load")

    def compute_from_host_async(self, tiles, first_tile: int = 0) -> None:
        """Steps 1-7 with the host-to-device copy pipelined under the transforms: `tiles` is a
        HOST run of consecutive tiles from `first_tile` (numpy or pinned torch CPU tensor,
        [k, H, W] or [rows, m, H, W]) covering resident_range().  Keep it alive and unmodified
        until get_translations() / synchronize()."""
        if isinstance(tiles, np.ndarray):
            if tiles.dtype != np.uint16 or not tiles.flags.c_contiguous:
                raise ValueError("tiles must be C-contiguous uint16")
            ptr, count = tiles.ctypes.data, tiles.size // (self.H * self.W)
        else:
            if tiles.is_cuda or not tiles.is_contiguous() or tiles.element_size() != 2:
                raise ValueError("tiles must be a contiguous 16-bit host tensor")
            ptr, count = tiles.data_ptr(), tiles.numel() // (self.H * self.W)
        self._keep = tiles
        self._check(self.lib.stitch_compute_translations_from_host_async(self._ctx, ptr,
                                                                         first_tile, count),
                    "compute from host")

    # -- steps 2-7 -------------------------------------------------------------
    def compute_translations_async(self) -> None:
        self._check(self.lib.stitch_compute_translations_async(self._ctx), "compute")

    def forward_async(self) -> None:
        self._check(self.lib.stitch_forward_async(self._ctx), "forward")

    def forward_range_async(self, first_tile: int, count: int) -> None:
        """Step 2 for resident tiles [first_tile, first_tile + count) (global indices)."""
        self._check(self.lib.stitch_forward_range_async(self._ctx, first_tile, count), "forward")

    def pairs_async(self, part: int = 0) -> None:
        """Steps 3-7 (spectra already resident) for part 0 = every pair of the context,
        1 = the interior pairs (tile A owned), 2 = the boundary pairs (tile A in the halo)."""
        self._check(self.lib.stitch_pairs_part_async(self._ctx, int(part)), "pairs")

    def spectra_range(self, first_tile: int, count: int) -> tuple[int, int]:
        """(device address, bytes) of the resident spectra of tiles [first_tile, +count)."""
        ptr, nbytes = ctypes.c_void_p(), ctypes.c_size_t()
        self._check(self.lib.stitch_spectra_range(self._ctx, first_tile, count, ctypes.byref(ptr),
                                                  ctypes.byref(nbytes)), "spectra range")
        return ptr.value or 0, nbytes.value

    def spectra_view(self, first_tile: int, count: int):
        """The resident spectra of a tile range as a uint8 view of the torch workspace
        (for torch.distributed send/recv); requires the torch workspace."""
        if self._ws is None:
            raise RuntimeError("spectra_view needs the torch workspace (use_torch=True)")
        ptr, nbytes = self.spectra_range(first_tile, count)
        off = ptr - self._ws.data_ptr()
        return self._ws[off: off + nbytes]

    def get_translations(self, west: np.ndarray | None = None, north: np.ndarray | None = None):
        """Copy the last compute's results out: (west, north) PAIR_DTYPE arrays [n, m].  Caller
        arrays (to merge several band contexts) must be C-contiguous PAIR_DTYPE of n*m entries;
        only the owned tiles' entries are written."""
        nt = self.n * self.m
        if west is None:
            west = np.zeros(nt, PAIR_DTYPE)
        if north is None:
            north = np.zeros(nt, PAIR_DTYPE)
        for a in (west, north):
            if not isinstance(a, np.ndarray) or a.dtype != PAIR_DTYPE or a.size != nt or \
                    not a.flags.c_contiguous or not a.flags.writeable:
                raise ValueError(f"result arrays must be writeable C-contiguous PAIR_DTYPE "
                                 f"arrays of n*m = {nt} entries")
        self._check(self.lib.stitch_get_translations(self._ctx, west.ctypes.data,
                                                     north.ctypes.data), "get")
        return west.reshape(self.n, self.m), north.reshape(self.n, self.m)

    def compute_translations(self):
        """Fig. 4: (west, north) arrays of PAIR_DTYPE, shape [n, m] (owned tiles filled)."""
        west = np.zeros(self.n * self.m, PAIR_DTYPE)
        north = np.zeros(self.n * self.m, PAIR_DTYPE)
        self._check(self.lib.stitch_compute_translations(self._ctx, west.ctypes.data,
                                                         north.ctypes.data), "compute")
        return west.reshape(self.n, self.m), north.reshape(self.n, self.m)

    def spectrum(self, tile: int) -> np.ndarray:
        """Half spectrum of a tile, [H, W//2 + 1], complex64 (fp32 context) or complex128
        (fp64 context), recomputed by the context's forward kernels (test hook)."""
        if self.precision:
            out = np.empty((self.H, self.W // 2 + 1), np.complex128)
            self._check(self.lib.stitch_debug_spectrum_f64(self._ctx, tile, out.ctypes.data),
                        "spectrum")
            return out
        out = np.empty((self.H, self.W // 2 + 1), np.complex64)
        self._check(self.lib.stitch_debug_spectrum(self._ctx, tile, out.ctypes.data), "spectrum")
        return out

    def surface(self, tile: int, kind: int) -> np.ndarray:
        """Test hook (reading C11): the normalised correlation surface |iFFT2(NCC)|/(HW),
        float32 [H, W], of the (kind 0 west / 1 north) pair of `tile`, computed by the step's
        K3 + K4 transforms from the last computed spectra."""
        out = np.empty((self.H, self.W), np.float32)
        self._check(self.lib.stitch_debug_surface(self._ctx, int(tile), int(kind),
                                                  out.ctypes.data), "surface")
        return out

    def synchronize(self) -> None:
        self._check(self.lib.stitch_synchronize(self._ctx), "synchronize")

    def last_counts(self) -> dict:
        a, b, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        self._check(self.lib.stitch_last_counts(self._ctx, ctypes.byref(a), ctypes.byref(b),
                                                ctypes.byref(c)), "counts")
        return {"launches": a.value, "forward_ffts": b.value, "pairs": c.value}

    def set_timing(self, mode: int) -> None:
        """0 off, 1 per-stage events, 2 per-stage + per-launch events, 3 timeline."""
        self._check(self.lib.stitch_set_timing(self._ctx, int(mode)), "timing")

    def kernel_timings(self) -> dict:
        """Mode-2 per-kernel (K1..K6) summed device ms and launch counts of the last compute."""
        ms = (ctypes.c_float * 6)()
        cnt = (ctypes.c_int64 * 6)()
        self._check(self.lib.stitch_kernel_timings(self._ctx, ms, cnt), "kernel timings")
        names = ["k1_fwd_rows", "k2_fwd_cols", "k3_pair_cols", "k4_pair_rows",
                 "k5_ccf_moments", "k6_finalize"]
        return {n: {"ms": ms[i], "launches": cnt[i]} for i, n in enumerate(names)}

    def timeline(self) -> dict:
        """Timing-mode-3 launch timeline of the last compute: arrays kernel (0..5 = K1..K6),
        stream (0 forward, 1 pairs, 2 CCF), start_ms, end_ms (from the step's start)."""
        cnt = ctypes.c_int64(0)
        self._check(self.lib.stitch_timeline(self._ctx, None, None, None, None, 0,
                                             ctypes.byref(cnt)), "timeline")
        k = np.zeros(cnt.value, np.int32)
        st = np.zeros(cnt.value, np.int32)
        a = np.zeros(cnt.value, np.float32)
        b = np.zeros(cnt.value, np.float32)
        self._check(self.lib.stitch_timeline(self._ctx, k.ctypes.data, st.ctypes.data,
                                             a.ctypes.data, b.ctypes.data, cnt.value,
                                             ctypes.byref(cnt)), "timeline")
        return {"kernel": k, "stream": st, "start_ms": a, "end_ms": b}

    def last_timings(self) -> dict:
        ms = (ctypes.c_float * 4)()
        self._check(self.lib.stitch_last_timings(self._ctx, ms), "timings")
        return {"forward_ms": ms[0], "pairs_ms": ms[1], "ccf_ms": ms[2], "total_ms": ms[3]}

    def close(self) -> None:
        if self._ctx:
            self.lib.stitch_destroy(self._ctx)
            self._ctx = ctypes.c_void_p(None)
        self._ws = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
