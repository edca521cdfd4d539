"""CPU-only checks of the C-ABI library and host logic (no compute calls, no GPU needed).

  * libstitch_b200.so loads and exports every function include/stitch.h declares;
  * host-only entry points: status strings, config validation, workspace size,
    Table I pair counts, row-band pair ownership;
  * the generated DFT codelets (csrc/codelets.cuh) evaluate, on the host, to the
    DFT definition (the arithmetic the kernels execute, checked symbolically).
"""
import ctypes
import math
import os
import re

import numpy as np
import pytest

import __graft_entry__
import paper_conf_icpp_blattnerkcsbz14_b200 as pkg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    __graft_entry__.build()
    return pkg.load_library()


def header_functions():
    src = open(os.path.join(ROOT, "include", "stitch.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(stitch_[a-z_0-9]+)\s*\(", src)))


def test_exports_every_declared_symbol(lib):
    names = header_functions()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(pkg.EXPORTS) == names


def test_status_strings(lib):
    assert lib.stitch_status_string(0) == b"ok"
    assert b"unsupported" in lib.stitch_status_string(2)


def test_config_validation(lib):
    ctx = ctypes.c_void_p()
    assert lib.stitch_init(None, ctypes.byref(ctx)) == 1
    cfg = pkg.make_config(3, 3, 191, 256)            # no plan for 256x191
    assert lib.stitch_init(ctypes.byref(cfg), ctypes.byref(ctx)) == 2
    cfg = pkg.make_config(0, 3, 192, 256)
    assert lib.stitch_init(ctypes.byref(cfg), ctypes.byref(ctx)) == 1
    cfg = pkg.make_config(3, 3, 192, 256, tile_begin=5, tile_end=4)
    b = ctypes.c_size_t()
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 1
    lib.stitch_destroy(None)  # NULL-safe


@pytest.mark.parametrize("n,m", [(3, 3), (18, 22), (42, 59), (100, 100), (1, 1), (1, 7), (5, 1)])
def test_table1_pair_counts(lib, n, m):
    cfg = pkg.make_config(n, m, 1040, 1392)
    assert pkg.pair_count(cfg) == 2 * n * m - n - m   # Table I


@pytest.mark.parametrize("R", [2, 3, 4, 8])
def test_row_band_pairs_partition_the_grid(lib, R):
    n, m = 42, 59
    nt = n * m
    total = 0
    for k in range(R):
        b, e = k * nt // R, (k + 1) * nt // R
        total += pkg.pair_count(pkg.make_config(n, m, 1040, 1392, tile_begin=b, tile_end=e))
    assert total == 2 * n * m - n - m


def test_workspace_size_matches_layout(lib):
    cfg = pkg.make_config(42, 59, 1040, 1392, chunk_pairs=8, chunk_tiles=8)
    ws = pkg.workspace_size(cfg)
    H, W, WP = 1040, 1392, 704
    raw = 2478 * H * W * 2
    spec = 2478 * WP * 1044 * 4       # resident Q15 unit phasors (u32), column pitch 1044
    chunks = 2 * 8 * H * WP * 8       # G (forward chunk) + Q (pair chunk), complex (8 each)
    assert raw + spec + chunks < ws < raw + spec + chunks + 5 * 2**20


def test_fp64_workspace_and_precision_validation(lib):
    """precision = 1 (f2): resident unit phasors and chunk intermediates in double2, plus the
    per-row-block argmax partials; any other precision value is rejected."""
    cfg = pkg.make_config(42, 59, 1040, 1392, chunk_pairs=8, chunk_tiles=8, precision=1)
    ws = pkg.workspace_size(cfg)
    H, W, WP = 1040, 1392, 704
    raw = 2478 * H * W * 2
    spec = 2478 * WP * 1048 * 8       # resident Q31 unit phasors (int2), column pitch 1048
    chunks = 2 * 8 * H * WP * 16      # Gd + Qd
    part = 4855 * (H // 4) * 12       # (double, u32) per pair and 4-row block
    assert raw + spec + chunks + part < ws < raw + spec + chunks + part + 5 * 2**20
    b = ctypes.c_size_t()
    for bad in (2, -1):
        cfg = pkg.make_config(3, 3, 192, 256, precision=bad)
        assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 1


def _eval_codelet(body, x):
    def fmaf(a, b, c):
        return a * b + c
    out = {}
    py = []
    for line in body.split("\n"):
        line = line.strip().rstrip(";")
        line = re.sub(r"\((-?[0-9.e+-]+)f\)", r"(\1)", line).replace("0.0f", "0.0")
        line = line.replace("fma(", "fmaf(")
        for ty in ("const float ", "const double "):
            if line.startswith(ty):
                line = line[len(ty):]
                if "v[" in line:
                    py.extend(line.split(", "))
                else:
                    py.append(line)
        if line.startswith("v["):
            mm = re.match(r"v\[(\d+)\] = make_(?:float|double)2\((.*), (.*)\)", line)
            py.append(f"out[{mm.group(1)}] = complex({mm.group(2)}, {mm.group(3)})")

    class F:
        def __init__(self, z):
            self.x, self.y = z.real, z.imag
    env = {"fmaf": fmaf, "v": [F(z) for z in x], "out": out}
    exec("\n".join(py), env)
    return np.array([out[k] for k in range(len(x))])


def _eval_packed_codelet(body, x):
    """The fp32 codelets are packed complex programs (f32x2.cuh): every value is a complex
    number, f2add / f2sub / f2mul / f2fma act component-wise, K(c) is a real constant, and the
    views I / MI / NEG multiply by i, -i, -1."""
    env = {"f2add": lambda a, b: a + b, "f2sub": lambda a, b: a - b,
           "f2mul": lambda a, b: a * b, "f2fma": lambda a, b, c: a * b + c,
           "K": lambda c: float(c), "I": lambda v: 1j * v, "MI": lambda v: -1j * v,
           "NEG": lambda v: -v, "v": list(x), "out": {}}
    py = []
    for line in body.split("\n"):
        line = re.sub(r"\((-?[0-9.e+-]+)f\)", r"(\1)", line.strip().rstrip(";"))
        if line.startswith("const float2 "):
            py.append(line[len("const float2 "):])
        elif line.startswith("v["):
            mm = re.match(r"v\[(\d+)\] = (.*)", line)
            py.append(f"out[{mm.group(1)}] = {mm.group(2)}")
        else:
            assert not line or line.startswith("//"), line
    exec("\n".join(py), env)
    return np.array([env["out"][k] for k in range(len(x))])


def test_generated_codelets_are_dfts():
    """fp32 codelets (packed complex operations) evaluate to the DFT; each costs about half
    the instructions of its scalar fp64 twin (one packed operation per complex step)."""
    src = open(os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200", "csrc",
                            "codelets.cuh")).read()
    funcs = re.findall(r"void dft(\d+)([mp])\(float2\* __restrict__ v\) \{\n(.*?)\n\}", src, re.S)
    assert len(funcs) >= 20
    twins = dict(((n, t), b) for n, t, b in re.findall(
        r"void dft(\d+)([mp])_d\(double2\* __restrict__ v\) \{\n(.*?)\n\}", src, re.S))
    rng = np.random.default_rng(0)
    for n, tag, body in funcs:
        assert "float " not in body and "fmaf" not in body, (n, tag)
        packed_ops = body.count("const float2 t")
        scalar_ops = twins[(n, tag)].count("const double t")
        assert packed_ops <= 0.55 * scalar_ops + 2, (n, tag, packed_ops, scalar_ops)
        n = int(n)
        sign = -1 if tag == "m" else 1
        x = rng.standard_normal(n) + 1j * rng.standard_normal(n)
        got = _eval_packed_codelet(body, x)
        j = np.arange(n)
        ref = np.exp(sign * 2j * math.pi * np.outer(j, j) / n) @ x
        assert np.abs(got - ref).max() <= 1e-6 * np.abs(ref).max(), (n, tag)


def test_generated_fp64_codelets_are_dfts():
    """The fp64 twins (f2 path) are the same programs with double temporaries and
    full-precision constants: evaluated in Python doubles they are the DFT to ~1e-15."""
    src = open(os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200", "csrc",
                            "codelets.cuh")).read()
    funcs = re.findall(r"void dft(\d+)([mp])_d\(double2\* __restrict__ v\) \{\n(.*?)\n\}", src,
                       re.S)
    assert len(funcs) >= 20
    assert not any("float" in body or "fmaf" in body for _, _, body in funcs)
    rng = np.random.default_rng(1)
    for n, tag, body in funcs:
        n = int(n)
        sign = -1 if tag == "m" else 1
        x = rng.standard_normal(n) + 1j * rng.standard_normal(n)
        got = _eval_codelet(body, x)
        j = np.arange(n)
        ref = np.exp(sign * 2j * math.pi * np.outer(j, j) / n) @ x
        assert np.abs(got - ref).max() <= 1e-13 * np.abs(ref).max(), (n, tag)


def _q15_encode(z):
    """Host emulation of pciam_kernels.cuh phasor_q15 (fp32 rsqrt of |v|^2 + 1e-36, scale
    32767, magic-number rounding fmaf(x, r, 1.5*2^23), low 16 bits of each field)."""
    x, y = z.real.astype(np.float32), z.imag.astype(np.float32)
    s2 = (x.astype(np.float64) ** 2 + y.astype(np.float64) ** 2 + 1e-36).astype(np.float32)
    r = (np.float32(1.0) / np.sqrt(s2)).astype(np.float32)
    r = (r * np.float32(32767.0)).astype(np.float32)
    fx = (x.astype(np.float64) * r + 12582912.0).astype(np.float32)   # one rounding (ulp 1)
    fy = (y.astype(np.float64) * r + 12582912.0).astype(np.float32)
    lo = fx.view(np.uint32) & np.uint32(0xFFFF)
    hi = fy.view(np.uint32) & np.uint32(0xFFFF)
    return lo | (hi << np.uint32(16))


def _q15_decode(w):
    lo = (w & np.uint32(0xFFFF)).astype(np.uint16).view(np.int16).astype(np.int64)
    hi = (w >> np.uint32(16)).astype(np.uint16).view(np.int16).astype(np.int64)
    return lo, hi


def test_q15_phasor_encoder_and_ncps_decoder():
    """The K2 resident-spectrum encoder (Q15 unit phasor, pciam_kernels.cuh phasor_q15) and
    the K3 NCPS decoder (exact int32 U_A conj(U_B)) re-evaluated on the host: the code's
    constants and byte selectors are read from the source; each decoded field is within
    half a Q15 step (+ rsqrt rounding) of 32767 F/|F|; a zero F is the zero phasor (reading
    C4); the integer NCPS equals 32767^2 F_A conj(F_B)/|F_A conj(F_B)| within 1e-4; the int32
    products cannot overflow."""
    src = open(os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200", "csrc",
                            "pciam_kernels.cuh")).read()
    body = src[src.index("__device__ __forceinline__ uint32_t phasor_q15"):]
    body = body[:body.index("\n}\n")]
    assert "1e-36f)" in body and "* 32767.0f" in body and body.count("12582912.0f") == 2
    assert "0x5410" in body
    dec = src[src.index("int32_t q15_lo"):src.index("NCPS_Q15_SCALE")]
    assert "0x9910" in dec and "(int32_t)w >> 16" in dec
    assert "32767.0 * 32767.0" in src
    rng = np.random.default_rng(5)
    z = (rng.standard_normal(200000) * 10.0 ** rng.uniform(-3, 10, 200000)
         + 1j * rng.standard_normal(200000) * 10.0 ** rng.uniform(-3, 10, 200000)).astype(np.complex64)
    z[:4] = [0, 1e-30, -7e10 + 1e-3j, 1j]
    w = _q15_encode(z)
    ax, ay = _q15_decode(w)
    assert ax[0] == 0 and ay[0] == 0                       # zero F -> zero phasor
    # |F| < 1e-18 (|F|^2 under the 1e-36 floor: rounding noise of a vanishing bin) encodes
    # as a phasor shorter than unit, here exactly zero; every larger F as its unit phasor
    assert ax[1] == 0 and ay[1] == 0
    assert np.abs(ax).max() <= 32767 and np.abs(ay).max() <= 32767
    keep = np.abs(z) >= 1e-17
    keep[:2] = False
    ax, ay, z = ax[keep], ay[keep], z[keep]
    zz = z.astype(np.complex128)
    u = zz / np.abs(zz) * 32767.0
    assert np.abs(ax - u.real).max() <= 0.5 + 0.02
    assert np.abs(ay - u.imag).max() <= 0.5 + 0.02
    bx, by = ax[1:], ay[1:]
    ax, ay = ax[:-1], ay[:-1]
    re, im = ax * bx + ay * by, ay * bx - ax * by           # the K3 int32 products
    assert max(np.abs(re).max(), np.abs(im).max()) < 2 ** 31
    za, zb = zz[:-1], zz[1:]
    p = za * np.conj(zb)
    ref = p / np.abs(p) * 32767.0 ** 2
    assert np.abs((re + 1j * im) - ref).max() <= 1e-4 * 32767.0 ** 2

def test_flags_and_multirank_validation(lib):
    """stitch_config.flags accepts only STITCH_FLAG_*; rank / world_size / nccl_id are
    validated on the host (the library derives the band only when it owns the exchange)."""
    b = ctypes.c_size_t()
    cfg = pkg.make_config(3, 3, 192, 256, flags=4)
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 1
    cfg = pkg.make_config(3, 3, 192, 256, flags=pkg.FLAG_NO_GRAPH | pkg.FLAG_SERIAL)
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 0
    nid = ctypes.create_string_buffer(128)
    vid = ctypes.cast(nid, ctypes.c_void_p)
    for kw in (dict(world_size=1, nccl_id=vid),                         # no peers
               dict(world_size=2, rank=2, nccl_id=vid),                 # rank out of range
               dict(world_size=2, rank=0, tile_begin=0, tile_end=4, nccl_id=vid),
               dict(world_size=10, rank=0)):                            # more ranks than tiles
        cfg = pkg.make_config(3, 3, 192, 256, **kw)
        assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 1, kw
    cfg = pkg.make_config(3, 3, 192, 256, world_size=2, rank=0, nccl_id=vid, precision=1)
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 2


@pytest.mark.parametrize("R", [2, 3, 8])
def test_library_derived_bands_partition_the_pairs(lib, R):
    """world_size > 1 with tile_begin = tile_end = 0: the library's balanced band of each rank
     -- the bands' pairs partition Table I's count."""
    n, m = 42, 59
    total = sum(pkg.pair_count(pkg.make_config(n, m, 1040, 1392, rank=k, world_size=R))
                for k in range(R))
    assert total == 2 * n * m - n - m


def test_nccl_unique_id(lib):
    """stitch_nccl_unique_id loads NCCL at run time (no GPU needed for the id)."""
    a, b = pkg.nccl_unique_id(), pkg.nccl_unique_id()
    assert len(a) == 128 and len(b) == 128 and a != b
    assert lib.stitch_nccl_unique_id(None) == 1


def test_bounded_pool_validation_and_size(lib):
    """Bounded mode (row f1): the host simulation of the refcounted slot schedule rejects a pool
    that cannot hold one tile row + one forward chunk (INVALID_ARG), accepts the smallest one
    that can, and the workspace then shrinks with the pool instead of the grid."""
    b = ctypes.c_size_t()
    n, m, H, W = 6, 7, 192, 256
    for pool, want in ((4, 1), (8, 1), (9, 0), (12, 0)):
        cfg = pkg.make_config(n, m, H, W, pool_tiles=pool, chunk_tiles=2, chunk_pairs=3)
        assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == want, pool
    cfg = pkg.make_config(n, m, H, W, pool_tiles=-1)
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 1
    cfg = pkg.make_config(n, m, H, W, pool_tiles=12, precision=1)
    assert lib.stitch_workspace_size(ctypes.byref(cfg), ctypes.byref(b)) == 2
    # 42x59 @ 1392x1040: 128 slots instead of 2478 tiles
    big = pkg.workspace_size(pkg.make_config(42, 59, 1040, 1392))
    small = pkg.workspace_size(pkg.make_config(42, 59, 1040, 1392, pool_tiles=128))
    per_tile = 1040 * 1392 * 2 + 1044 * 704 * 4
    assert big - small >= (2478 - 128) * per_tile
    assert small < 2.0e9
