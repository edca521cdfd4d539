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
    spec = 2478 * H * WP * 4          # resident phase codes (u32)
    chunks = 2 * 8 * H * WP * 8       # G (forward chunk) + Q (pair chunk), complex (8 each)
    assert raw + spec + chunks < ws < raw + spec + chunks + 5 * 2**20


def test_fp64_workspace_and_precision_validation(lib):
    """precision = 1 (f2): resident unit phasors and chunk intermediates in double2, plus the
    per-row-block argmax partials; any other precision value is rejected."""
    cfg = pkg.make_config(42, 59, 1040, 1392, chunk_pairs=8, chunk_tiles=8, precision=1)
    ws = pkg.workspace_size(cfg)
    H, W, WP = 1040, 1392, 704
    raw = 2478 * H * W * 2
    spec = 2478 * H * WP * 16         # resident unit phasors (double2)
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


def test_generated_codelets_are_dfts():
    src = open(os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200", "csrc",
                            "codelets.cuh")).read()
    funcs = re.findall(r"void dft(\d+)([mp])\(float2\* __restrict__ v\) \{\n(.*?)\n\}", src, re.S)
    assert len(funcs) >= 20
    rng = np.random.default_rng(0)
    for n, tag, body in funcs:
        n = int(n)
        sign = -1 if tag == "m" else 1
        x = rng.standard_normal(n) + 1j * rng.standard_normal(n)
        got = _eval_codelet(body, x)
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


def test_phase_code_polynomial_matches_atan2():
    """The K2 phase encoder's atan2 (octant reduction + fitted polynomial, pciam_kernels.cuh)
    re-evaluated in float32 on the host: within 3e-7 rad of the exact angle, and the
    NCPS decoder's wrap-around difference of two codes recovers phase differences."""
    src = open(os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200", "csrc",
                            "pciam_kernels.cuh")).read()
    body = src[src.index("__device__ __forceinline__ uint32_t phase_code"):]
    body = body[:body.index("\n}\n")]
    coef = [float(c) for c in re.findall(r"fmaf\(p, s, (-?\d\.\d+)f\)", body)]
    coef = [float(re.search(r"float p = (-?\d\.\d+)f;", body).group(1))] + coef
    assert len(coef) == 9
    rng = np.random.default_rng(5)
    z = (rng.standard_normal(200000) + 1j * rng.standard_normal(200000)).astype(np.complex64)
    x, y = z.real.astype(np.float32), z.imag.astype(np.float32)
    ax, ay = np.abs(x), np.abs(y)
    mx, mn = np.maximum(ax, ay), np.minimum(ax, ay)
    t = (mn / mx).astype(np.float32)
    s = (t * t).astype(np.float32)
    p = np.float32(coef[0])
    for c in coef[1:]:
        p = (p * s + np.float32(c)).astype(np.float32)
    r = (p * t).astype(np.float32)
    r = np.where(ay > ax, np.float32(0.5) - r, r)
    r = np.where(x < 0, np.float32(1.0) - r, r)
    r = np.copysign(r, y)
    err = np.abs(np.angle(np.exp(1j * (np.pi * r.astype(np.float64) - np.angle(z.astype(np.complex128))))))
    assert err.max() <= 3e-7
    q = np.clip(np.rint(r.astype(np.float64) * 2**31), -2**31, 2**31 - 1).astype(np.int64)
    code = (q.astype(np.uint32) & np.uint32(0xFFFFFFFE)) | np.uint32(1)
    d = (code[:-1] - code[1:]).astype(np.uint32).view(np.int32).astype(np.float64) * (2 * np.pi / 2**32)
    ref = np.angle(z[:-1].astype(np.complex128) * np.conj(z[1:].astype(np.complex128)))
    assert np.abs(np.angle(np.exp(1j * (d - ref)))).max() <= 1e-6
