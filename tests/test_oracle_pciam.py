"""Pins for the oracle's PCIAM steps 3-7 and grid driver (oracle.c), independent of it.

  * shift theorem (closed form): B = circular shift of A by d  =>  the normalised
    surface |iFFT(NCC)|/(HW) is exactly 1 at d and ~0 elsewhere (steps 3-5, C2, C5);
  * CCF identities (Fig. 3): ccf(a,a)=1, ccf(a, alpha a + beta) = sign(alpha),
    symmetry, two-pass == exact integer moments, a naive numpy re-evaluation;
  * candidate rules (Fig. 2 l.8-12, readings C7, C8);
  * brute-force spatial NCC on tiny textured tiles: the true shift is the
    brute-force maximum and PCIAM returns it;
  * exact recovery of the generator's known shifts (config 1, and 1392x1040);
  * Table I counts (golden).
"""
import json
import os

import numpy as np
import pytest

import oracle
import synthgrid

GOLD = os.path.join(os.path.dirname(__file__), "golden", "paper_counts.json")
RNG = np.random.default_rng(99)


def tex(H, W, seed=5):
    return synthgrid.make_grid(1, 1, H, W, seed=seed).tiles[0, 0]


@pytest.mark.parametrize("shape,d", [((40, 48), (0, 0)), ((40, 48), (7, 3)), ((26, 58), (57, 25)),
                                     ((192, 256), (230, 5)), ((192, 256), (3, 170))])
def test_shift_theorem_exact_delta(shape, d):
    H, W = shape
    dx, dy = d
    A = tex(H, W)
    B = np.roll(A, shift=(-dy, -dx), axis=(0, 1))  # B(n) = A(n + d): B's origin is d in A
    s = oracle.surface(A, B)
    assert np.unravel_index(np.argmax(s), s.shape) == (dy, dx)
    assert abs(s[dy, dx] - 1.0) <= 1e-12
    s2 = s.copy(); s2[dy, dx] = 0
    assert s2.max() <= 1e-12
    p = oracle.pciam(A, B)
    assert (p["peak_x"], p["peak_y"]) == (dx, dy)
    assert abs(p["peak"] - 1.0) <= 1e-12
    assert p["max_imag_ratio"] <= 1e-9


def naive_ccf(A, B, dx, dy):
    H, W = A.shape
    a = A[dy:H, dx:W].astype(np.float64).ravel()
    b = B[0:H - dy, 0:W - dx].astype(np.float64).ravel()
    if a.size == 0:
        return None
    a = a - a.mean(); b = b - b.mean()
    den = np.sqrt((a * a).sum() * (b * b).sum())
    return None if den == 0 else float((a * b).sum() / den)


def test_ccf_identities():
    H, W = 40, 48
    A = tex(H, W).astype(np.int64) // 8
    c, v = oracle.ccf(A.astype(np.uint16), A.astype(np.uint16), 0, 0)
    assert v and abs(c - 1.0) <= 1e-12
    for dx, dy in [(0, 0), (5, 3), (30, 20), (40, 33)]:
        B = np.zeros((H, W), np.int64)
        B[0:H - dy, 0:W - dx] = 3 * A[dy:, dx:] + 100
        c, v = oracle.ccf(A.astype(np.uint16), B.astype(np.uint16), dx, dy)
        assert v and abs(c - 1.0) <= 1e-12
        B[0:H - dy, 0:W - dx] = 60000 - 2 * A[dy:, dx:]
        c, v = oracle.ccf(A.astype(np.uint16), B.astype(np.uint16), dx, dy)
        assert v and abs(c + 1.0) <= 1e-12


def test_ccf_symmetry_moments_and_naive():
    H, W = 40, 48
    A, B = tex(H, W, 1), tex(H, W, 2)
    for dx, dy in [(0, 0), (5, 3), (31, 22), (47, 0), (0, 39), (46, 38)]:
        c, v = oracle.ccf(A, B, dx, dy)
        # symmetry: swap the roles of the two regions (both cropped to origin 0)
        a = np.zeros_like(A); b = np.zeros_like(B)
        a[0:H - dy, 0:W - dx] = A[dy:, dx:]
        b[0:H - dy, 0:W - dx] = B[0:H - dy, 0:W - dx]
        c2, v2 = oracle.ccf(np.ascontiguousarray(b), np.ascontiguousarray(a), 0, 0)
        # the zero padding changes the region for (0,0), so compare on the true region only
        cm, vm, mom = oracle.ccf_moments(A, B, dx, dy)
        nv = naive_ccf(A, B, dx, dy)
        assert v == vm == (nv is not None)
        if v:
            assert abs(c - cm) <= 1e-12
            assert abs(c - nv) <= 1e-12
            assert int(mom[0]) == (H - dy) * (W - dx)
        if (dx, dy) == (0, 0):
            assert abs(c - c2) <= 1e-12


def test_ccf_invalid_cases():
    H, W = 20, 24
    A, B = tex(H, W, 1), tex(H, W, 2)
    assert oracle.ccf(A, B, W, 0)[1] is False
    assert oracle.ccf(A, B, 0, H)[1] is False
    const = np.full((H, W), 1234, np.uint16)
    assert oracle.ccf(const, B, 3, 3)[1] is False
    assert oracle.ccf(A, const, 3, 3)[1] is False


def test_eval_peak_candidate_rules():
    H, W = 40, 48
    A = tex(H, W, 3)
    # peak (0, 0) on A vs A: c1 = (0,0) ccf 1; c2 dx=W, c3 dy=H, c4 both -> invalid (C8)
    p = oracle.eval_peak(A, A, 0, 0)
    assert p["candidate"] == 1 and (p["dx"], p["dy"]) == (0, 0) and abs(p["ccf"] - 1) <= 1e-12
    assert np.isnan(p["ccf_k"][1]) and np.isnan(p["ccf_k"][2]) and np.isnan(p["ccf_k"][3])
    # x = W/2, y = H/2: all four candidates name the same region -> c1 wins the tie (C7)
    p = oracle.eval_peak(A, tex(H, W, 4), W // 2, H // 2)
    assert p["candidate"] == 1
    assert p["ccf_k"][0] == p["ccf_k"][1] == p["ccf_k"][2] == p["ccf_k"][3]
    # the chosen candidate is the max of the valid ones, mapped per Fig. 2 l.12
    B = tex(H, W, 5)
    for x, y in [(5, 7), (40, 3), (11, 35), (47, 39)]:
        p = oracle.eval_peak(A, B, x, y)
        cands = [(x, y), (W - x, y), (x, H - y), (W - x, H - y)]
        vals = [naive_ccf(A, B, dx, dy) for dx, dy in cands]
        best = max((v, -k) for k, v in enumerate(vals) if v is not None)
        k = -best[1]
        assert p["candidate"] == k + 1
        assert (p["dx"], p["dy"]) == cands[k]
        assert abs(p["ccf"] - vals[k]) <= 1e-12


def brute_ncc_argmax(A, B, min_frac=0.2):
    """Brute-force spatial NCC over every (dx, dy) with overlap >= min_frac * H W."""
    H, W = A.shape
    best, arg = -2.0, None
    for dy in range(H):
        for dx in range(W):
            if (H - dy) * (W - dx) < min_frac * H * W:
                continue
            v = naive_ccf(A, B, dx, dy)
            if v is not None and v > best:
                best, arg = v, (dx, dy)
    return arg, best


@pytest.mark.parametrize("H,W,seed", [(40, 48, 11), (26, 58, 12), (20, 24, 13), (40, 48, 14)])
def test_brute_force_spatial_ncc_tiny_tiles(H, W, seed):
    g = synthgrid.make_grid(2, 2, H, W, overlap=0.5, delta=2, seed=seed)
    tw, tn = g.true_west(), g.true_north()
    pairs = [((0, 0), (0, 1), (tw[0][0, 1], tw[1][0, 1])),
             ((1, 0), (1, 1), (tw[0][1, 1], tw[1][1, 1])),
             ((0, 0), (1, 0), (tn[0][1, 0], tn[1][1, 0])),
             ((0, 1), (1, 1), (tn[0][1, 1], tn[1][1, 1]))]
    for a, b, truth in pairs:
        A, B = g.tiles[a], g.tiles[b]
        arg, _ = brute_ncc_argmax(A, B)
        assert arg == tuple(int(t) for t in truth)
        p = oracle.pciam(A, B)
        assert (p["dx"], p["dy"]) == arg


def test_config1_exact_recovery(cfg1_grid, cfg1_oracle):
    g = cfg1_grid
    west, north = cfg1_oracle
    tw, tn = g.true_west(), g.true_north()
    assert np.array_equal(west["dx"][:, 1:], tw[0][:, 1:])
    assert np.array_equal(west["dy"][:, 1:], tw[1][:, 1:])
    assert np.array_equal(north["dx"][1:], tn[0][1:])
    assert np.array_equal(north["dy"][1:], tn[1][1:])
    assert (west["candidate"][:, 0] == 0).all() and (north["candidate"][0] == 0).all()
    assert np.isnan(west["ccf"][:, 0]).all() and np.isnan(north["ccf"][0]).all()
    valid = np.concatenate([west[:, 1:].ravel(), north[1:].ravel()])
    assert (valid["ccf"] > 0.99).all()
    # peak margin far above any rounding (C17) and Im(c) ~ 0 (C3)
    assert ((valid["peak"] - valid["runner_up"]) / valid["peak"] > 1e-2).all()
    assert (valid["max_imag_ratio"] <= 1e-9).all()


def test_table1_counts(cfg1_oracle):
    gold = json.load(open(GOLD))
    west, north = cfg1_oracle
    n, m = west.shape
    pairs = int((west["candidate"] != 0).sum() + (north["candidate"] != 0).sum())
    assert pairs == 2 * n * m - n - m                     # Table I
    a = gold["a10_grid"]
    n, m, h, w = a["n"], a["m"], a["h"], a["w"]
    assert 2 * n * m - n - m == 4855
    assert 3 * n * m - n - m == 7333
    assert abs(2 * h * w / 2**20 - a["tile_mib"]) < 0.01  # 2hw bytes
    assert abs(n * m * 2 * h * w / 2**30 - a["dataset_gib"]) < 0.01
    t = gold["transform_size"]
    assert abs(16 * h * w / 2**20 - t["per_transform_mib_approx"]) < 0.2   # 16hw
    assert abs(n * m * 16 * h * w / 2**30 - t["grid_forward_gib"]) < 0.05
    ts = gold["time_series"]
    assert abs(ts["scans"] * ts["channels"] * ts["n"] * ts["m"] * 2 * 1392 * 1040 / 2**30
               - ts["raw_gib"]) < 0.5


@pytest.mark.slow
@pytest.mark.parametrize("overlap", [0.10, 0.70])
def test_full_size_exact_recovery(overlap):
    g = synthgrid.make_grid(2, 2, 1040, 1392, overlap=overlap, delta=12, seed=7)
    west, north = oracle.grid(g.tiles)
    tw, tn = g.true_west(), g.true_north()
    assert np.array_equal(west["dx"][:, 1:], tw[0][:, 1:])
    assert np.array_equal(west["dy"][:, 1:], tw[1][:, 1:])
    assert np.array_equal(north["dx"][1:], tn[0][1:])
    assert np.array_equal(north["dy"][1:], tn[1][1:])
    valid = np.concatenate([west[:, 1:].ravel(), north[1:].ravel()])
    assert (valid["candidate"] == 1).all()
    assert ((valid["peak"] - valid["runner_up"]) / valid["peak"] > 1e-2).all()


@pytest.mark.parametrize("shape", [(1, 2), (3, 4), (40, 48)])
def test_zero_spectrum_branch_and_first_index_tie(shape):
    """Readings C4 and C6 pinned with exact arithmetic.  Tile B all zeros: F_B = 0 exactly in
    every bin (0 times any twiddle is 0), so |F_A conj(F_B)| = 0 everywhere and step 3's
    branch sets NCC = 0 (C4) -- without it every bin is 0/0 = NaN.  The inverse of an all-zero
    NCC is exactly 0, so all H*W surface values tie and step 5 must return the first index in
    row-major order, (0, 0) (C6: a '>=' scan would return the last).  Every candidate then has
    B's zero variance, so none is valid (C8): candidate 0, ccf NaN, (dx, dy) = the peak."""
    H, W = shape
    A = tex(max(H, 2), max(W, 2))[:H, :W] if H > 1 else np.array([[1, 0]], np.uint16)
    B = np.zeros((H, W), np.uint16)
    for a, b in ((A, B), (B, A)):   # also A all zeros (F_A = 0)
        s = oracle.surface(a, b)
        assert np.all(s == 0.0)                  # exactly zero, no NaN
        p = oracle.pciam(a, b)
        assert (p["peak_x"], p["peak_y"]) == (0, 0)
        assert p["peak"] == 0.0 and p["runner_up"] == 0.0
        assert p["candidate"] == 0 and np.isnan(p["ccf"]) and (p["dx"], p["dy"]) == (0, 0)
        assert np.isnan(p["ccf_k"]).all()
