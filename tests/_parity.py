"""Element-wise comparison of the CUDA path's results with the fp64 oracle's (test helper).

Tolerances (BASELINE.json north_star):
  * translations (dx, dy), chosen candidate, peak location: bit-exact;
  * CCF: |gpu - oracle| <= 1e-4 (the fp32 contract); the GPU CCF comes from exact integer
    moments, so it is also held to 1e-9 here (each candidate's ccf_k too);
  * peak height max|c|/(HW): relative 1e-4;
  * margin-aware argmax (reading C17): where the oracle's runner-up is within 1e-4 of its
    max, any GPU peak in that near-tie set is accepted, and the GPU's (dx, dy, candidate,
    ccf) must equal oracle.eval_peak at the GPU's peak;
  * candidates whose oracle CCFs tie within 1e-12 (tiny regions whose CCF is +-1, reading
    C10) are interchangeable: either choice is a correct "first maximum" up to rounding.
  * the fp64 path (precision = 1, fp64=True) is held to the fp64 bands of test_gpu_fp64.py:
    near-tie margin 1e-9 (its error above fp64 rounding is the Q31 phasor rounding, ~4e-12 of
    the peak at 1392x1040, reading C11-f2) and the peak height to the float storage
    of stitch_pair.peak (2^-23 relative).
"""
from __future__ import annotations

import numpy as np

import oracle

NEAR_TIE = 1e-4
NEAR_TIE_F64 = 1e-9


def compare_pairs(got, ref, tiles_a, tiles_b, mask, stats=None, fp64=False):
    """got/ref: [n, m] result arrays (GPU PAIR_DTYPE / oracle PAIR_DTYPE); tiles_a/b: index ->
    uint16 tile A (neighbour) / B (tile); mask: pairs to compare; fp64: the precision = 1 path
    (near-tie margin NEAR_TIE_F64).  Returns the number of near-tie (C17) pairs."""
    amb = 0
    for idx in zip(*np.nonzero(mask)):
        g, r = got[idx], ref[idx]
        if r["candidate"] == 0 and np.isnan(r["ccf"]) and r["peak"] == 0:
            continue
        band = NEAR_TIE_F64 if fp64 else NEAR_TIE
        near = (r["peak"] - r["runner_up"]) < band * r["peak"] or r["peak"] <= 0
        if near:
            amb += 1
            A, B = tiles_a(idx), tiles_b(idx)
            s = oracle.surface(A, B)
            v = s[g["peak_y"], g["peak_x"]]
            assert v >= s.max() * (1 - band), (idx, "gpu peak outside the near-tie set")
            if stats is not None:
                stats.setdefault("near_tie", []).append(
                    (tuple(int(i) for i in idx), (int(r["peak_x"]), int(r["peak_y"])),
                     (int(g["peak_x"]), int(g["peak_y"]))))
            r = oracle.eval_peak(A, B, g["peak_x"], g["peak_y"])
        else:
            assert (g["peak_x"], g["peak_y"]) == (r["peak_x"], r["peak_y"]), idx
            assert abs(g["peak"] - r["peak"]) <= (2.0 ** -23 if fp64 else NEAR_TIE) * r["peak"], idx
        gc, rc = int(g["candidate"]), int(r["candidate"])
        if gc != rc:   # only a rounding-level CCF tie between two valid candidates may differ
            assert gc > 0 and rc > 0, (idx, gc, rc)
            assert abs(r["ccf_k"][gc - 1] - r["ccf_k"][rc - 1]) <= 1e-12, (idx, gc, rc)
            r = r.copy()
            W, H = tiles_b(idx).shape[1], tiles_b(idx).shape[0]
            x, y = int(r["peak_x"]), int(r["peak_y"])
            r["dx"], r["dy"] = [(x, y), (W - x, y), (x, H - y), (W - x, H - y)][gc - 1]
            r["ccf"] = r["ccf_k"][gc - 1]
            if stats is not None:
                stats["ccf_ties"] = stats.get("ccf_ties", 0) + 1
        assert (g["dx"], g["dy"]) == (r["dx"], r["dy"]), idx
        if gc:
            assert abs(g["ccf"] - r["ccf"]) <= 1e-4, idx
            assert abs(g["ccf"] - r["ccf"]) <= 1e-9, idx
        else:
            assert np.isnan(g["ccf"])
        for k in range(4):
            if np.isnan(r["ccf_k"][k]):
                assert np.isnan(g["ccf_k"][k]), (idx, k)
            else:
                assert abs(g["ccf_k"][k] - r["ccf_k"][k]) <= 1e-9, (idx, k)
    return amb


def grid_parity(tiles, west, north, ow, on, stats=None, fp64=False):
    """Every west and north pair of a grid against the oracle's (ow, on); returns the number of
    near-tie pairs."""
    n, m = tiles.shape[:2]
    wmask = np.zeros((n, m), bool)
    wmask[:, 1:] = True
    nmask = np.zeros((n, m), bool)
    nmask[1:, :] = True
    amb = compare_pairs(west, ow, lambda i: tiles[i[0], i[1] - 1], lambda i: tiles[i], wmask,
                        stats, fp64)
    amb += compare_pairs(north, on, lambda i: tiles[i[0] - 1, i[1]], lambda i: tiles[i], nmask,
                         stats, fp64)
    assert (west["candidate"][:, 0] == 0).all() and np.isnan(west["ccf"][:, 0]).all()
    assert (north["candidate"][0] == 0).all() and np.isnan(north["ccf"][0]).all()
    return amb
