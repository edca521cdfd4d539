"""NEXT rows f3 (phase 2: absolute positions) and f4 (phase 3: overlay composition).

f3 is host code: pinned here on CPU against the generator's known tile origins, with the
phase-1 translations taken from the oracle (reading C19: maximum
spanning tree on CCF, positions = path sums).  f4 runs on the GPU and is compared with a
plain numpy overlay (later tile on top, row-major order).
"""
import numpy as np
import pytest

import oracle
import synthgrid
from paper_conf_icpp_blattnerkcsbz14_b200 import PAIR_DTYPE, global_positions


def to_pairs(res):
    out = np.zeros(res.shape, PAIR_DTYPE)
    for f in ("dx", "dy", "ccf", "candidate", "peak_x", "peak_y"):
        out[f] = res[f]
    return out


@pytest.fixture(scope="module")
def grid_and_oracle():
    g = synthgrid.make_grid(4, 5, 192, 256, overlap=0.2, delta=4, seed=51)
    w, n = oracle.grid(g.tiles)
    return g, to_pairs(w), to_pairs(n)


def test_global_positions_recover_origins(grid_and_oracle):
    g, w, n = grid_and_oracle
    pos, parent = global_positions(w, n)
    ref = g.origins - g.origins[0, 0]
    assert np.array_equal(pos, ref)
    assert parent[0, 0] == -1 and (parent.reshape(-1)[1:] >= 0).all()   # one spanning tree


def test_global_positions_skip_unreliable_edge(grid_and_oracle):
    g, w, n = grid_and_oracle
    w2 = w.copy()
    w2[2, 3]["dx"] += 17          # a wrong translation with a low CCF is left out of the tree
    w2[2, 3]["ccf"] = 0.05
    pos, _ = global_positions(w2, n)
    assert np.array_equal(pos, g.origins - g.origins[0, 0])


def test_global_positions_disconnected_components():
    pairs_w = np.zeros((2, 2), PAIR_DTYPE)
    pairs_n = np.zeros((2, 2), PAIR_DTYPE)
    pairs_w[0, 1] = (5, 1, 0.9, 1, 0, 0, 0, [0, 0, 0, 0])     # only tile 0 -- tile 1 connected
    pos, parent = global_positions(pairs_w, pairs_n)
    assert pos[0, 1].tolist() == [5, 1] and parent[1, 0] == -1 and pos[1, 1].tolist() == [0, 0]


def numpy_overlay(tiles, pos):
    n, m, H, W = tiles.shape
    p = pos.reshape(-1, 2) - pos.reshape(-1, 2).min(axis=0)
    cw, ch = p[:, 0].max() + W, p[:, 1].max() + H
    canvas = np.zeros((ch, cw), np.uint16)
    for t in range(n * m):
        x, y = p[t]
        canvas[y:y + H, x:x + W] = tiles.reshape(n * m, H, W)[t]
    return canvas


@pytest.mark.gpu
@pytest.mark.parametrize("ov", [0.1, 0.7])
def test_compose_overlay_matches_numpy(ov):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay
    g = synthgrid.make_grid(4, 5, 192, 256, overlap=ov, delta=4, seed=52)
    dev = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
    canvas = compose_overlay(dev, g.origins)
    torch.cuda.synchronize()
    got = canvas.cpu().view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(got, numpy_overlay(g.tiles, g.origins))
