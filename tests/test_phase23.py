"""NEXT rows f3 (phase 2: absolute positions) and f4 (phase 3: overlay composition).

f3 is host code (stitch_global_positions): checked here against the oracle's phase 2
(oracle/phases.py: Prim's algorithm, where the product runs Kruskal's; PAPER.md L436-452,
reading C19: maximum spanning tree on CCF, positions = path sums), which is itself pinned by
brute-force enumeration of spanning forests on tiny grids, and against the generator's known
tile origins.  f4 runs on the GPU (stitch_compose_overlay) and is compared with the oracle's
overlay (later tile on top, row-major order), pinned per pixel.
"""
import itertools

import numpy as np
import pytest

import oracle
import synthgrid
from oracle import phases
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
    p = pos.reshape(-1, 2) - pos.reshape(-1, 2).min(axis=0)
    return phases.overlay(tiles, p.reshape(pos.shape))


# ---- pins of the oracle's phase 2 / phase 3 ------------------------------------------------
def random_pairs(n, m, rng, ties=False, invalid=0.0):
    """Random west/north records: translations, CCFs (optionally drawn from 3 values, so the
    pair-id tie rule decides), a fraction of invalid pairs (candidate 0 / NaN CCF)."""
    w = np.zeros((n, m), PAIR_DTYPE)
    no = np.zeros((n, m), PAIR_DTYPE)
    for rec, ok in ((w, np.arange(m)[None, :] >= 1), (no, np.arange(n)[:, None] >= 1)):
        valid = np.broadcast_to(ok, (n, m)) & (rng.random((n, m)) >= invalid)
        rec["dx"] = rng.integers(-40, 300, (n, m))
        rec["dy"] = rng.integers(-40, 300, (n, m))
        rec["ccf"] = (rng.choice([0.5, 0.7, 0.9], (n, m)) if ties else rng.random((n, m)))
        rec["candidate"] = np.where(valid, rng.integers(1, 5, (n, m)), 0)
        rec["ccf"] = np.where(valid, rec["ccf"], np.nan)
    return w, no


def brute_force_forest(nt, es):
    """The best spanning forest by definition: among all acyclic edge sets with as many edges
    as a spanning forest has, the one whose edge keys, sorted, are lexicographically smallest
    (the greedy optimum of a matroid under a strict total order on its elements)."""
    parent = list(range(nt))

    def find(u, par):
        while par[u] != u:
            u = par[u]
        return u
    for _, a, b, _, _ in es:
        ra, rb = find(a, parent), find(b, parent)
        if ra != rb:
            parent[ra] = rb
    k = nt - len({find(u, parent) for u in range(nt)})
    best = None
    for sub in itertools.combinations(es, k):
        par = list(range(nt))
        acyclic = True
        for _, a, b, _, _ in sub:
            ra, rb = find(a, par), find(b, par)
            if ra == rb:
                acyclic = False
                break
            par[ra] = rb
        if acyclic:
            keys = sorted(e[0] for e in sub)
            if best is None or keys < best[0]:
                best = (keys, sub)
    return sorted(best[1])


@pytest.mark.parametrize("shape,ties,invalid", [((2, 2), False, 0.0), ((2, 3), False, 0.0),
                                                ((3, 3), False, 0.0), ((2, 3), True, 0.0),
                                                ((3, 3), True, 0.0), ((3, 3), False, 0.3),
                                                ((2, 4), True, 0.4)])
def test_oracle_spanning_tree_is_the_brute_force_optimum(shape, ties, invalid):
    rng = np.random.default_rng(hash((shape, ties, invalid)) % 2**32)
    for _ in range(5):
        w, n = random_pairs(*shape, rng, ties, invalid)
        es = phases.edges(w, n)
        nt = shape[0] * shape[1]
        assert sorted(phases.spanning_tree(nt, es)) == brute_force_forest(nt, es)


def test_oracle_positions_are_path_sums():
    """Exact translations of known origins: any tree gives the origins back (path invariance),
    and every tile's position is its parent's plus the connecting translation."""
    rng = np.random.default_rng(3)
    n, m = 4, 6
    org = np.stack(np.meshgrid(np.arange(m) * 200, np.arange(n) * 150), -1)
    org = org + rng.integers(0, 9, (n, m, 2))
    w, no = random_pairs(n, m, rng)
    w["dx"][:, 1:] = org[:, 1:, 0] - org[:, :-1, 0]
    w["dy"][:, 1:] = org[:, 1:, 1] - org[:, :-1, 1]
    no["dx"][1:] = org[1:, :, 0] - org[:-1, :, 0]
    no["dy"][1:] = org[1:, :, 1] - org[:-1, :, 1]
    pos, parent = phases.global_positions(w, no)
    assert np.array_equal(pos, org - org[0, 0])
    assert parent[0, 0] == -1 and (parent.reshape(-1)[1:] >= 0).all()


def test_oracle_overlay_per_pixel():
    """Each canvas pixel is the pixel of the LAST tile (row-major) covering it, 0 if none."""
    rng = np.random.default_rng(4)
    tiles = rng.integers(1, 60000, (2, 3, 5, 7)).astype(np.uint16)
    pos = np.array([[[0, 0], [5, 1], [11, 0]], [[1, 4], [6, 3], [12, 5]]])
    canvas = phases.overlay(tiles, pos)
    for y in range(canvas.shape[0]):
        for x in range(canvas.shape[1]):
            want = 0
            for t in range(6):
                px, py = pos.reshape(-1, 2)[t]
                if px <= x < px + 7 and py <= y < py + 5:
                    want = tiles.reshape(6, 5, 7)[t, y - py, x - px]
            assert canvas[y, x] == want, (x, y)


# ---- the product's phase 2 against the oracle's ---------------------------------------------
@pytest.mark.parametrize("shape,ties,invalid", [((6, 7), False, 0.0), ((6, 7), True, 0.0),
                                                ((9, 5), False, 0.25), ((8, 8), True, 0.35),
                                                ((1, 9), False, 0.0), ((7, 1), True, 0.2)])
def test_global_positions_match_oracle(shape, ties, invalid):
    rng = np.random.default_rng(sum(shape) * 7 + int(ties) + int(invalid * 100))
    for _ in range(4):
        w, n = random_pairs(*shape, rng, ties, invalid)
        pos, parent = global_positions(w, n)
        opos, oparent = phases.global_positions(w, n)
        assert np.array_equal(pos, opos)
        assert np.array_equal(parent, oparent)


@pytest.mark.gpu
@pytest.mark.parametrize("shape,ov", [((4, 5, 192, 256), 0.1), ((4, 5, 192, 256), 0.7),
                                      ((3, 4, 26, 58), 0.3), ((2, 3, 1040, 1392), 0.1)])
def test_compose_overlay_matches_numpy(shape, ov):
    """The 16-byte vector path (W a multiple of 8: every source misalignment and canvas row
    phase occurs) and the pixel path (W = 58)."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay
    n, m, H, W = shape
    g = synthgrid.make_grid(n, m, H, W, overlap=ov, delta=4, seed=52)
    dev = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
    canvas = compose_overlay(dev, g.origins)
    torch.cuda.synchronize()
    got = canvas.cpu().view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(got, numpy_overlay(g.tiles, g.origins))


@pytest.mark.gpu
def test_compose_overlay_stays_inside_the_canvas():
    """compute-sanitizer is unavailable on the GPU pool: the canvas is a view into a larger
    buffer at an odd element offset (so its rows start at every 16-byte phase), the bytes
    around it hold a sentinel, and the overlay must leave them untouched."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay
    for n, m, H, W, ov in ((3, 4, 192, 256, 0.1), (3, 4, 26, 58, 0.3), (2, 2, 1040, 1392, 0.1)):
        g = synthgrid.make_grid(n, m, H, W, overlap=ov, delta=4, seed=53)
        p = g.origins.reshape(-1, 2) - g.origins.reshape(-1, 2).min(axis=0)
        cw, ch = int(p[:, 0].max()) + W, int(p[:, 1].max()) + H
        pad = 4099
        big = torch.full((2 * pad + ch * cw,), 0xBEEF - 65536, dtype=torch.int16, device="cuda")
        big[pad:pad + ch * cw] = 0
        canvas = big[pad:pad + ch * cw].view(torch.uint16).view(ch, cw)
        dev = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
        compose_overlay(dev, g.origins, canvas)
        torch.cuda.synchronize()
        b = big.cpu().numpy().view(np.uint16)
        assert (b[:pad] == 0xBEEF).all() and (b[pad + ch * cw:] == 0xBEEF).all(), (n, m, H, W)
        got = b[pad:pad + ch * cw].reshape(ch, cw)
        assert np.array_equal(got, numpy_overlay(g.tiles, g.origins)), (n, m, H, W)


@pytest.mark.gpu
def test_compose_overlay_async_is_stream_ordered():
    """stitch_compose_overlay_async returns once enqueued: on a side stream, after work that
    fills the tiles on that same stream, the canvas equals the synchronous call's."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_icpp_blattnerkcsbz14_b200 import compose_overlay
    g = synthgrid.make_grid(3, 4, 192, 256, overlap=0.2, delta=4, seed=54)
    ref_tiles = torch.from_numpy(g.tiles.view(np.int16)).view(torch.uint16).cuda()
    want = compose_overlay(ref_tiles, g.origins)
    torch.cuda.synchronize()
    side = torch.cuda.Stream()
    with torch.cuda.stream(side):
        tiles = torch.zeros_like(ref_tiles)
        tiles.copy_(ref_tiles)                  # the producer, on the same stream
        canvas = torch.zeros_like(want)
        compose_overlay(tiles, g.origins, canvas, sync=False)
    side.synchronize()
    assert torch.equal(canvas, want)
