"""Pins for the oracle's mixed-radix DFT (oracle.c dft_rec / dft2), independent of it.

Pins (SURVEY.md 8(c) "What pins each part", DFT row):
  * brute force: the O(N^2) DFT definition, evaluated here with numpy matrices,
    for every N <= 64 and the paper's factor lengths (13, 29, 696, 1040, 1392, ...);
  * invariants: Parseval, linearity, inverse(forward(x)) = N x;
  * closed forms: DFT(delta) = 1, DFT(1) = N delta, DFT(cos) = two spikes;
  * library cross-check (test-only): numpy.fft (pocketfft) in 1-D and 2-D.
"""
import numpy as np
import pytest

import oracle

RNG = np.random.default_rng(1234)


def brute_dft(x, inverse=False):
    """X[k] = sum_j x[j] exp(-+2 pi i j k / N), straight from the definition."""
    N = x.size
    j = np.arange(N)
    s = 1.0 if inverse else -1.0
    Wm = np.exp(s * 2j * np.pi * np.outer(j, j) / N)
    return Wm @ x


def rand_c(n):
    return RNG.standard_normal(n) + 1j * RNG.standard_normal(n)


@pytest.mark.parametrize("N", list(range(1, 65)))
def test_dft_matches_definition_small(N):
    x = rand_c(N)
    for inv in (False, True):
        ref = brute_dft(x, inv)
        got = oracle.dft(x, inverse=inv)
        assert np.abs(got - ref).max() <= 1e-12 * max(1.0, np.abs(ref).max())


@pytest.mark.parametrize("N", [13, 26, 29, 58, 65, 87, 96, 128, 192, 256, 520, 696, 1040, 1392])
def test_dft_matches_definition_paper_lengths(N):
    x = rand_c(N)
    ref = brute_dft(x)
    got = oracle.dft(x)
    assert np.abs(got - ref).max() <= 1e-12 * np.abs(ref).max()
    # independent library, test-only
    assert np.abs(got - np.fft.fft(x)).max() <= 1e-12 * np.abs(ref).max()


@pytest.mark.parametrize("N", [29, 1040, 1392])
def test_parseval_linearity_roundtrip(N):
    x, y = rand_c(N), rand_c(N)
    X, Y = oracle.dft(x), oracle.dft(y)
    assert np.isclose(np.sum(np.abs(x) ** 2), np.sum(np.abs(X) ** 2) / N, rtol=1e-12)
    a, b = 0.7 - 0.2j, -1.3 + 0.5j
    assert np.abs(oracle.dft(a * x + b * y) - (a * X + b * Y)).max() <= 1e-11 * np.abs(X).max()
    assert np.abs(oracle.dft(X, inverse=True) - N * x).max() <= 1e-11 * N * np.abs(x).max()


@pytest.mark.parametrize("N", [13, 29, 696, 1040, 1392])
def test_closed_forms(N):
    d = np.zeros(N, complex); d[0] = 1
    assert np.abs(oracle.dft(d) - 1).max() <= 1e-13
    one = np.ones(N, complex)
    ref = np.zeros(N, complex); ref[0] = N
    assert np.abs(oracle.dft(one) - ref).max() <= 1e-12 * N
    f = 5
    c = np.cos(2 * np.pi * f * np.arange(N) / N).astype(complex)
    ref = np.zeros(N, complex); ref[f] += N / 2; ref[N - f] += N / 2
    assert np.abs(oracle.dft(c) - ref).max() <= 1e-11 * N


@pytest.mark.parametrize("shape", [(20, 24), (26, 58), (192, 256)])
def test_dft2_matches_library_and_definition(shape):
    H, W = shape
    x = RNG.standard_normal(shape) + 1j * RNG.standard_normal(shape)
    got = oracle.dft2(x)
    assert np.abs(got - np.fft.fft2(x)).max() <= 1e-12 * np.abs(got).max()
    if H * W <= 1600:  # separable definition, rows (x) then columns (y)
        ref = brute_2d(x)
        assert np.abs(got - ref).max() <= 1e-12 * np.abs(ref).max()
    back = oracle.dft2(got, inverse=True)
    assert np.abs(back - H * W * x).max() <= 1e-11 * H * W * np.abs(x).max()


def brute_2d(x):
    H, W = x.shape
    ky, y = np.meshgrid(np.arange(H), np.arange(H), indexing="ij")
    kx, xx = np.meshgrid(np.arange(W), np.arange(W), indexing="ij")
    EH = np.exp(-2j * np.pi * ky * y / H)
    EW = np.exp(-2j * np.pi * kx * xx / W)
    return EH @ x @ EW.T


@pytest.mark.slow
def test_fft2_u16_full_tile_matches_library():
    img = RNG.integers(0, 65536, size=(1040, 1392)).astype(np.uint16)
    got = oracle.fft2_u16(img)
    ref = np.fft.fft2(img.astype(np.float64))
    assert np.abs(got - ref).max() <= 1e-12 * np.abs(ref).max()
