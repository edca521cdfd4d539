"""Design study (CPU, numpy; not a test and not the oracle): how storing an FFT intermediate in
fp16 moves the normalised correlation surface of a 1392x1040 pair.  The fp32 kernels are modelled in
fp64 (their own rounding is ~1e-7, far below these effects); the Q15 resident phasor is modelled
exactly.  Used for DESIGN.md reading C11-Q: fp16 Q (K3 -> K4) moves the surface by ~2e-5 of its
peak (the GPU measures 1.9-2.3e-5), fp16 G (K1 -> K2) by ~2e-4 -- more than the 1e-4 near-tie
margin, so G stays float.  Run: python tools/sim_storage_precision.py"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synthgrid
g = synthgrid.make_grid(1, 2, 1040, 1392, seed=82)
A = g.tiles[0, 0].astype(np.float64); B = g.tiles[0, 1].astype(np.float64)
H, W = A.shape
def spec(T, g16):
    G = np.fft.rfft(T, axis=1)                      # row R2C (fp64 stand-in for the fp32 K1)
    if g16:
        s = 2.0 ** -11
        G = (G.real * s).astype(np.float16).astype(np.float64) / s + 1j * ((G.imag * s).astype(np.float16).astype(np.float64) / s)
    return np.fft.fft(G, axis=0)                    # column C2C
def q15(F):
    r = 32767.0 / np.sqrt(np.abs(F) ** 2 + 1e-36)
    return np.round(F.real * r) + 1j * np.round(F.imag * r)
def surface(g16, q16):
    UA, UB = q15(spec(A, g16)), q15(spec(B, g16))
    N = UA * np.conj(UB)
    Q = np.fft.ifft(N, axis=0) * H                  # unnormalised column inverse
    if q16:
        s = 2.0 ** -25
        Q = (Q.real * s).astype(np.float16).astype(np.float64) / s + 1j * ((Q.imag * s).astype(np.float16).astype(np.float64) / s)
    c = np.fft.irfft(Q, n=W, axis=1) * W
    return np.abs(c) / (H * W * 32767.0 ** 2)
FA, FB = np.fft.fft2(A), np.fft.fft2(B)
P = FA * np.conj(FB); mag = np.abs(P); Nx = np.where(mag > 0, P / np.where(mag > 0, mag, 1), 0)
ref = np.abs(np.fft.ifft2(Nx).real)
peak = ref.max()
for g16, q16 in ((False, False), (False, True), (True, False), (True, True)):
    s = surface(g16, q16)
    print(f"G16={g16} Q16={q16}: max err {np.abs(s - ref).max() / peak:.3g} of peak; argmax same {np.argmax(s) == np.argmax(ref)}")
Gr = np.fft.rfft(A, axis=1)
s = 2.0 ** -11
G16 = ((Gr.real * s).astype(np.float16).astype(np.float64) / s
       + 1j * (Gr.imag * s).astype(np.float16).astype(np.float64) / s)
F, F16 = np.fft.fft(Gr, axis=0), np.fft.fft(G16, axis=0)
print("spectrum rel L2 with an fp16 G:", np.linalg.norm(F16 - F) / np.linalg.norm(F))
