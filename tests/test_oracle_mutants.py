"""The oracle's pins catch plausible mistakes: mutation testing of oracle/oracle.c.

Each mutant below is a one-line change a careful implementer could plausibly make while writing
the oracle from the paper (a dropped conjugate, a wrong transform sign, a missing zero branch, an
off-by-one region, a '>=' tie rule, a swapped candidate, a mean of the wrong image, ...).  Every
mutant is compiled into its own library and run through a compact battery of the pins of
test_oracle_dft.py / test_oracle_pciam.py (the DFT definition, the shift theorem, the exact C4/C6
zero-tile case, the CCF identities, the candidate rules, brute-force spatial NCC, exact recovery
of the generator's shifts); the test asserts that the unmodified oracle passes every pin and that
EVERY mutant fails at least one.  Nothing here is an input to any other test.
"""
import importlib.util
import math
import os
import subprocess

import numpy as np
import pytest

import synthgrid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "oracle.c")

# (name, what the mistake is, original text, mutated text) -- every occurrence is replaced
MUTANTS = [
    ("no_conj", "Fig. 2 l.4 read literally: F_A F_B, no conjugate (C2)",
     "FA[i] * conj(FB[i])", "FA[i] * FB[i]"),
    ("conj_on_a", "conjugate on the wrong operand: the peak lands at -d",
     "FA[i] * conj(FB[i])", "conj(FA[i]) * FB[i]"),
    ("no_zero_branch", "NCC = fc/|fc| without the zero branch (C4)",
     "c[i] = a > 0.0 ? fc / a : 0.0;", "c[i] = fc / a;"),
    ("tie_last", "argmax ties to the last index (C6)",
     "if (v > vbest) { vbest = v; best = i; }", "if (v >= vbest) { vbest = v; best = i; }"),
    ("inverse_forward", "step 4 with the forward kernel", "dft2(c, H, W, -1);", "dft2(c, H, W, +1);"),
    ("twiddle_sign", "mixed-radix combine with the conjugate twiddle",
     "                const cplx w = sign > 0 ? tab[e * step] : conj(tab[e * step]);\n"
     "                acc += w * Y",
     "                const cplx w = sign > 0 ? conj(tab[e * step]) : tab[e * step];\n"
     "                acc += w * Y"),
    ("prime_index", "naive prime DFT exponent off by one",
     "const int e = (int)(((long)j * k) % n);", "const int e = (int)(((long)j * (k + 1)) % n);"),
    ("region_rows", "candidate region one row short (Fig. 2 l.8-11)",
     "const int h = H - dy, w = W - dx;\n    *valid = 0;",
     "const int h = H - dy - 1, w = W - dx;\n    *valid = 0;"),
    ("candidate_swap", "c2 and c3 swapped (Fig. 2 l.9-10 order)",
     "{{x, y}, {W - x, y}, {x, H - y}, {W - x, H - y}}",
     "{{x, y}, {x, H - y}, {W - x, y}, {W - x, H - y}}"),
    ("ccf_tie_ge", "CCF ties to the last candidate (C7)",
     "if (valid && (best == 0 || c > best_ccf))", "if (valid && (best == 0 || c >= best_ccf))"),
    ("invalid_selected", "invalid (empty / zero-variance) candidates may win (C8)",
     "if (valid && (best == 0 || c > best_ccf))", "if ((best == 0 || c > best_ccf))"),
    ("mean_of_a", "Fig. 3 CCF with B centred on A's mean",
     "const double ma = sa / n, mb = sb / n;", "const double ma = sa / n, mb = sa / n;"),
    ("peak_unnormalised", "peak not divided by H W (C5)",
     "out->peak = vbest / (double)N;", "out->peak = vbest;"),
    ("abs_of_imag", "step 5 on the imaginary part (C3)",
     "const double v = fabs(creal(c[i]));", "const double v = fabs(cimag(c[i]));"),
    ("pair_order", "grid pairs as pciam(tile, neighbour) (C1)",
     "ncc_peak(g->spec[nb], g->spec[t], g->H, g->W, out);\n            const double peak",
     "ncc_peak(g->spec[t], g->spec[nb], g->H, g->W, out);\n            const double peak"),
    ("rows_only", "2-D transform skips the column pass",
     "    for (int x = 0; x < W; ++x) {\n        dft_rec(f + x, W, H, line, tH, H, sign, work);",
     "    for (int x = 0; x < 0; ++x) {\n        dft_rec(f + x, W, H, line, tH, H, sign, work);"),
]


def load_oracle(lib_path, name):
    """A private copy of the oracle binding bound to `lib_path` (no rebuild)."""
    spec = importlib.util.spec_from_file_location(name, os.path.join(ROOT, "oracle", "__init__.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    mod._LIB = lib_path
    mod._lib = None
    mod.build = lambda force=False: lib_path
    return mod


def compile_variant(src_text, out_dir, name):
    c = os.path.join(out_dir, f"{name}.c")
    so = os.path.join(out_dir, f"lib{name}.so")
    with open(c, "w") as f:
        f.write(src_text)
    subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-shared", "-fPIC", "-pthread",
                           "-fno-fast-math", c, "-o", so, "-lm"])
    return so


def tex(H, W, seed):
    return synthgrid.make_grid(1, 1, H, W, seed=seed).tiles[0, 0]


def naive_ccf(A, B, dx, dy):
    H, W = A.shape
    a = A[dy:H, dx:W].astype(np.float64).ravel()
    b = B[0:H - dy, 0:W - dx].astype(np.float64).ravel()
    if a.size == 0:
        return None
    a = a - a.mean()
    b = b - b.mean()
    den = np.sqrt((a * a).sum() * (b * b).sum())
    return None if den == 0 else float((a * b).sum() / den)


# ---- the pin battery: each returns normally or raises AssertionError -------------------------
def pin_dft_definition(o):
    rng = np.random.default_rng(1)
    for n in (2, 3, 5, 12, 13, 29, 58):
        x = rng.standard_normal(n) + 1j * rng.standard_normal(n)
        j = np.arange(n)
        for inv, sgn in ((False, -1), (True, 1)):
            ref = np.exp(sgn * 2j * math.pi * np.outer(j, j) / n) @ x
            assert np.abs(o.dft(x, inverse=inv) - ref).max() <= 1e-10 * np.abs(ref).max()


def pin_dft2_separable(o):
    rng = np.random.default_rng(2)
    x = rng.standard_normal((6, 10)) + 1j * rng.standard_normal((6, 10))
    assert np.abs(o.dft2(x) - np.fft.fft2(x)).max() <= 1e-10 * np.abs(x).sum()


def pin_shift_theorem(o):
    for (H, W), (dx, dy) in (((40, 48), (7, 3)), ((26, 58), (57, 25)), ((40, 48), (0, 0))):
        A = tex(H, W, 5)
        B = np.roll(A, shift=(-dy, -dx), axis=(0, 1))
        p = o.pciam(A, B)
        assert (p["peak_x"], p["peak_y"]) == (dx, dy)
        assert abs(p["peak"] - 1.0) <= 1e-12
        s = o.surface(A, B)
        assert abs(s[dy, dx] - 1.0) <= 1e-12


def pin_zero_tile(o):
    for H, W in ((3, 4), (40, 48)):
        A = tex(H, W, 6)
        B = np.zeros((H, W), np.uint16)
        for a, b in ((A, B), (B, A)):
            assert np.all(o.surface(a, b) == 0.0)
            p = o.pciam(a, b)
            assert (p["peak_x"], p["peak_y"]) == (0, 0) and p["peak"] == 0.0
            assert p["candidate"] == 0 and np.isnan(p["ccf"])


def pin_ccf_identities(o):
    H, W = 40, 48
    A = tex(H, W, 7).astype(np.int64) // 8
    c, v = o.ccf(A.astype(np.uint16), A.astype(np.uint16), 0, 0)
    assert v and abs(c - 1.0) <= 1e-12
    for dx, dy in ((5, 3), (30, 20)):
        B = np.zeros((H, W), np.int64)
        B[0:H - dy, 0:W - dx] = 3 * A[dy:, dx:] + 100
        c, v = o.ccf(A.astype(np.uint16), B.astype(np.uint16), dx, dy)
        assert v and abs(c - 1.0) <= 1e-12
    A, B = tex(H, W, 8), tex(H, W, 9)
    for dx, dy in ((0, 0), (31, 22), (46, 38)):
        c, v = o.ccf(A, B, dx, dy)
        nv = naive_ccf(A, B, dx, dy)
        assert v == (nv is not None) and (not v or abs(c - nv) <= 1e-12)


def pin_candidate_rules(o):
    H, W = 40, 48
    A = tex(H, W, 10)
    p = o.eval_peak(A, A, 0, 0)
    assert p["candidate"] == 1 and (p["dx"], p["dy"]) == (0, 0) and abs(p["ccf"] - 1) <= 1e-12
    p = o.eval_peak(A, tex(H, W, 11), W // 2, H // 2)
    assert p["candidate"] == 1
    B = tex(H, W, 12)
    for x, y in ((5, 7), (40, 3), (11, 35)):
        p = o.eval_peak(A, B, x, y)
        cands = [(x, y), (W - x, y), (x, H - y), (W - x, H - y)]
        vals = [naive_ccf(A, B, dx, dy) for dx, dy in cands]
        k = -max((v, -i) for i, v in enumerate(vals) if v is not None)[1]
        assert p["candidate"] == k + 1 and (p["dx"], p["dy"]) == cands[k]
        assert abs(p["ccf"] - vals[k]) <= 1e-12


def pin_brute_force_ncc(o):
    g = synthgrid.make_grid(2, 2, 26, 58, overlap=0.5, delta=2, seed=12)
    tw = g.true_west()
    A, B = g.tiles[0, 0], g.tiles[0, 1]
    p = o.pciam(A, B)
    assert (p["dx"], p["dy"]) == (int(tw[0][0, 1]), int(tw[1][0, 1]))


def pin_grid_recovery(o):
    g = synthgrid.make_config(1)
    west, north = o.grid(g.tiles)
    tw, tn = g.true_west(), g.true_north()
    assert np.array_equal(west["dx"][:, 1:], tw[0][:, 1:])
    assert np.array_equal(west["dy"][:, 1:], tw[1][:, 1:])
    assert np.array_equal(north["dx"][1:], tn[0][1:])
    assert np.array_equal(north["dy"][1:], tn[1][1:])
    assert (west["candidate"][:, 1:] == 1).all() and (north["candidate"][1:] == 1).all()


PINS = [pin_dft_definition, pin_dft2_separable, pin_shift_theorem, pin_zero_tile,
        pin_ccf_identities, pin_candidate_rules, pin_brute_force_ncc, pin_grid_recovery]


def run_pins(o):
    failed = []
    for pin in PINS:
        try:
            pin(o)
        except (AssertionError, FloatingPointError, ValueError) as e:  # noqa: PERF203
            failed.append((pin.__name__, str(e)[:80]))
    return failed


@pytest.fixture(scope="module")
def source():
    return open(SRC).read()


def test_unmodified_oracle_passes_the_battery(source, tmp_path):
    o = load_oracle(compile_variant(source, str(tmp_path), "orig"), "oracle_orig")
    assert run_pins(o) == []


@pytest.mark.parametrize("name,why,old,new", MUTANTS, ids=[m[0] for m in MUTANTS])
def test_every_plausible_mistake_fails_a_pin(source, tmp_path, name, why, old, new):
    assert source.count(old) >= 1, f"mutation site of {name} not found: {old!r}"
    o = load_oracle(compile_variant(source.replace(old, new), str(tmp_path), name),
                    f"oracle_{name}")
    failed = run_pins(o)
    assert failed, f"mutant {name} ({why}) passes every pin"
