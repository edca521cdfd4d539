#!/usr/bin/env python3
"""Generate straight-line fp32 and fp64 DFT codelets (codelets.cuh) for the CUDA FFT engine.

Each codelet computes, in registers, an unnormalised length-R DFT
    X[k] = sum_j x[j] exp(SIGN * 2 pi i j k / R),   SIGN = -1 (forward) or +1 (inverse)
in place on a float2[R] array.  Primes use the symmetric (x_j +- x_{R-j}) form,
composites a split R = R1*R2: prime-factor (Good-Thomas, index maps only, no twiddles)
when R1 and R2 are coprime, else Cooley-Tukey with constant twiddles (trivial ones --
multiples of pi/4 -- special-cased).  Constants are computed in double here and
rounded once to float literals (fp32) or kept as double literals (fp64 path, f2: the same
straight-line program with every float replaced by double).

This is part of the CUDA product path only (it shares nothing with oracle/).
Run:  python gen_codelets.py > codelets.cuh
"""
import math
import re
import sys

RADICES = [2, 3, 4, 5, 6, 8, 10, 12, 13, 16, 20, 24, 26, 29, 40]


def flit(x: float) -> str:
    if x == 0.0:
        return "0.0f"
    s = repr(float(x))
    if "e" not in s and "." not in s:
        s += ".0"
    return f"({s}f)"


class Em:
    def __init__(self):
        self.lines = []
        self.n = 0

    def let(self, expr: str) -> str:
        self.n += 1
        name = f"t{self.n}"
        self.lines.append(f"    const float {name} = {expr};")
        return name


def cadd(e, a, b):
    return (e.let(f"{a[0]} + {b[0]}"), e.let(f"{a[1]} + {b[1]}"))


def csub(e, a, b):
    return (e.let(f"{a[0]} - {b[0]}"), e.let(f"{a[1]} - {b[1]}"))


def twiddle(e, a, num, den, sign):
    """a * exp(sign * 2 pi i num / den)."""
    num %= den
    if num == 0:
        return a
    g = math.gcd(num, den)
    num //= g
    den //= g
    if den == 2:                       # -1
        return (e.let(f"-{a[0]}"), e.let(f"-{a[1]}"))
    if den == 4:                       # (sign i)^num
        q = num if sign > 0 else (4 - num) % 4   # exponent of +i
        if q == 1:                     # i * a = (-a.im, a.re)
            return (e.let(f"-{a[1]}"), a[0])
        if q == 3:                     # -i * a = (a.im, -a.re)
            return (a[1], e.let(f"-{a[0]}"))
    ang = sign * 2.0 * math.pi * num / den
    c, s = math.cos(ang), math.sin(ang)
    if den == 8:                       # (+-1 +- i)/sqrt2
        h = flit(math.sqrt(0.5))
        cs, ss = (1 if c > 0 else -1), (1 if s > 0 else -1)
        # re = a.re*c - a.im*s ; im = a.re*s + a.im*c
        re = e.let(f"{h} * ({'' if cs > 0 else '-'}{a[0]} {'-' if ss > 0 else '+'} {a[1]})")
        im = e.let(f"{h} * ({'' if ss > 0 else '-'}{a[0]} {'+' if cs > 0 else '-'} {a[1]})")
        return (re, im)
    re = e.let(f"fmaf({a[0]}, {flit(c)}, -({a[1]} * {flit(s)}))")
    im = e.let(f"fmaf({a[0]}, {flit(s)}, {a[1]} * {flit(c)})")
    return (re, im)


_BEST = {}


def _cost(n, sp):
    """Instruction count of the codelet for n when its top-level split is sp."""
    e = Em()
    xs = [(f"x{j}r", f"x{j}i") for j in range(n)]
    _FORCE[n] = sp
    try:
        gen(e, xs, -1)
    finally:
        del _FORCE[n]
    # one instruction per line; a product inside an fmaf argument and a scaled sum
    # "h * (a +- b)" (an add and a multiply) count one more
    return sum(1 + l.count(" * ") * ("fmaf(" in l) + (" * (" in l) for l in e.lines
               if not (l.count("= -t") and l.count("t") == 2))


_FORCE = {}


def split(n):
    """Split n = n1 * n2 of a composite radix (prime-factor / Good-Thomas when the factors
    are coprime, Cooley-Tukey with twiddles otherwise), chosen (recursively, memoised) to
    minimise the straight-line instruction count; None for a prime."""
    if n in _FORCE:
        return _FORCE[n]
    divs = [d for d in range(2, n) if n % d == 0]
    if not divs:
        return None
    if n not in _BEST:
        _BEST[n] = min(((d, n // d) for d in divs), key=lambda sp: (_cost(n, sp), sp))
    return _BEST[n]


def primitive_root(p):
    for g in range(2, p):
        if all(pow(g, (p - 1) // q, p) != 1 for q in range(2, p) if (p - 1) % q == 0
               and all(q % r for r in range(2, q))):
            return g
    raise ValueError(p)


def prime_rader(e, xs, sign):
    """Prime p with h = (p-1)/2 even: symmetric form with the cosine half evaluated as a
    cyclic correlation of length h (Rader ordering j = g^a, k = g^-b; C_m = cos(2 pi g^m/p)
    is h-periodic) split by CRT into a cyclic and a negacyclic correlation of length h/2:
    126 instead of 196 FMAs per component at p = 29.  The sine half (anti-periodic, a
    negacyclic correlation) stays direct."""
    n = len(xs)
    h = (n - 1) // 2
    g = primitive_root(n)
    ja = [pow(g, a, n) for a in range(h)]                    # representatives of +-j
    kb = [pow(g, (n - 1 - b) % (n - 1), n) for b in range(h)]  # g^-b
    s = [cadd(e, xs[j], xs[n - j]) for j in ja]
    d = [csub(e, xs[j], xs[n - j]) for j in ja]
    q = h // 2
    up = [[e.let(f"{s[a][c]} + {s[a + q][c]}") for a in range(q)] for c in (0, 1)]
    um = [[e.let(f"{s[a][c]} - {s[a + q][c]}") for a in range(q)] for c in (0, 1)]
    out = [None] * n
    acc = xs[0]                        # X_0 = x_0 + sum of the q pair sums up_a
    for a in range(q):
        acc = (e.let(f"{acc[0]} + {up[0][a]}"), e.let(f"{acc[1]} + {up[1][a]}"))
    out[0] = acc
    C = [math.cos(2.0 * math.pi * pow(g, m, n) / n) for m in range(h)]
    P = [0.5 * (C[m] + C[(m + q) % h]) for m in range(q)]    # period q
    Nm = [0.5 * (C[m] - C[(m + q) % h]) for m in range(h)]   # anti-periodic (q), index mod h
    A = [[None, None] for _ in range(h)]
    for comp in (0, 1):
        for b in range(q):
            pp = xs[0][comp]
            for a in range(q):
                pp = e.let(f"fmaf({up[comp][a]}, {flit(P[(a - b) % q])}, {pp})")
            ap = pp                            # A_b = pp + nn, the nn chain started from pp
            for a in range(q):
                m = a - b                      # N_{a-b}: N_{m+q} = -N_m
                c = Nm[m] if m >= 0 else -Nm[m + q]
                ap = e.let(f"fmaf({um[comp][a]}, {flit(c)}, {ap})")
            A[b][comp] = ap
            A[b + q][comp] = e.let(f"fmaf({pp}, {flit(2.0)}, -{ap})")   # pp - nn
    # Sine half: B = T d with T[b][a] = S(a - b), S(m) = sin(2 pi g^m / p), S(m + h) = -S(m).
    # In q x q blocks T = [[A, C], [-C, A]] (A = S(a0 - b0), C = S(a0 - b0 + q)), i.e. the
    # product (A - iC)(u + iv) of the halves u, v of d; three block products, two of them
    # started from the previous result so the block sums cost no separate adds:
    #   t1 = A u,  y0 = C v + t1,  y1 = (A - C)(u + v) + (y0 - 2 t1)  [= A v - C u].
    def S(m):
        return math.sin(2.0 * math.pi * pow(g, m % (n - 1), n) / n)
    Bv = [[None, None] for _ in range(h)]
    for comp in (0, 1):
        u = [d[a][comp] for a in range(q)]
        v = [d[a + q][comp] for a in range(q)]
        uv = [e.let(f"{u[a]} + {v[a]}") for a in range(q)]
        for b in range(q):
            t1 = None
            for a in range(q):
                c = S(a - b)
                t1 = e.let(f"{u[a]} * {flit(c)}") if t1 is None else \
                    e.let(f"fmaf({u[a]}, {flit(c)}, {t1})")
            y0 = t1
            for a in range(q):
                y0 = e.let(f"fmaf({v[a]}, {flit(S(a - b + q))}, {y0})")
            y1 = e.let(f"fmaf({t1}, {flit(-2.0)}, {y0})")
            for a in range(q):
                y1 = e.let(f"fmaf({uv[a]}, {flit(S(a - b) - S(a - b + q))}, {y1})")
            Bv[b][comp] = y0
            Bv[b + q][comp] = y1
    for b in range(h):
        k = kb[b]
        br, bi = Bv[b]
        ar, ai = A[b]
        if sign < 0:
            out[k] = (e.let(f"{ar} + {bi}"), e.let(f"{ai} - {br}"))
            out[n - k] = (e.let(f"{ar} - {bi}"), e.let(f"{ai} + {br}"))
        else:
            out[k] = (e.let(f"{ar} - {bi}"), e.let(f"{ai} + {br}"))
            out[n - k] = (e.let(f"{ar} + {bi}"), e.let(f"{ai} - {br}"))
    return out


RADER_MIN = 13   # primes from here use prime_rader (h even); smaller ones the plain form


def gen(e, xs, sign):
    n = len(xs)
    if n == 1:
        return list(xs)
    if n == 2:
        return [cadd(e, xs[0], xs[1]), csub(e, xs[0], xs[1])]
    sp = split(n)
    if sp is None and n >= RADER_MIN and ((n - 1) // 2) % 2 == 0:
        return prime_rader(e, xs, sign)
    if sp is None:                     # prime: symmetric form
        h = (n - 1) // 2
        s = [None] + [cadd(e, xs[j], xs[n - j]) for j in range(1, h + 1)]
        d = [None] + [csub(e, xs[j], xs[n - j]) for j in range(1, h + 1)]
        out = [None] * n
        acc = xs[0]
        for j in range(1, h + 1):
            acc = cadd(e, acc, s[j])
        out[0] = acc
        for k in range(1, h + 1):
            ar, ai = xs[0]
            br, bi = None, None
            if h == 1:                 # n = 3: the single sine product fused into the outputs
                m = k % n
                c = math.cos(2.0 * math.pi * m / n)
                sn = math.sin(2.0 * math.pi * m / n) * (1 if sign < 0 else -1)
                ar = e.let(f"fmaf({s[1][0]}, {flit(c)}, {ar})")
                ai = e.let(f"fmaf({s[1][1]}, {flit(c)}, {ai})")
                # X_k = A + sign i B, B = sn d:  (ar + sn d.im, ai - sn d.re) for sign < 0
                out[k] = (e.let(f"fmaf({d[1][1]}, {flit(sn)}, {ar})"),
                          e.let(f"fmaf({d[1][0]}, {flit(-sn)}, {ai})"))
                out[n - k] = (e.let(f"fmaf({d[1][1]}, {flit(-sn)}, {ar})"),
                              e.let(f"fmaf({d[1][0]}, {flit(sn)}, {ai})"))
                continue
            for j in range(1, h + 1):
                c = math.cos(2.0 * math.pi * ((j * k) % n) / n)
                ar = e.let(f"fmaf({s[j][0]}, {flit(c)}, {ar})")
                ai = e.let(f"fmaf({s[j][1]}, {flit(c)}, {ai})")
            # B = sum_j sn_j d_j = sn_0 * (d_j0 + sum_{j != j0} (sn_j / sn_j0) d_j), j0 the
            # largest |sn_j|: the inner sum starts from d_j0 and the common factor goes into
            # the two output FMAs (X_k = A + sign i B, X_{n-k} = A - sign i B, i B = (-B.im, B.re))
            sn = [None] + [math.sin(2.0 * math.pi * ((j * k) % n) / n) for j in range(1, h + 1)]
            j0 = max(range(1, h + 1), key=lambda j: abs(sn[j]))
            ir, ii = d[j0]
            for j in range(1, h + 1):
                if j != j0:
                    r = sn[j] / sn[j0]
                    ir = e.let(f"fmaf({d[j][0]}, {flit(r)}, {ir})")
                    ii = e.let(f"fmaf({d[j][1]}, {flit(r)}, {ii})")
            f = sn[j0] if sign < 0 else -sn[j0]
            out[k] = (e.let(f"fmaf({ii}, {flit(f)}, {ar})"), e.let(f"fmaf({ir}, {flit(-f)}, {ai})"))
            out[n - k] = (e.let(f"fmaf({ii}, {flit(-f)}, {ar})"),
                          e.let(f"fmaf({ir}, {flit(f)}, {ai})"))
        return out
    n1, n2 = sp
    if math.gcd(n1, n2) == 1:
        # Good-Thomas prime-factor split: no twiddles.  Input map (Ruritanian)
        # j = (n2*a + n1*b) mod n, output map (CRT) k = (n2*u*k1 + n1*w*k2) mod n with
        # u = n2^-1 mod n1, w = n1^-1 mod n2, so that exp(2 pi i j k / n) =
        # exp(2 pi i a k1 / n1) exp(2 pi i b k2 / n2): a 2-D DFT with no cross term.
        u, w = pow(n2, -1, n1), pow(n1, -1, n2)
        Y = [gen(e, [xs[(n2 * a + n1 * b) % n] for a in range(n1)], sign) for b in range(n2)]
        out = [None] * n
        for k1 in range(n1):
            X = gen(e, [Y[b][k1] for b in range(n2)], sign)
            for k2 in range(n2):
                out[(n2 * u * k1 + n1 * w * k2) % n] = X[k2]
        return out
    # x index j = n2*a + b ; X index k = k1 + n1*k2
    Y = [gen(e, [xs[n2 * a + b] for a in range(n1)], sign) for b in range(n2)]
    out = [None] * n
    for k1 in range(n1):
        if n2 == 2 and pi4_twiddle(k1, n):
            # outer radix 2 after a (+-1 +- i)/sqrt2 twiddle: X = Y0 +- h t with t the
            # unscaled rotation of Y1 (two adds), the scale h folded into the output FMAs
            y0, y1 = Y[0][k1], Y[1][k1]
            ang = sign * 2.0 * math.pi * k1 / n
            cs, ss = (1 if math.cos(ang) > 0 else -1), (1 if math.sin(ang) > 0 else -1)
            tr = e.let(f"{'' if cs > 0 else '-'}{y1[0]} {'-' if ss > 0 else '+'} {y1[1]}")
            ti = e.let(f"{'' if ss > 0 else '-'}{y1[0]} {'+' if cs > 0 else '-'} {y1[1]}")
            h = flit(math.sqrt(0.5))
            hm = flit(-math.sqrt(0.5))
            out[k1] = (e.let(f"fmaf({tr}, {h}, {y0[0]})"), e.let(f"fmaf({ti}, {h}, {y0[1]})"))
            out[k1 + n1] = (e.let(f"fmaf({tr}, {hm}, {y0[0]})"), e.let(f"fmaf({ti}, {hm}, {y0[1]})"))
            continue
        X = gen(e, [twiddle(e, Y[b][k1], b * k1, n, sign) for b in range(n2)], sign)
        for k2 in range(n2):
            out[k1 + n1 * k2] = X[k2]
    return out


def pi4_twiddle(num, den):
    """exp(+-2 pi i num/den) is an odd multiple of pi/4."""
    num %= den
    if num == 0:
        return False
    g = math.gcd(num, den)
    return den // g == 8


# ---------------------------------------------------------------------------------------
# Packed fp32 codelets (sm_100a FADD2 / FMUL2 / FFMA2, f32x2.cuh): the same algorithms at the
# level of complex values.  Every complex add, complex x real constant, and complex fma with a
# real constant is ONE packed instruction (the scalar codelets above spend two), and a
# multiplication by a power of i is free: a value is (name, r) meaning i^r * name, emitted as
# the operand view name / I(name) / NEG(name) / MI(name) that ptxas folds into the packed
# instruction's source selectors.

class PEm:
    def __init__(self):
        self.lines = []
        self.n = 0

    def new(self, expr: str):
        self.n += 1
        name = f"t{self.n}"
        self.lines.append(f"    const float2 {name} = {expr};")
        return (name, 0)


def pop(v):
    name, r = v
    return (name, f"I({name})", f"NEG({name})", f"MI({name})")[r % 4]


def prot(v, k):
    """i^k * v (free)."""
    return (v[0], (v[1] + k) % 4)


def padd(e, a, b):
    return e.new(f"f2add({pop(a)}, {pop(b)})")


def psub(e, a, b):
    return e.new(f"f2sub({pop(a)}, {pop(b)})")


def pmul(e, a, c):
    return e.new(f"f2mul({pop(a)}, K({flit(c)}))")


def pfma(e, a, c, acc):
    """a * c + acc, c real."""
    return e.new(f"f2fma({pop(a)}, K({flit(c)}), {pop(acc)})")


def ptwiddle(e, a, num, den, sign):
    """a * exp(sign * 2 pi i num / den)."""
    num %= den
    if num == 0:
        return a
    g = math.gcd(num, den)
    num //= g
    den //= g
    if den == 2:
        return prot(a, 2)
    if den == 4:
        return prot(a, num if sign > 0 else (4 - num) % 4)
    ang = sign * 2.0 * math.pi * num / den
    c, s = math.cos(ang), math.sin(ang)
    if den == 8:                       # sqrt(1/2) (+-a +- i a)
        t = padd(e, prot(a, 0 if c > 0 else 2), prot(a, 1 if s > 0 else 3))
        return pmul(e, t, math.sqrt(0.5))
    return pfma(e, prot(a, 1), s, pmul(e, a, c))        # a c + (i a) s


def pprime_rader(e, xs, sign):
    """prime_rader on complex values (same Rader / CRT structure, one packed op per step)."""
    n = len(xs)
    h = (n - 1) // 2
    g = primitive_root(n)
    ja = [pow(g, a, n) for a in range(h)]
    kb = [pow(g, (n - 1 - b) % (n - 1), n) for b in range(h)]
    s = [padd(e, xs[j], xs[n - j]) for j in ja]
    d = [psub(e, xs[j], xs[n - j]) for j in ja]
    q = h // 2
    up = [padd(e, s[a], s[a + q]) for a in range(q)]
    um = [psub(e, s[a], s[a + q]) for a in range(q)]
    out = [None] * n
    acc = xs[0]
    for a in range(q):
        acc = padd(e, acc, up[a])
    out[0] = acc
    C = [math.cos(2.0 * math.pi * pow(g, m, n) / n) for m in range(h)]
    P = [0.5 * (C[m] + C[(m + q) % h]) for m in range(q)]
    Nm = [0.5 * (C[m] - C[(m + q) % h]) for m in range(h)]
    A = [None] * h
    for b in range(q):
        pp = xs[0]
        for a in range(q):
            pp = pfma(e, up[a], P[(a - b) % q], pp)
        ap = pp
        for a in range(q):
            m = a - b
            ap = pfma(e, um[a], Nm[m] if m >= 0 else -Nm[m + q], ap)
        A[b] = ap
        A[b + q] = pfma(e, pp, 2.0, prot(ap, 2))          # pp - nn

    def S(m):
        return math.sin(2.0 * math.pi * pow(g, m % (n - 1), n) / n)
    u = [d[a] for a in range(q)]
    v = [d[a + q] for a in range(q)]
    uv = [padd(e, u[a], v[a]) for a in range(q)]
    Bv = [None] * h
    for b in range(q):
        t1 = None
        for a in range(q):
            t1 = pmul(e, u[a], S(a - b)) if t1 is None else pfma(e, u[a], S(a - b), t1)
        y0 = t1
        for a in range(q):
            y0 = pfma(e, v[a], S(a - b + q), y0)
        y1 = pfma(e, t1, -2.0, y0)
        for a in range(q):
            y1 = pfma(e, uv[a], S(a - b) - S(a - b + q), y1)
        Bv[b] = y0
        Bv[b + q] = y1
    for b in range(h):                 # X_k = A - sign i B... as the scalar form:
        k = kb[b]                      # sign < 0: X_k = A - i B, X_{n-k} = A + i B
        lo, hi = (3, 1) if sign < 0 else (1, 3)
        out[k] = padd(e, A[b], prot(Bv[b], lo))
        out[n - k] = padd(e, A[b], prot(Bv[b], hi))
    return out


def pgen(e, xs, sign):
    n = len(xs)
    if n == 1:
        return list(xs)
    if n == 2:
        return [padd(e, xs[0], xs[1]), psub(e, xs[0], xs[1])]
    sp = psplit(n)
    if sp is None and n >= RADER_MIN and ((n - 1) // 2) % 2 == 0:
        return pprime_rader(e, xs, sign)
    if sp is None:                     # prime: symmetric form
        h = (n - 1) // 2
        s = [None] + [padd(e, xs[j], xs[n - j]) for j in range(1, h + 1)]
        d = [None] + [psub(e, xs[j], xs[n - j]) for j in range(1, h + 1)]
        out = [None] * n
        acc = xs[0]
        for j in range(1, h + 1):
            acc = padd(e, acc, s[j])
        out[0] = acc
        for k in range(1, h + 1):
            if h == 1:                 # n = 3
                c = math.cos(2.0 * math.pi * k / n)
                sn = math.sin(2.0 * math.pi * k / n) * (1 if sign < 0 else -1)
                A = pfma(e, s[1], c, xs[0])
                out[k] = pfma(e, prot(d[1], 3), sn, A)          # A + sn (-i d)
                out[n - k] = pfma(e, prot(d[1], 3), -sn, A)
                continue
            A = xs[0]
            for j in range(1, h + 1):
                A = pfma(e, s[j], math.cos(2.0 * math.pi * ((j * k) % n) / n), A)
            sn = [None] + [math.sin(2.0 * math.pi * ((j * k) % n) / n) for j in range(1, h + 1)]
            j0 = max(range(1, h + 1), key=lambda j: abs(sn[j]))
            Iv = d[j0]
            for j in range(1, h + 1):
                if j != j0:
                    Iv = pfma(e, d[j], sn[j] / sn[j0], Iv)
            f = sn[j0] if sign < 0 else -sn[j0]
            out[k] = pfma(e, prot(Iv, 3), f, A)                  # A + f (-i I)
            out[n - k] = pfma(e, prot(Iv, 3), -f, A)
        return out
    n1, n2 = sp
    if math.gcd(n1, n2) == 1:
        u, w = pow(n2, -1, n1), pow(n1, -1, n2)
        Y = [pgen(e, [xs[(n2 * a + n1 * b) % n] for a in range(n1)], sign) for b in range(n2)]
        out = [None] * n
        for k1 in range(n1):
            X = pgen(e, [Y[b][k1] for b in range(n2)], sign)
            for k2 in range(n2):
                out[(n2 * u * k1 + n1 * w * k2) % n] = X[k2]
        return out
    Y = [pgen(e, [xs[n2 * a + b] for a in range(n1)], sign) for b in range(n2)]
    out = [None] * n
    for k1 in range(n1):
        if n2 == 2 and pi4_twiddle(k1, n):
            y0, y1 = Y[0][k1], Y[1][k1]
            ang = sign * 2.0 * math.pi * k1 / n
            cs, ss = (1 if math.cos(ang) > 0 else -1), (1 if math.sin(ang) > 0 else -1)
            t = padd(e, prot(y1, 0 if cs > 0 else 2), prot(y1, 1 if ss > 0 else 3))
            out[k1] = pfma(e, t, math.sqrt(0.5), y0)
            out[k1 + n1] = pfma(e, t, -math.sqrt(0.5), y0)
            continue
        X = pgen(e, [ptwiddle(e, Y[b][k1], b * k1, n, sign) for b in range(n2)], sign)
        for k2 in range(n2):
            out[k1 + n1 * k2] = X[k2]
    return out


_PBEST = {}
_PFORCE = {}


def psplit(n):
    """split() for the packed codelets (instruction count = emitted operations)."""
    if n in _PFORCE:
        return _PFORCE[n]
    divs = [d for d in range(2, n) if n % d == 0]
    if not divs:
        return None
    if n not in _PBEST:
        def cost(sp):
            e = PEm()
            _PFORCE[n] = sp
            try:
                outs = pgen(e, [(f"x{j}", 0) for j in range(n)], -1)
            finally:
                del _PFORCE[n]
            return len(e.lines) + sum(1 for o in outs if o[1] % 4)
        _PBEST[n] = min(((d, n // d) for d in divs), key=lambda sp: (cost(sp), sp))
    return _PBEST[n]


def codelet_packed(n, sign):
    e = PEm()
    outs = pgen(e, [(f"x{j}", 0) for j in range(n)], sign)
    tag = "m" if sign < 0 else "p"
    lines = [f"__device__ __forceinline__ void dft{n}{tag}(float2* __restrict__ v) {{"]
    for j in range(n):
        lines.append(f"    const float2 x{j} = v[{j}];")
    lines += e.lines
    for k in range(n):
        lines.append(f"    v[{k}] = {pop(outs[k])};")
    lines.append("}")
    return "\n".join(lines)


def codelet(n, sign):
    e = Em()
    xs = []
    for j in range(n):
        xs.append((f"x{j}r", f"x{j}i"))
    outs = gen(e, xs, sign)
    tag = "m" if sign < 0 else "p"
    lines = [f"__device__ __forceinline__ void dft{n}{tag}(float2* __restrict__ v) {{"]
    for j in range(n):
        lines.append(f"    const float x{j}r = v[{j}].x, x{j}i = v[{j}].y;")
    lines += e.lines
    for k in range(n):
        lines.append(f"    v[{k}] = make_float2({outs[k][0]}, {outs[k][1]});")
    lines.append("}")
    return "\n".join(lines)


_FLIT = re.compile(r"\(([-+0-9.e]+)f\)")


def to_double(src: str) -> str:
    """The fp64 twin of an fp32 codelet: double temporaries, fma, full-precision literals
    (flit printed the double constant before appending 'f')."""
    src = src.replace("const float ", "const double ").replace("fmaf(", "fma(")
    src = src.replace("float2*", "double2*").replace("make_float2(", "make_double2(")
    src = re.sub(r"void dft(\d+)([mp])\(", r"void dft\1\2_d(", src)
    src = _FLIT.sub(r"(\1)", src)
    return src.replace("0.0f", "0.0")


def main():
    out = ["// GENERATED by gen_codelets.py -- do not edit.",
           "// Straight-line fp32 / fp64 DFT codelets: v[k] <- sum_j v[j] exp(SIGN 2 pi i j k / R).",
           "// fp32: packed complex operations (f32x2.cuh); fp64: scalar double.",
           "#pragma once", "", '#include "f32x2.cuh"', "", "namespace stitch {", "",
           "template <int R, int SIGN> struct Dft;", ""]
    for r in RADICES:
        for sign in (-1, 1):
            out.append(codelet_packed(r, sign))         # fp32: packed f32x2
            out.append(to_double(codelet(r, sign)))     # fp64 (f2): the scalar program in double
            tag = "m" if sign < 0 else "p"
            out.append(f"template <> struct Dft<{r}, {sign}> {{\n"
                       f"    static __device__ __forceinline__ void run(float2* v) {{ dft{r}{tag}(v); }}\n"
                       f"    static __device__ __forceinline__ void run(double2* v) {{ dft{r}{tag}_d(v); }}\n"
                       f"}};")
            out.append("")
    out.append("}  // namespace stitch")
    sys.stdout.write("\n".join(out) + "\n")


if __name__ == "__main__":
    main()
