/*
 * oracle.c — PCIAM relative-displacement ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may
 * load or call this library.  The product (CUDA) path never does, and this
 * file shares no code, header, table or constant with it.
 *
 * Plain, slow, obviously-correct CPU implementation in double precision
 * (the paper's own precision: "double complex" transforms, PAPER.md L576;
 * the CCF returns a double, Fig. 3).  No FFT library, no
 * SIMD intrinsics.  Every step cites the passage it follows:
 *
 *   P:L494      step 2  forward 2-D Fourier transform of each image
 *   P:L496-500  step 3  NCC = element-wise normalised conjugate product
 *   P:L502-504  step 4  2-D inverse Fourier transform of the NCC
 *   P:L506-512  step 5  max of abs of the inverse, mapped to (x, y)
 *   P:L512-516  step 6  CCF of the four overlap modes (x|W-x, y|H-y)
 *   P:L518      step 7  max CCF, mapped back to (x, y)
 *   Fig. 2 pciam(Ii, Ij) pseudo-code, Fig. 3 ccf,
 *   Fig. 4 the grid of west/north pairs.
 *
 * Readings where the paper is silent or garbled (DESIGN.md "Readings" C1-C10):
 *   C1 both pair kinds are pciam(neighbour, tile): A = west/north tile, B = tile.
 *   C2 the product is F_A * conj(F_B) (the text's "conjugate multiplication";
 *      Fig. 2 l.4 drops the conj); forward kernel e^{-i}, inverse e^{+i}.
 *   C3 abs of the real part of the C2C inverse (its imaginary part is ~0).
 *   C4 NCC = 0 where |F_A conj(F_B)| = 0.
 *   C5 the inverse is unnormalised; the reported peak is max / (H W).
 *   C6 argmax ties -> smallest row-major index y*W + x.
 *   C7 CCF ties -> first of c1..c4 (Fig. 2 l.12 order).
 *   C8 an empty region (dx = W or dy = H) or a zero variance makes that
 *      candidate invalid; none valid -> candidate 0, (dx,dy) = peak, ccf NaN.
 *
 * Parity pins: tests/test_oracle_*.py (brute-force DFT definition, Parseval,
 * linearity, closed forms, shift theorem, CCF identities, brute-force spatial
 * NCC, exact recovery of known synthetic shifts).
 */
#include <complex.h>
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef double complex cplx;

/* ---------------------------------------------------------------- DFT --- */

/* Table of the N-th roots of unity: tab[e] = exp(-2 pi i e / N).
 * W_n^e for any n | N is tab[e * (N / n) mod N]. */
static cplx* roots_table(int N) {
    cplx* t = (cplx*)malloc(sizeof(cplx) * (size_t)N);
    for (int e = 0; e < N; ++e) {
        const double a = -2.0 * M_PI * (double)e / (double)N;
        t[e] = cos(a) + I * sin(a);
    }
    return t;
}

static int smallest_prime_factor(int n) {
    for (int p = 2; p * p <= n; ++p)
        if (n % p == 0) return p;
    return n;
}

/*
 * Recursive mixed-radix Cooley-Tukey DFT, decimation in time.
 *   X[k] = sum_{j<n} x[j*stride] * W_n^{sign * j k},  W_n = exp(-2 pi i / n)
 * (sign = +1 forward e^{-i}, sign = -1 inverse e^{+i}, unnormalised).
 * n = p * M with p the smallest prime factor:
 *   Y_r[k] = DFT_M of the decimated sequence x[(p m + r) * stride], m < M
 *   X[k + M q] = sum_{r<p} W_n^{r (k + M q)} Y_r[k]
 * and a prime n is evaluated straight from the definition.
 * `tab` holds the roots of the top-level length N0 (n | N0); `work` has room
 * for 2n values at this level and below.
 */
static void dft_rec(const cplx* x, long stride, int n, cplx* X, const cplx* tab, int N0,
                    int sign, cplx* work) {
    const int step = N0 / n;  /* W_n^e = tab[e * step] */
    if (n == 1) {
        X[0] = x[0];
        return;
    }
    const int p = smallest_prime_factor(n);
    if (p == n) {             /* prime length: the definition */
        for (int k = 0; k < n; ++k) {
            cplx acc = 0;
            for (int j = 0; j < n; ++j) {
                const int e = (int)(((long)j * k) % n);
                const cplx w = sign > 0 ? tab[e * step] : conj(tab[e * step]);
                acc += x[(long)j * stride] * w;
            }
            X[k] = acc;
        }
        return;
    }
    const int M = n / p;
    cplx* Y = work;           /* Y[r*M + k] */
    for (int r = 0; r < p; ++r)
        dft_rec(x + (long)r * stride, stride * p, M, Y + (long)r * M, tab, N0, sign, work + n);
    for (int q = 0; q < p; ++q) {
        for (int k = 0; k < M; ++k) {
            const int kk = k + M * q;
            cplx acc = 0;
            for (int r = 0; r < p; ++r) {
                const int e = (int)(((long)r * kk) % n);
                const cplx w = sign > 0 ? tab[e * step] : conj(tab[e * step]);
                acc += w * Y[(long)r * M + k];
            }
            X[kk] = acc;
        }
    }
}

/* 1-D DFT of length n (exported for the pins).  sign = +1 forward, -1 inverse. */
void oracle_dft(const double* in_ri, double* out_ri, int n, int sign) {
    cplx* x = (cplx*)malloc(sizeof(cplx) * (size_t)n);
    cplx* X = (cplx*)malloc(sizeof(cplx) * (size_t)n);
    cplx* work = (cplx*)malloc(sizeof(cplx) * (size_t)(4 * n + 8));
    cplx* tab = roots_table(n);
    for (int i = 0; i < n; ++i) x[i] = in_ri[2 * i] + I * in_ri[2 * i + 1];
    dft_rec(x, 1, n, X, tab, n, sign, work);
    for (int i = 0; i < n; ++i) {
        out_ri[2 * i] = creal(X[i]);
        out_ri[2 * i + 1] = cimag(X[i]);
    }
    free(x); free(X); free(work); free(tab);
}

/*
 * Full 2-D C2C DFT of an H x W complex array (row-major, W contiguous):
 *   F(ky, kx) = sum_y sum_x f(y, x) exp(-+ 2 pi i (ky y / H + kx x / W))
 * rows first (along x), then columns (along y).  In place.
 */
static void dft2(cplx* f, int H, int W, int sign) {
    const int L = H > W ? H : W;
    cplx* line = (cplx*)malloc(sizeof(cplx) * (size_t)L);
    cplx* work = (cplx*)malloc(sizeof(cplx) * (size_t)(4 * L + 8));
    cplx* tW = roots_table(W);
    cplx* tH = roots_table(H);
    for (int y = 0; y < H; ++y) {
        dft_rec(f + (size_t)y * W, 1, W, line, tW, W, sign, work);
        memcpy(f + (size_t)y * W, line, sizeof(cplx) * (size_t)W);
    }
    for (int x = 0; x < W; ++x) {
        dft_rec(f + x, W, H, line, tH, H, sign, work);
        for (int y = 0; y < H; ++y) f[(size_t)y * W + x] = line[y];
    }
    free(line); free(work); free(tW); free(tH);
}

/* Exported: forward 2-D transform of a uint16 image (P:L494 step 2), complex out [H][W][2]. */
void oracle_fft2_u16(const uint16_t* img, int H, int W, double* out_ri) {
    cplx* f = (cplx*)malloc(sizeof(cplx) * (size_t)H * W);
    for (size_t i = 0; i < (size_t)H * W; ++i) f[i] = (double)img[i];
    dft2(f, H, W, +1);
    for (size_t i = 0; i < (size_t)H * W; ++i) {
        out_ri[2 * i] = creal(f[i]);
        out_ri[2 * i + 1] = cimag(f[i]);
    }
    free(f);
}

/* Exported: 2-D transform of a complex array (sign +1 forward, -1 inverse, unnormalised). */
void oracle_dft2(const double* in_ri, double* out_ri, int H, int W, int sign) {
    cplx* f = (cplx*)malloc(sizeof(cplx) * (size_t)H * W);
    for (size_t i = 0; i < (size_t)H * W; ++i) f[i] = in_ri[2 * i] + I * in_ri[2 * i + 1];
    dft2(f, H, W, sign);
    for (size_t i = 0; i < (size_t)H * W; ++i) {
        out_ri[2 * i] = creal(f[i]);
        out_ri[2 * i + 1] = cimag(f[i]);
    }
    free(f);
}

/* ---------------------------------------------------------------- CCF --- */

/*
 * Fig. 3: ccf(I1, I2) = (I1 - mean I1) . (I2 - mean I2) / (|..| |..|),
 * two-pass in double.  Region of candidate (dx, dy) (Fig. 2 l.8-11, unified):
 *   a = A[dy:H, dx:W],  b = B[0:H-dy, 0:W-dx].
 * Returns 0 and sets *valid = 0 for an empty region or a zero variance (C8).
 */
double oracle_ccf(const uint16_t* A, const uint16_t* B, int H, int W, int dx, int dy,
                  int* valid) {
    const int h = H - dy, w = W - dx;
    *valid = 0;
    if (h <= 0 || w <= 0) return 0.0;
    const double n = (double)h * (double)w;
    double sa = 0, sb = 0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            sa += A[(size_t)(dy + i) * W + (dx + j)];
            sb += B[(size_t)i * W + j];
        }
    const double ma = sa / n, mb = sb / n;
    double sab = 0, saa = 0, sbb = 0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            const double a = A[(size_t)(dy + i) * W + (dx + j)] - ma;
            const double b = B[(size_t)i * W + j] - mb;
            sab += a * b;
            saa += a * a;
            sbb += b * b;
        }
    if (saa == 0.0 || sbb == 0.0) return 0.0;
    *valid = 1;
    return sab / (sqrt(saa) * sqrt(sbb));
}

/*
 * Same quantity from exact integer moments (cross-check only):
 *   ccf = (n Sab - Sa Sb) / sqrt((n Saa - Sa^2)(n Sbb - Sb^2)),
 * numerator and the two factors formed exactly in 128-bit integers.
 */
double oracle_ccf_moments(const uint16_t* A, const uint16_t* B, int H, int W, int dx, int dy,
                          uint64_t* moments /* [6]: n, Sa, Sb, Saa, Sbb, Sab */, int* valid) {
    const int h = H - dy, w = W - dx;
    uint64_t n = 0, sa = 0, sb = 0, saa = 0, sbb = 0, sab = 0;
    *valid = 0;
    if (h > 0 && w > 0) {
        for (int i = 0; i < h; ++i)
            for (int j = 0; j < w; ++j) {
                const uint64_t a = A[(size_t)(dy + i) * W + (dx + j)];
                const uint64_t b = B[(size_t)i * W + j];
                n += 1; sa += a; sb += b; saa += a * a; sbb += b * b; sab += a * b;
            }
    }
    if (moments) {
        moments[0] = n; moments[1] = sa; moments[2] = sb;
        moments[3] = saa; moments[4] = sbb; moments[5] = sab;
    }
    if (n == 0) return 0.0;
    const __int128 num = (__int128)n * sab - (__int128)sa * sb;
    const __int128 va = (__int128)n * saa - (__int128)sa * sa;
    const __int128 vb = (__int128)n * sbb - (__int128)sb * sb;
    if (va == 0 || vb == 0) return 0.0;
    *valid = 1;
    return (double)num / (sqrt((double)va) * sqrt((double)vb));
}

/* ---------------------------------------------------------- the pair --- */

typedef struct {
    int32_t dx, dy;        /* chosen translation: origin of B in A's frame */
    double ccf;            /* CCF of the chosen candidate (NaN if none valid) */
    int32_t candidate;     /* 1..4 (Fig. 2 order), 0 = none valid */
    int32_t peak_x, peak_y;/* argmax of |iFFT(NCC)| */
    double peak;           /* max / (H W) */
    double runner_up;      /* largest |iFFT| value elsewhere / (H W) (margin check, C17) */
    double ccf_k[4];       /* per-candidate CCF (NaN if invalid) */
    double max_imag_ratio; /* max|Im c| / max|Re c| (C3 check) */
} oracle_pair;

/* Steps 6-7 from a given peak (x, y): Fig. 2 l.8-12. */
void oracle_eval_peak(const uint16_t* A, const uint16_t* B, int H, int W, int x, int y,
                      oracle_pair* out) {
    const int cand[4][2] = {{x, y}, {W - x, y}, {x, H - y}, {W - x, H - y}};
    int best = 0;
    double best_ccf = 0.0;
    out->peak_x = x;
    out->peak_y = y;
    for (int k = 0; k < 4; ++k) {
        int valid = 0;
        const double c = oracle_ccf(A, B, H, W, cand[k][0], cand[k][1], &valid);
        out->ccf_k[k] = valid ? c : NAN;
        if (valid && (best == 0 || c > best_ccf)) {  /* first maximum wins (C7) */
            best = k + 1;
            best_ccf = c;
        }
    }
    out->candidate = best;
    if (best) {
        out->dx = cand[best - 1][0];
        out->dy = cand[best - 1][1];
        out->ccf = best_ccf;
    } else {
        out->dx = x;
        out->dy = y;
        out->ccf = NAN;
    }
}

/* Steps 3-5 from two forward spectra FA, FB (complex [H][W]); fills peak fields. */
static void ncc_peak(const cplx* FA, const cplx* FB, int H, int W, oracle_pair* out) {
    const size_t N = (size_t)H * W;
    cplx* c = (cplx*)malloc(sizeof(cplx) * N);
    /* step 3: NCC = fc ./ abs(fc), fc = FA .* conj(FB)  (C2, C4) */
    for (size_t i = 0; i < N; ++i) {
        const cplx fc = FA[i] * conj(FB[i]);
        const double a = cabs(fc);
        c[i] = a > 0.0 ? fc / a : 0.0;
    }
    /* step 4: unnormalised inverse 2-D transform (C5) */
    dft2(c, H, W, -1);
    /* step 5: max of abs, first in row-major order (C3, C6) */
    size_t best = 0;
    double vbest = -1.0, max_re = 0.0, max_im = 0.0;
    for (size_t i = 0; i < N; ++i) {
        const double v = fabs(creal(c[i]));
        if (v > vbest) { vbest = v; best = i; }
        if (v > max_re) max_re = v;
        if (fabs(cimag(c[i])) > max_im) max_im = fabs(cimag(c[i]));
    }
    double v2 = 0.0;
    for (size_t i = 0; i < N; ++i)
        if (i != best && fabs(creal(c[i])) > v2) v2 = fabs(creal(c[i]));
    out->peak_x = (int32_t)(best % (size_t)W);
    out->peak_y = (int32_t)(best / (size_t)W);
    out->peak = vbest / (double)N;
    out->runner_up = v2 / (double)N;
    out->max_imag_ratio = max_re > 0 ? max_im / max_re : 0.0;
    free(c);
}

static cplx* spectrum_u16(const uint16_t* img, int H, int W) {
    cplx* f = (cplx*)malloc(sizeof(cplx) * (size_t)H * W);
    for (size_t i = 0; i < (size_t)H * W; ++i) f[i] = (double)img[i];
    dft2(f, H, W, +1);  /* step 2 */
    return f;
}

/* pciam(A, B): Fig. 2, steps 2-7 for one pair of equally sized images. */
void oracle_pciam(const uint16_t* A, const uint16_t* B, int H, int W, oracle_pair* out) {
    cplx* FA = spectrum_u16(A, H, W);
    cplx* FB = spectrum_u16(B, H, W);
    ncc_peak(FA, FB, H, W, out);
    const double peak = out->peak, ru = out->runner_up, ir = out->max_imag_ratio;
    oracle_eval_peak(A, B, H, W, out->peak_x, out->peak_y, out);
    out->peak = peak; out->runner_up = ru; out->max_imag_ratio = ir;
    free(FA);
    free(FB);
}

/* Returns the normalised correlation surface |Re c| / (HW) (test helper, [H][W]). */
void oracle_surface(const uint16_t* A, const uint16_t* B, int H, int W, double* surf) {
    cplx* FA = spectrum_u16(A, H, W);
    cplx* FB = spectrum_u16(B, H, W);
    const size_t N = (size_t)H * W;
    cplx* c = (cplx*)malloc(sizeof(cplx) * N);
    for (size_t i = 0; i < N; ++i) {
        const cplx fc = FA[i] * conj(FB[i]);
        const double a = cabs(fc);
        c[i] = a > 0.0 ? fc / a : 0.0;
    }
    dft2(c, H, W, -1);
    for (size_t i = 0; i < N; ++i) surf[i] = fabs(creal(c[i])) / (double)N;
    free(c); free(FA); free(FB);
}

/* ---------------------------------------------------------- the grid --- */

typedef struct {
    const uint16_t* tiles;  /* [n][m][H][W] */
    int n, m, H, W;
    cplx** spec;            /* [n*m] forward spectra, computed once per tile */
    oracle_pair* west;      /* [n*m] */
    oracle_pair* north;     /* [n*m] */
    long next;
    int phase;
    pthread_mutex_t mu;
} grid_job;

static const uint16_t* tile_ptr(const grid_job* g, int t) {
    return g->tiles + (size_t)t * (size_t)g->H * (size_t)g->W;
}

static void absent(oracle_pair* p) {
    memset(p, 0, sizeof(*p));
    p->ccf = NAN;
    for (int k = 0; k < 4; ++k) p->ccf_k[k] = NAN;
}

static void* grid_worker(void* arg) {
    grid_job* g = (grid_job*)arg;
    const int nt = g->n * g->m;
    for (;;) {
        pthread_mutex_lock(&g->mu);
        const long job = g->next++;
        pthread_mutex_unlock(&g->mu);
        if (g->phase == 0) {
            if (job >= nt) break;
            g->spec[job] = spectrum_u16(tile_ptr(g, (int)job), g->H, g->W);
        } else {
            if (job >= 2L * nt) break;
            const int t = (int)(job / 2), kind = (int)(job % 2);
            const int r = t / g->m, c = t % g->m;
            /* Fig. 4: west[I] and north[I], both as pciam(neighbour, I) (C1) */
            oracle_pair* out = kind == 0 ? &g->west[t] : &g->north[t];
            const int nb = kind == 0 ? (c >= 1 ? t - 1 : -1) : (r >= 1 ? t - g->m : -1);
            if (nb < 0) { absent(out); continue; }
            ncc_peak(g->spec[nb], g->spec[t], g->H, g->W, out);
            const double peak = out->peak, ru = out->runner_up, ir = out->max_imag_ratio;
            oracle_eval_peak(tile_ptr(g, nb), tile_ptr(g, t), g->H, g->W, out->peak_x,
                             out->peak_y, out);
            out->peak = peak; out->runner_up = ru; out->max_imag_ratio = ir;
        }
    }
    return NULL;
}

/* Fig. 4: translations of every west and north pair of an n x m grid. */
int oracle_grid(const uint16_t* tiles, int n, int m, int H, int W, int threads,
                oracle_pair* west, oracle_pair* north) {
    if (!tiles || !west || !north || n < 1 || m < 1 || H < 1 || W < 1) return 1;
    if (threads < 1) threads = 1;
    if (threads > 512) threads = 512;
    grid_job g;
    g.tiles = tiles; g.n = n; g.m = m; g.H = H; g.W = W;
    g.spec = (cplx**)calloc((size_t)n * m, sizeof(cplx*));
    g.west = west; g.north = north;
    pthread_mutex_init(&g.mu, NULL);
    pthread_t th[512];
    for (g.phase = 0; g.phase < 2; ++g.phase) {
        g.next = 0;
        for (int i = 0; i < threads; ++i) pthread_create(&th[i], NULL, grid_worker, &g);
        for (int i = 0; i < threads; ++i) pthread_join(th[i], NULL);
    }
    for (int t = 0; t < n * m; ++t) free(g.spec[t]);
    free(g.spec);
    pthread_mutex_destroy(&g.mu);
    return 0;
}

/* Sizes of the exported struct, for the Python binding's layout check. */
int oracle_pair_size(void) { return (int)sizeof(oracle_pair); }
