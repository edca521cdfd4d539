// pciam_kernels.cuh — the PCIAM hot path (§III, Fig. 1 steps 2-7) on sm_100a.
//
// Data layout in HBM:
//   raw   uint16 [tiles][H][W]           W contiguous (the caller's tile layout)
//   spec  float2 [tiles][H][WP]          half spectrum kx in [0, W/2], WP = pad16(W/2+1),
//                                        resident for reuse by <= 4 pairs
//   Q     float2 [chunk][H][WP]          per-pair column-inverse intermediate (L2-sized chunk)
//   keys  u64    [pairs]                 packed (|c| bits << 32 | ~index) argmax per pair
//   mom   u64    [pairs][4][5]           exact integer CCF moments per candidate
//
// Kernels (one launch covers a chunk of tiles or pairs):
//   K1 fwd_rows   raw -> spec   R2C along x: length-W real row as a W/2 complex FFT + post-twiddle
//                               (step 2 first half; uint16->fp32 fused into the load)
//   K2 fwd_cols   spec -> spec  C2C along y, in place on column panels (step 2 second half)
//   K3 pair_cols  2 spec -> Q   NCPS F_A conj(F_B)/|..| fused into the loads (step 3), then the
//                               inverse C2C along y (step 4 first half)
//   K4 pair_rows  Q -> keys     C2R along x (step 4 second half) with |.| + argmax fused in the
//                               epilogue; the real correlation surface is never stored (step 5)
//   K5 ccf_mom    raw -> mom    integer moments of the 4 candidate overlaps (step 6, Fig. 3)
//   K6 finalize   mom -> pairs  CCF in fp64 from exact int128 moments, candidate selection (step 7)
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "fft_engine.cuh"
#include "../../include/stitch.h"

namespace stitch {

constexpr int pad16(int x) { return (x + 15) / 16 * 16; }

// A compiled tile-size plan: row transform (length W/2 complex) and column
// transform (length H) radices, CTA shapes.
template <int W_, int H_, class RowRX, class ColRX, int ROW_L_, int ROW_T_, int COL_P_, int COL_T_>
struct Plan {
    static constexpr int W = W_, H = H_;
    static constexpr int M = W / 2;           // complex row length
    static constexpr int WC = M + 1;          // kept bins kx in [0, M]
    static constexpr int WP = pad16(WC);      // row pitch of spectra (float2)
    using Row = RowRX;
    using Col = ColRX;
    static constexpr int ROW_L = ROW_L_, ROW_T = ROW_T_;
    static constexpr int COL_P = COL_P_, COL_T = COL_T_;
    static constexpr int ROW_STRIDE = WC + (WC >> 4) + 1;   // padded smem line (RowSmem)
    static constexpr size_t ROW_SMEM = sizeof(float2) * ROW_L * ROW_STRIDE;
    static constexpr size_t COL_SMEM = sizeof(float2) * COL_P * H;
    static_assert(W % 2 == 0, "W must be even");
    static_assert(Row::N == M && Col::N == H, "plan radices do not match the tile");
    static_assert(H % ROW_L == 0, "rows per CTA must divide H");
    static_assert(WP % COL_P == 0, "column panel must divide the pitch");
};

struct PairIdx {
    int32_t a, b;  // local tile indices: A = west/north neighbour, B = tile
};

// ------------------------------------------------------------------ K1 ----
template <class PL>
struct U16RowSrc {  // z[n] = x[2n] + i x[2n+1], straight from the uint16 row
    const uint32_t* p;
    __device__ __forceinline__ float2 load(int line, int n) const {
        const uint32_t u = __ldg(p + line * (PL::W / 2) + n);
        return make_float2((float)(u & 0xFFFFu), (float)(u >> 16));
    }
};

template <class PL>
__global__ void __launch_bounds__(PL::ROW_T) k1_fwd_rows(const uint16_t* __restrict__ raw,
                                                         float2* __restrict__ spec, int tile0,
                                                         const float2* __restrict__ twM,
                                                         const float2* __restrict__ twW) {
    extern __shared__ float2 smem[];
    constexpr int L = PL::ROW_L, T = PL::ROW_T, M = PL::M;
    const size_t t = (size_t)tile0 + blockIdx.y;
    const int y0 = blockIdx.x * L;
    U16RowSrc<PL> src{reinterpret_cast<const uint32_t*>(raw + (t * PL::H + y0) * PL::W)};
    RowSmem<PL::ROW_STRIDE> sm{smem};
    FftRun<typename PL::Row, -1, L, T, RowMap, true>::run(src, sm, sm, twM);
    __syncthreads();
    // Real-to-complex post-processing, q in [0, M] (Z[M] == Z[0]):
    //   E = (Z[q] + conj Z[M-q]) / 2,  O = (Z[q] - conj Z[M-q]) / (2i),  X[q] = E + w_W^q O
    float2* out = spec + (t * PL::H + y0) * PL::WP;
    for (int i = threadIdx.x; i < L * PL::WP; i += T) {
        const int line = i / PL::WP, q = i - line * PL::WP;
        float2 X = make_float2(0.f, 0.f);
        if (q <= M) {
            const float2 zq = sm.load(line, q == M ? 0 : q);
            const float2 zm = sm.load(line, q == 0 ? 0 : M - q);
            const float2 E = make_float2(0.5f * (zq.x + zm.x), 0.5f * (zq.y - zm.y));
            const float2 O = make_float2(0.5f * (zq.y + zm.y), -0.5f * (zq.x - zm.x));
            const float2 w = __ldg(&twW[q]);
            const float2 wo = cmul(w, O);
            X = make_float2(E.x + wo.x, E.y + wo.y);
        }
        out[(size_t)line * PL::WP + q] = X;
    }
}

// ------------------------------------------------------------------ K2 ----
template <class PL>
struct PanelIO {  // a panel of COL_P columns of one [H][WP] array
    float2* p;
    __device__ __forceinline__ float2 load(int line, int n) const { return p[(size_t)n * PL::WP + line]; }
    __device__ __forceinline__ void store(int line, int n, float2 v) const { p[(size_t)n * PL::WP + line] = v; }
};

template <class PL>
__global__ void __launch_bounds__(PL::COL_T) k2_fwd_cols(float2* __restrict__ spec, int tile0,
                                                         const float2* __restrict__ twH) {
    extern __shared__ float2 smem[];
    const size_t t = (size_t)tile0 + blockIdx.y;
    PanelIO<PL> io{spec + t * PL::H * PL::WP + blockIdx.x * PL::COL_P};
    ColSmem<PL::COL_P> sm{smem};
    FftRun<typename PL::Col, -1, PL::COL_P, PL::COL_T, ColMap, false>::run(io, sm, io, twH);
}

// ------------------------------------------------------------------ K3 ----
template <class PL>
struct NcpsSrc {  // step 3: NCC = F_A conj(F_B) / |F_A conj(F_B)|, 0 where it vanishes
    const float2* a;
    const float2* b;
    __device__ __forceinline__ float2 load(int line, int n) const {
        const float2 fa = a[(size_t)n * PL::WP + line];
        const float2 fb = b[(size_t)n * PL::WP + line];
        // |F_A conj F_B| = |F_A| |F_B|: normalise each factor first so no
        // intermediate exceeds |F|^2 (<= ~1e22, safely inside fp32).
        const float ma = fmaf(fa.x, fa.x, fa.y * fa.y);
        const float mb = fmaf(fb.x, fb.x, fb.y * fb.y);
        const float ra = ma > 0.f ? rsqrtf(ma) : 0.f;
        const float rb = mb > 0.f ? rsqrtf(mb) : 0.f;
        const float ax = fa.x * ra, ay = fa.y * ra, bx = fb.x * rb, by = fb.y * rb;
        return make_float2(fmaf(ax, bx, ay * by), fmaf(ay, bx, -ax * by));
    }
};

template <class PL>
__global__ void __launch_bounds__(PL::COL_T) k3_pair_cols(const float2* __restrict__ spec,
                                                          float2* __restrict__ Q,
                                                          const PairIdx* __restrict__ pairs,
                                                          int pair0,
                                                          const float2* __restrict__ twH) {
    extern __shared__ float2 smem[];
    const PairIdx pr = pairs[pair0 + blockIdx.y];
    const int c0 = blockIdx.x * PL::COL_P;
    const size_t img = (size_t)PL::H * PL::WP;
    NcpsSrc<PL> src{spec + pr.a * img + c0, spec + pr.b * img + c0};
    PanelIO<PL> dst{Q + blockIdx.y * img + c0};
    ColSmem<PL::COL_P> sm{smem};
    FftRun<typename PL::Col, +1, PL::COL_P, PL::COL_T, ColMap, false>::run(src, sm, dst, twH);
}

// ------------------------------------------------------------------ K4 ----
template <class PL>
struct C2RSrc {  // complex-to-real pre-processing of row X[0..M] into Z[0..M)
    const float2* rows;
    const float2* twW;
    __device__ __forceinline__ float2 load(int line, int n) const {
        const float2* r = rows + (size_t)line * PL::WP;
        const float2 xn = r[n];
        const float2 xm = r[PL::M - n];
        // E = X[n] + conj X[M-n];  O = (X[n] - conj X[M-n]) e^{+2 pi i n / W};  Z = E + i O
        const float2 w = __ldg(&twW[n]);
        const float2 d = make_float2(xn.x - xm.x, xn.y + xm.y);
        const float2 o = make_float2(fmaf(d.x, w.x, d.y * w.y), fmaf(d.y, w.x, -d.x * w.y));
        return make_float2(xn.x + xm.x - o.y, xn.y - xm.y + o.x);
    }
};

struct ArgmaxDst {  // step 5: running max of |x| with its row-major index, never stored
    unsigned long long best;
    int row_base;  // (y0 + line) * W added per line
    int W;
    __device__ __forceinline__ void store(int line, int n, float2 v) {
        const uint32_t idx = (uint32_t)((row_base + line) * W + 2 * n);
        const unsigned long long k0 =
            ((unsigned long long)__float_as_uint(fabsf(v.x)) << 32) | (0xFFFFFFFFu - idx);
        const unsigned long long k1 =
            ((unsigned long long)__float_as_uint(fabsf(v.y)) << 32) | (0xFFFFFFFFu - (idx + 1));
        best = max(best, max(k0, k1));
    }
};

template <int T>
__device__ __forceinline__ unsigned long long block_max_u64(unsigned long long v) {
    __shared__ unsigned long long red[T / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xFFFFFFFFu, v, o));
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) red[w] = v;
    __syncthreads();
    if (threadIdx.x < 32) {
        v = threadIdx.x < T / 32 ? red[threadIdx.x] : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xFFFFFFFFu, v, o));
    }
    return v;
}

template <class PL>
__global__ void __launch_bounds__(PL::ROW_T) k4_pair_rows(const float2* __restrict__ Q,
                                                          unsigned long long* __restrict__ keys,
                                                          int pair0,
                                                          const float2* __restrict__ twM,
                                                          const float2* __restrict__ twW) {
    extern __shared__ float2 smem[];
    constexpr int L = PL::ROW_L, T = PL::ROW_T;
    const int y0 = blockIdx.x * L;
    C2RSrc<PL> src{Q + ((size_t)blockIdx.y * PL::H + y0) * PL::WP, twW};
    ArgmaxDst dst{0ull, y0, PL::W};
    RowSmem<PL::ROW_STRIDE> sm{smem};
    FftRun<typename PL::Row, +1, L, T, RowMap, false>::run(src, sm, dst, twM);
    const unsigned long long best = block_max_u64<T>(dst.best);
    if (threadIdx.x == 0) atomicMax(&keys[pair0 + blockIdx.y], best);
}

// ------------------------------------------------------------------ K5 ----
// Rows of the four candidate overlaps of pair p, concatenated (2H rows in all):
//   c1 (dx,dy)=(x,y): H-y rows | c2 (W-x,y): H-y | c3 (x,H-y): y | c4 (W-x,H-y): y
// region a = A[dy:H, dx:W], b = B[0:H-dy, 0:W-dx] (Fig. 2 l.8-11 unified, Fig. 3).
constexpr int CCF_ROWS = 8;
constexpr int CCF_T = 256;

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
    return v;
}

__global__ void __launch_bounds__(CCF_T) k5_ccf_moments(const uint16_t* __restrict__ raw,
                                                        const PairIdx* __restrict__ pairs,
                                                        const unsigned long long* __restrict__ keys,
                                                        unsigned long long* __restrict__ mom,
                                                        int H, int W, int pair0) {
    __shared__ unsigned long long red[5][CCF_T / 32];
    const int p = pair0 + blockIdx.y;
    const PairIdx pr = pairs[p];
    const uint32_t lo = 0xFFFFFFFFu - (uint32_t)(keys[p] & 0xFFFFFFFFull);
    const int x = (int)(lo % (uint32_t)W), y = (int)(lo / (uint32_t)W);
    const uint16_t* A = raw + (size_t)pr.a * H * W;
    const uint16_t* B = raw + (size_t)pr.b * H * W;
    const int r0 = blockIdx.x * CCF_ROWS;
    const int r1 = min(r0 + CCF_ROWS, 2 * H);
    unsigned long long sa = 0, sb = 0, saa = 0, sbb = 0, sab = 0;
    int cur = -1;
    for (int r = r0; r <= r1; ++r) {
        int k = 4, i = 0;
        if (r < r1) {
            const int h12 = H - y;
            if (r < h12) { k = 0; i = r; }
            else if (r < 2 * h12) { k = 1; i = r - h12; }
            else if (r < 2 * h12 + y) { k = 2; i = r - 2 * h12; }
            else { k = 3; i = r - 2 * h12 - y; }
        }
        if (k != cur) {  // block-uniform: flush the previous candidate's partial sums
            if (cur >= 0) {
                unsigned long long v[5] = {sa, sb, saa, sbb, sab};
#pragma unroll
                for (int q = 0; q < 5; ++q) {
                    v[q] = warp_sum_u64(v[q]);
                    if ((threadIdx.x & 31) == 0) red[q][threadIdx.x >> 5] = v[q];
                }
                __syncthreads();
                if (threadIdx.x < 5) {
                    unsigned long long s = 0;
                    for (int w = 0; w < CCF_T / 32; ++w) s += red[threadIdx.x][w];
                    if (s) atomicAdd(&mom[((size_t)p * 4 + cur) * 5 + threadIdx.x], s);
                }
                __syncthreads();
            }
            cur = k;
            sa = sb = saa = sbb = sab = 0;
        }
        if (k == 4) break;
        const int dx = (k & 1) ? W - x : x;
        const int dy = (k & 2) ? H - y : y;
        const int w = W - dx;
        const uint16_t* ar = A + (size_t)(dy + i) * W + dx;
        const uint16_t* br = B + (size_t)i * W;
        for (int j = threadIdx.x; j < w; j += CCF_T) {
            const uint32_t a = __ldg(ar + j), b = __ldg(br + j);
            sa += a;
            sb += b;
            saa += (unsigned long long)(a * a);
            sbb += (unsigned long long)(b * b);
            sab += (unsigned long long)(a * b);
        }
    }
}

// ------------------------------------------------------------------ K6 ----
__device__ __forceinline__ double i128_to_double(__int128 v) {
    const bool neg = v < 0;
    const unsigned __int128 m = neg ? (unsigned __int128)(-v) : (unsigned __int128)v;
    const double d = (double)(unsigned long long)(m >> 64) * 18446744073709551616.0 +
                     (double)(unsigned long long)m;
    return neg ? -d : d;
}

__global__ void k6_finalize(const unsigned long long* __restrict__ keys,
                            const unsigned long long* __restrict__ mom,
                            stitch_pair* __restrict__ out, int H, int W, int npairs) {
    const int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= npairs) return;
    const unsigned long long key = keys[p];
    const uint32_t lo = 0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFull);
    const int x = (int)(lo % (uint32_t)W), y = (int)(lo / (uint32_t)W);
    stitch_pair r;
    r.peak_x = x;
    r.peak_y = y;
    r.peak = __uint_as_float((uint32_t)(key >> 32)) / ((float)W * (float)H);
    const int cdx[4] = {x, W - x, x, W - x};
    const int cdy[4] = {y, y, H - y, H - y};
    int best = 0;
    double bestv = 0.0;
    for (int k = 0; k < 4; ++k) {
        const long long n = (long long)(H - cdy[k]) * (long long)(W - cdx[k]);
        const unsigned long long* m = mom + ((size_t)p * 4 + k) * 5;
        double c = __longlong_as_double(0x7FF8000000000000ll);  // NaN = invalid (C8)
        if (n > 0) {
            const __int128 sa = m[0], sb = m[1], saa = m[2], sbb = m[3], sab = m[4];
            const __int128 num = (__int128)n * sab - sa * sb;
            const __int128 va = (__int128)n * saa - sa * sa;
            const __int128 vb = (__int128)n * sbb - sb * sb;
            if (va > 0 && vb > 0) {
                c = i128_to_double(num) / (sqrt(i128_to_double(va)) * sqrt(i128_to_double(vb)));
                if (best == 0 || c > bestv) {  // first maximum wins (C7)
                    best = k + 1;
                    bestv = c;
                }
            }
        }
        r.ccf_k[k] = c;
    }
    r.candidate = best;
    if (best) {
        r.dx = cdx[best - 1];
        r.dy = cdy[best - 1];
        r.ccf = bestv;
    } else {
        r.dx = x;
        r.dy = y;
        r.ccf = __longlong_as_double(0x7FF8000000000000ll);
    }
    out[p] = r;
}

}  // namespace stitch
