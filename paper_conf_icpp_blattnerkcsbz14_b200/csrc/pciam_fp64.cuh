// pciam_fp64.cuh — the fp64 path: PCIAM steps 2-5 in double precision.
//
// The paper computes its transforms in "double complex" and the CCF in double
// (Fig. 3); north_star makes fp64 the optional tighter-tolerance path (CCF within
// 1e-9 of the oracle).  Same method, same FFT engine (fft_engine.cuh instantiated with
// C = double2 and the fp64 twins of the generated codelets), same pair list, CCF (K5) and
// selection (K6) as the fp32 path; what differs:
//   * the resident spectrum is the unit phasor U = F/|F| (0 where F = 0) as double2 -- step 3
//     F_A conj(F_B) / |F_A conj(F_B)| = U_A conj(U_B) exactly in real arithmetic (reading C4),
//     and a 64-bit phase code would need a double-precision sincos per bin;
//   * the argmax (step 5) compares doubles: per row block a (max |c|, smallest index) partial,
//     then one warp per pair reduces the partials into the same 64-bit key K5/K6 consume
//     (the key's value field carries |c| rounded to float, used only for the reported peak).
// Kernels (plain CTA-per-block launches, coalesced global loads; no TMA: the fp64 path is
// FP64-issue-bound on B200 long before it is HBM-bound):
//   D1 fwd_rows   raw -> Gd   R2C along x (uint16 -> double fused into the load); Gd is
//                             panel-blocked ([tile][WP/4][H][4]) like the fp32 G
//   D2 fwd_cols   Gd -> U     C2C along y on a panel landed by one bulk copy, epilogue: unit
//                             phasor, U column-major [slot][WP][HP64] (or the complex spectrum
//                             row-major into Qd for the parity hook)
//   D3 pair_cols  U -> Qd     the two tiles' panels land by one bulk copy each; step 3
//                             (U_A conj U_B) fused into the inverse C2C along y
//   D4 pair_rows  Qd -> part  C2R along x, |.| + per-block argmax (surface never stored)
//   D5 argmax     part -> key per-pair reduction of the block partials
#pragma once
#include "pciam_kernels.cuh"

namespace stitch {

template <class PL>
struct Plan64 {
    static constexpr int W = PL::W, H = PL::H, M = PL::M, WP = PL::WP;
    using Row = typename PL::Row;
    using Col = typename PL::Col;
    using RI = typename PL::RI;
    using CI = typename PL::CI;
    static constexpr int ROW_L = PL::ROW_L, ROW_T = PL::ROW_T;
    using RowX = RowXchg<RI::R0, RI::R1, PL::ROW_PAD, double2>;
    static constexpr size_t ROW_SMEM = sizeof(double2) * ROW_L * RowX::LSTRIDE;
    static constexpr int NBLK = H / ROW_L;    // row blocks (argmax partials) per pair
    // column panels: 4 columns of double2 = 64-byte row segments
    static constexpr int COL_P = 4;
    static constexpr int COL_WORK = CI::STAGES == 1 ? COL_P
                                                    : (COL_P * CI::R1 > COL_P * CI::R0
                                                           ? COL_P * CI::R1
                                                           : COL_P * CI::R0);
    static constexpr int COL_T = (COL_WORK + 31) / 32 * 32;
    using ColX = ColXchg<CI::R0, CI::R1, PL::COL_PAD, COL_P, double2>;
    static constexpr size_t COL_XCH =
        CI::STAGES == 1 ? 16 : sizeof(double2) * COL_P * CI::R1 * (CI::R0 + PL::COL_PAD);
    // column pitch of the column-major Q31 unit phasor U (int2, 8 bytes per bin): >= H and
    // 8 mod 16, so the 8-byte loads of a landed 2-column panel (16 lanes per wavefront: 2
    // columns x 8 rows) are bank-conflict-free (and every column run is 16-byte aligned)
    static constexpr int HP64 = H % 16 <= 8 ? H + (8 - H % 16) : H + (24 - H % 16);
    static constexpr size_t PANEL_G = sizeof(double2) * COL_P * H;      // D2's landed Gd panel
    static constexpr size_t D2_SMEM = (PANEL_G > COL_XCH ? PANEL_G : COL_XCH);
    // D3 takes 2-column panels of U (any column run of the column-major U is contiguous): two
    // landed panels (2 x 33 KB) + the aliased exchange let two 3-warp CTAs share an SM, so one
    // CTA's landing overlaps the other's butterflies (the radix-40 double butterfly's 254
    // registers allow no more warps)
    static constexpr int COL_P3 = 2;
    static constexpr int COL_WORK3 = CI::STAGES == 1 ? COL_P3
                                                     : (CI::R1 > CI::R0 ? COL_P3 * CI::R1
                                                                        : COL_P3 * CI::R0);
    static constexpr int COL_T3 = (COL_WORK3 + 31) / 32 * 32;
    using ColX3 = ColXchg<CI::R0, CI::R1, PL::COL_PAD, COL_P3, double2>;
    static constexpr size_t COL_XCH3 =
        CI::STAGES == 1 ? 16 : sizeof(double2) * COL_P3 * CI::R1 * (CI::R0 + PL::COL_PAD);
    static constexpr size_t PANEL_U = sizeof(int2) * COL_P3 * HP64;     // one tile's U panel
    static constexpr size_t U_B_OFF = (PANEL_U + 127) / 128 * 128;      // D3's second panel
    static constexpr size_t D3_SMEM =
        (U_B_OFF + PANEL_U > COL_XCH3 ? U_B_OFF + PANEL_U : COL_XCH3);
    // D4: the block's ROW_L rows of Q land by one bulk copy, reused as the exchange
    static constexpr size_t ROWS_Q = sizeof(double2) * ROW_L * WP;
    static constexpr size_t D4_SMEM = ROWS_Q > ROW_SMEM ? ROWS_Q : ROW_SMEM;
    static_assert(WP % COL_P == 0, "fp64 column panel must divide the pitch");
    static_assert(D2_SMEM <= 200 * 1024 && D3_SMEM <= 200 * 1024 && D4_SMEM <= 200 * 1024,
                  "fp64 shared memory");
};

// Prime-factor (Good-Thomas) two-stage transform of L lines of length N = R0 R1 (coprime) by a
// CTA, for D4's rows (696 = 29 x 24): no stage-2 twiddles (in double each was a complex multiply
// plus a 16-byte twiddle load), only index maps --
//   stage 1 (radix R0, butterfly b < R1):  element a at n = (R0 b + R1 a) mod N -> exchange (a, b)
//   stage 2 (radix R1, butterfly k1 < R0): reads (k1, j), output j at n = (C1 k1 + C2 j) mod N.
// IN_PLACE: the source is the exchange buffer (every stage-1 input is loaded before a barrier).
// SLOT_OUT: stage 2 writes its outputs back into the slots it read (conflict-free, in place);
// Z[q] is then at exchange (q mod R0, q mod R1) (CRT) -- D1's R2C post-pass reads it there.
template <class RX, int SIGN, int L, int T, class C = double2>
struct FftRunPfa;
template <int N, int R0, int R1, int SIGN, int L, int T, class C>
struct FftRunPfa<Radix<N, R0, R1>, SIGN, L, T, C> {
    static constexpr bool OK = gcd_c(R0, R1) == 1;
    static constexpr int C1 = (R1 * modinv(R1 % R0, R0)) % N;
    static constexpr int C2 = (R0 * modinv(R0 % R1, R1)) % N;
    template <bool IN_PLACE, bool SLOT_OUT = false, class Src, class Xc, class Dst>
    static __device__ __forceinline__ void run(const Src& src, const Xc& xc, Dst& dst) {
        {
            constexpr int TOTAL = L * R1;
            constexpr int ITER = (TOTAL + T - 1) / T;
            C v[ITER][R0];
#pragma unroll
            for (int it = 0; it < ITER; ++it) {
                const int g = threadIdx.x + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    const int line = g / R1, b = g - line * R1;
                    int n = R0 * b;
#pragma unroll
                    for (int a = 0; a < R0; ++a) {
                        v[it][a] = src.load(line, n);
                        n += R1;
                        if (n >= N) n -= N;
                    }
                }
            }
            if constexpr (IN_PLACE) __syncthreads();
#pragma unroll
            for (int it = 0; it < ITER; ++it) {
                const int g = threadIdx.x + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    const int line = g / R1, b = g - line * R1;
                    Dft<R0, SIGN>::run(v[it]);
#pragma unroll
                    for (int a = 0; a < R0; ++a) xc.at(line, a, b) = v[it][a];
                }
            }
        }
        __syncthreads();
        {
            constexpr int TOTAL = L * R0;
            constexpr int ITER = (TOTAL + T - 1) / T;
#pragma unroll 1
            for (int it = 0; it < ITER; ++it) {
                const int g = threadIdx.x + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    const int line = g / R0, k1 = g - line * R0;
                    C v[R1];
#pragma unroll
                    for (int j = 0; j < R1; ++j) v[j] = xc.at(line, k1, j);
                    Dft<R1, SIGN>::run(v);
                    if constexpr (SLOT_OUT) {
#pragma unroll
                        for (int j = 0; j < R1; ++j) xc.at(line, k1, j) = v[j];
                    } else if constexpr (Dst::PFA_BATCH) {
                        dst.template store_pfa<R1, C1, C2, N>(line, k1, v);
                    } else {
                        int n = (C1 * k1) % N;
#pragma unroll
                        for (int j = 0; j < R1; ++j) {
                            dst.store(line, n, v[j]);
                            n += C2;
                            if (n >= N) n -= N;
                        }
                    }
                }
            }
        }
    }
};

// ------------------------------------------------------------------ D1 ----
template <class PL>
struct U16RowSrcD {  // z[n] = x[2n] + i x[2n+1] (exact in double)
    const uint32_t* p;
    __device__ __forceinline__ double2 load(int line, int n) const {
        const uint32_t u = __ldg(p + line * (PL::W / 2) + n);
        return make_double2((double)(u & 0xFFFFu), (double)(u >> 16));
    }
};

// R2C post-processing of one line in double (the fp32 r2c_post_line, pciam_kernels.cuh):
//   E = (Z[q] + conj Z[M-q]) / 2,  O = (Z[q] - conj Z[M-q]) / (2i)
//   X[q] = E + w_W^q O,   X[M-q] = conj(E - w_W^q O)
// Gd's panel-blocked layout (the fp32 GRow with 4-column double2 panels: 64-byte runs)
template <class PL>
struct GRowD {
    double2* t;
    int y;
    __device__ __forceinline__ double2& operator[](int q) const {
        constexpr int P = Plan64<PL>::COL_P;
        return t[((size_t)(q / P) * PL::H + y) * P + q % P];
    }
};

template <class PL, class Xc>
__device__ __forceinline__ void r2c_post_line_d(const Xc& xc, int line, const GRowD<PL>& out,
                                                const double2* __restrict__ twW) {
    constexpr int M = PL::M;
    for (int q = threadIdx.x; q <= M / 2; q += PL::ROW_T) {
        const double2 zq = xc.nat(line, q);
        const double2 zm = xc.nat(line, q == 0 ? 0 : M - q);
        const double2 E = make_double2(0.5 * (zq.x + zm.x), 0.5 * (zq.y - zm.y));
        const double2 O = make_double2(0.5 * (zq.y + zm.y), -0.5 * (zq.x - zm.x));
        const double2 wo = cmul(__ldg(&twW[q]), O);
        out[q] = make_double2(E.x + wo.x, E.y + wo.y);
        if (2 * q != M) out[M - q] = make_double2(E.x - wo.x, wo.y - E.y);
    }
    for (int q = M + 1 + threadIdx.x; q < PL::WP; q += PL::ROW_T) out[q] = make_double2(0.0, 0.0);
}

template <class PL>
__global__ void __launch_bounds__(PL::ROW_T) d1_fwd_rows(const uint16_t* __restrict__ raw,
                                                         double2* __restrict__ G, int tile0,
                                                         const double2* __restrict__ tw2,
                                                         const double2* __restrict__ twW) {
    using P64 = Plan64<PL>;
    extern __shared__ __align__(128) unsigned char smem64[];
    constexpr int L = P64::ROW_L, T = P64::ROW_T;
    const size_t t = (size_t)tile0 + blockIdx.y;
    const int y0 = blockIdx.x * L;
    U16RowSrcD<PL> src{reinterpret_cast<const uint32_t*>(raw + (t * PL::H + y0) * PL::W)};
    typename P64::RowX xc{reinterpret_cast<double2*>(smem64)};
    using RI = typename P64::RI;
    if constexpr (RI::STAGES == 2 && gcd_c(RI::R0, RI::R1) == 1) {
        // prime-factor transform, outputs left in their slots: Z[q] at (q mod R0, q mod R1)
        FftRunPfa<typename P64::Row, -1, L, T>::template run<false, true>(src, xc, xc);
        __syncthreads();
        struct {
            typename P64::RowX x;
            __device__ __forceinline__ double2 nat(int line, int q) const {
                return x.at(line, q % RI::R0, q % RI::R1);
            }
        } z{xc};
#pragma unroll 1
        for (int line = 0; line < L; ++line)
            r2c_post_line_d<PL>(z, line, GRowD<PL>{G + (size_t)blockIdx.y * PL::H * PL::WP, y0 + line},
                                twW);
    } else {
        FftRun<typename P64::Row, -1, L, T, RowMap, false, double2>::run(src, xc, xc, tw2);
        __syncthreads();
#pragma unroll 1
        for (int line = 0; line < L; ++line)
            r2c_post_line_d<PL>(xc, line, GRowD<PL>{G + (size_t)blockIdx.y * PL::H * PL::WP,
                                                    y0 + line},
                                twW);
    }
}

// ------------------------------------------------------------------ D2 ----
template <class PL>
struct PanelIOD {  // a panel of columns of one [H][WP] double2 array
    double2* p;
    __device__ __forceinline__ double2 load(int line, int n) const {
        return p[(size_t)n * PL::WP + line];
    }
    __device__ __forceinline__ void store(int line, int n, double2 v) const {
        p[(size_t)n * PL::WP + line] = v;
    }
};

// The fp64 path's resident spectrum: the unit phasor U = F/|F| (0 where F = 0, reading C4) in
// Q31 fixed point, round(S Re U), round(S Im U) with S = 2^31 - 1 (per-component error <= 2^-32 of
// the unit circle, reading C11-f2), column-major.  D3 forms U_A conj(U_B) exactly in int64.
constexpr double Q31_S = 2147483647.0;
template <class PL>
struct UnitDst {
    int2* p;
    __device__ __forceinline__ void store(int line, int n, double2 v) const {
        const double m2 = fma(v.x, v.x, v.y * v.y);
        const double r = m2 > 0.0 ? rsqrt(m2) * Q31_S : 0.0;
        p[(size_t)line * Plan64<PL>::HP64 + n] =
            make_int2(__double2int_rn(v.x * r), __double2int_rn(v.y * r));
    }
};

template <class PL>
struct LandSrcD {  // a landed Gd panel [H][COL_P] in shared memory
    const double2* s;
    __device__ __forceinline__ double2 load(int line, int n) const {
        return s[n * Plan64<PL>::COL_P + line];
    }
};

// The panel lands by one bulk copy (Gd is panel-blocked); the landing buffer becomes the
// exchange once stage 1 has read it (IN_PLACE).  UNIT_OUT = false: the parity hook's complex
// spectrum, row-major [H][WP], into `out`.
// two 5-warp CTAs per SM (register-budgeted by the launch bounds)
template <class PL, bool UNIT_OUT>
__global__ void __launch_bounds__(Plan64<PL>::COL_T, 2) d2_fwd_cols(const double2* __restrict__ G,
                                                                 int2* __restrict__ U,
                                                                 double2* __restrict__ out,
                                                                 int tile0,
                                                                 const double2* __restrict__ tw2) {
    using P64 = Plan64<PL>;
    extern __shared__ __align__(128) unsigned char smem64[];
    __shared__ uint64_t bar;
    const int tl = blockIdx.y, c0 = blockIdx.x * P64::COL_P;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, (uint32_t)P64::PANEL_G);
        bulk_g2s(smem64, G + ((size_t)tl * PL::WP + c0) * PL::H, (uint32_t)P64::PANEL_G, &bar);
    }
    mbar_wait(&bar, 0);
    LandSrcD<PL> src{reinterpret_cast<const double2*>(smem64)};
    typename P64::ColX xc{reinterpret_cast<double2*>(smem64)};
    using Run = FftRun<typename P64::Col, -1, P64::COL_P, P64::COL_T, ColMap, false, double2>;
    if constexpr (UNIT_OUT) {
        UnitDst<PL> dst{U + ((size_t)(tile0 + tl) * PL::WP + c0) * P64::HP64};
        Run::template run<true>(src, xc, dst, tw2);
    } else {
        PanelIOD<PL> dst{out + (size_t)tl * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tw2);
    }
}

// ------------------------------------------------------------------ D3 ----
template <class PL>
struct NcpsUnitSrc {  // step 3: U_A conj(U_B) = F_A conj(F_B) / |F_A conj(F_B)| (x S^2; 0 if either is 0)
    const int2* a;     // landed column-major Q31 panels [COL_P3][HP64]
    const int2* b;
    __device__ __forceinline__ double2 load(int line, int n) const {
        const int o = line * Plan64<PL>::HP64 + n;
        const int2 ua = a[o], ub = b[o];
        // exact in int64: |.| <= |U_A| |U_B| S^2 < 2^62
        const long long re = (long long)ua.x * ub.x + (long long)ua.y * ub.y;
        const long long im = (long long)ua.y * ub.x - (long long)ua.x * ub.y;
        return make_double2((double)re, (double)im);
    }
};

template <class PL>
__global__ void __launch_bounds__(Plan64<PL>::COL_T3, 3) d3_pair_cols(const int2* __restrict__ U,
                                                                  double2* __restrict__ Q,
                                                                  const PairIdx* __restrict__ pairs,
                                                                  int pair0,
                                                                  const double2* __restrict__ tw2) {
    using P64 = Plan64<PL>;
    extern __shared__ __align__(128) unsigned char smem64[];
    __shared__ uint64_t bar;
    const PairIdx pr = pairs[pair0 + blockIdx.y];
    const int c0 = blockIdx.x * P64::COL_P3;
    int2* la = reinterpret_cast<int2*>(smem64);
    int2* lb = reinterpret_cast<int2*>(smem64 + P64::U_B_OFF);
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {   // each tile's panel is one contiguous run of U: one bulk copy each
        mbar_arrive_expect_tx(&bar, 2 * (uint32_t)P64::PANEL_U);
        bulk_g2s(la, U + ((size_t)pr.a * PL::WP + c0) * P64::HP64, (uint32_t)P64::PANEL_U, &bar);
        bulk_g2s(lb, U + ((size_t)pr.b * PL::WP + c0) * P64::HP64, (uint32_t)P64::PANEL_U, &bar);
    }
    mbar_wait(&bar, 0);
    NcpsUnitSrc<PL> src{la, lb};
    PanelIOD<PL> dst{Q + (size_t)blockIdx.y * PL::H * PL::WP + c0};
    typename P64::ColX3 xc{reinterpret_cast<double2*>(smem64)};
    FftRun<typename P64::Col, +1, P64::COL_P3, P64::COL_T3, ColMap, false, double2>::template run<
        true>(src, xc, dst, tw2);
}

// D3 as a three-factor prime-factor (Good-Thomas) column transform where H splits into three
// pairwise coprime radices with codelets (1040 = 16 x 5 x 13): no twiddles at all, and butterflies
// of at most 16 points -- ~90 registers instead of the radix-40 butterfly's 168-222 -- so four
// 5-warp CTAs share an SM.  With N = A B C, element (a, b, c) of the 3-D array is
//   input  n = (a N/A + b N/B + c N/C) mod N          (the Ruritanian map)
//   output k = (ka e_A + kb e_B + kc e_C) mod N,  e_X = (N/X) ((N/X)^-1 mod X)   (CRT)
// and the transform is three passes of 1-D DFTs along c (radix C), a (radix A), b (radix B).
// Pass 1 reads U_A conj(U_B) straight from the landed Q31 panels (lanes walk a: input stride
// N/A = 65 = 1 mod 16 banks) into registers, then -- after a barrier -- writes the work buffer,
// which reuses the landing; passes 2-3 work in place; pass 3 writes Q at the CRT index.
template <class PL>
struct D3P {
    using F = Pfa3<PL::H>;
    static constexpr int A = F::A, B = F::B, C = F::C, N = PL::H;
    static constexpr int P = 2;                                   // columns per CTA
    static constexpr int T = 160;
    static constexpr int SA = N / A, SB = N / B, SC = N / C;      // input-map strides
    static constexpr int EA = SA * modinv(SA % A, A) % N;         // CRT output weights
    static constexpr int EB = SB * modinv(SB % B, B) % N;
    static constexpr int EC = SC * modinv(SC % C, C) % N;
    static constexpr int CS = N + 4;                              // work-buffer column stride (16 B units)
    static constexpr size_t WORK = sizeof(double2) * P * CS;
    static constexpr size_t PANEL_U = sizeof(int2) * P * Plan64<PL>::HP64;
    static constexpr size_t U_B_OFF = (PANEL_U + 127) / 128 * 128;
    static constexpr size_t SMEM = U_B_OFF + PANEL_U > WORK ? U_B_OFF + PANEL_U : WORK;
    static_assert(!F::OK || (A * B * C == N && P * A * B == T), "pass 1: one butterfly per thread");
    // work element (col, a, b, c)
    static __device__ __forceinline__ int w(int col, int a, int b, int c) {
        return col * CS + (a * B + b) * C + c;
    }
};

template <class PL>
__global__ void __launch_bounds__(D3P<PL>::T, 4) d3p_pair_cols(const int2* __restrict__ U,
                                                               double2* __restrict__ Q,
                                                               const PairIdx* __restrict__ pairs,
                                                               int pair0) {
    using S = D3P<PL>;
    using P64 = Plan64<PL>;
    constexpr int A = S::A, B = S::B, C = S::C, N = S::N;
    extern __shared__ __align__(128) unsigned char smem64[];
    __shared__ uint64_t bar;
    const PairIdx pr = pairs[pair0 + blockIdx.y];
    const int c0 = blockIdx.x * S::P;
    int2* la = reinterpret_cast<int2*>(smem64);
    int2* lb = reinterpret_cast<int2*>(smem64 + S::U_B_OFF);
    double2* wk = reinterpret_cast<double2*>(smem64);   // reuses the landing after pass 1's loads
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {   // each tile's 2-column run of the column-major U: one bulk copy each
        mbar_arrive_expect_tx(&bar, 2 * (uint32_t)S::PANEL_U);
        bulk_g2s(la, U + ((size_t)pr.a * PL::WP + c0) * P64::HP64, (uint32_t)S::PANEL_U, &bar);
        bulk_g2s(lb, U + ((size_t)pr.b * PL::WP + c0) * P64::HP64, (uint32_t)S::PANEL_U, &bar);
    }
    mbar_wait(&bar, 0);
    const int t = threadIdx.x;
    {   // pass 1: radix C along c; butterfly (col, a, b) = thread, lanes walk a
        const int a = t % A, col = (t / A) % S::P, b = t / (A * S::P);
        NcpsUnitSrc<PL> src{la, lb};
        double2 v[C];
        int n = (a * S::SA + b * S::SB) % N;
#pragma unroll
        for (int c = 0; c < C; ++c) {
            v[c] = src.load(col, n);
            n += S::SC;
            if (n >= N) n -= N;
        }
        __syncthreads();   // every landed value is in registers: the buffer becomes the work array
        Dft<C, +1>::run(v);
#pragma unroll
        for (int c = 0; c < C; ++c) wk[S::w(col, a, b, c)] = v[c];
    }
    __syncthreads();
    // pass 2: radix A along a; butterflies (col, b, kc), lanes walk kc
    for (int g = t; g < S::P * B * C; g += S::T) {
        const int kc = g % C, b = (g / C) % B, col = g / (B * C);
        double2 v[A];
#pragma unroll
        for (int a = 0; a < A; ++a) v[a] = wk[S::w(col, a, b, kc)];
        Dft<A, +1>::run(v);
#pragma unroll
        for (int a = 0; a < A; ++a) wk[S::w(col, a, b, kc)] = v[a];
    }
    __syncthreads();
    // pass 3: radix B along b; butterflies (col, ka, kc), lanes walk col then kc; output at the
    // CRT index k of column c0 + col of this pair's Q (two adjacent lanes fill one 32-byte row run)
    double2* q = Q + (size_t)blockIdx.y * PL::H * PL::WP + c0;
    for (int g = t; g < S::P * A * C; g += S::T) {
        const int col = g % S::P, kc = (g / S::P) % C, ka = g / (S::P * C);
        double2 v[B];
#pragma unroll
        for (int b = 0; b < B; ++b) v[b] = wk[S::w(col, ka, b, kc)];
        Dft<B, +1>::run(v);
        int k = (ka * S::EA + kc * S::EC) % N;
#pragma unroll
        for (int kb = 0; kb < B; ++kb) {
            q[(size_t)k * PL::WP + col] = v[kb];
            k += S::EB;
            if (k >= N) k -= N;
        }
    }
}

// D2 on the same three-factor split (forward): a CTA takes one 4-column Gd panel (one bulk copy),
// pass 1 (radix C) reads it with the Ruritanian input map into registers, passes 2-3 (radix A, B)
// work in place on the work array that reuses the landing; pass 3 encodes the Q31 unit phasor at the
// CRT index into a staging panel [4][HPS] (a conflict-free pitch), stored with one bulk copy per
// column into the column-major U (or, UNIT_OUT = false, the complex spectrum row-major into `out`).
template <class PL>
struct D2P {
    using F = Pfa3<PL::H>;
    static constexpr int A = F::A, B = F::B, C = F::C, N = PL::H;
    static constexpr int P = Plan64<PL>::COL_P;                  // 4 columns: one Gd panel
    static constexpr int T = P * A * B;                           // pass 1: one butterfly each
    static constexpr int SA = N / A, SB = N / B, SC = N / C;
    static constexpr int EA = SA * modinv(SA % A, A) % N;
    static constexpr int EB = SB * modinv(SB % B, B) % N;
    static constexpr int EC = SC * modinv(SC % C, C) % N;
    static constexpr int CS = N % 8 <= 2 ? N + (2 - N % 8) : N + (10 - N % 8);   // 2 mod 8
    static constexpr int HPS = N % 16 <= 4 ? N + (4 - N % 16) : N + (20 - N % 16); // 4 mod 16
    static constexpr size_t LAND = sizeof(double2) * P * N;
    static constexpr size_t WORK = sizeof(double2) * P * CS;
    static constexpr size_t STG_OFF = ((LAND > WORK ? LAND : WORK) + 127) / 128 * 128;
    static constexpr size_t SMEM = STG_OFF + sizeof(int2) * P * HPS;
    static __device__ __forceinline__ int w(int col, int a, int b, int c) {
        return col * CS + (a * B + b) * C + c;
    }
};

template <class PL, bool UNIT_OUT>
__global__ void __launch_bounds__(D2P<PL>::T, 2) d2p_fwd_cols(const double2* __restrict__ G,
                                                              int2* __restrict__ U,
                                                              double2* __restrict__ out,
                                                              int tile0) {
    using S = D2P<PL>;
    using P64 = Plan64<PL>;
    constexpr int A = S::A, B = S::B, C = S::C, N = S::N, P = S::P;
    extern __shared__ __align__(128) unsigned char smem64[];
    __shared__ uint64_t bar;
    const int tl = blockIdx.y, c0 = blockIdx.x * P;
    const double2* land = reinterpret_cast<const double2*>(smem64);   // [n][P]
    double2* wk = reinterpret_cast<double2*>(smem64);
    int2* stage = reinterpret_cast<int2*>(smem64 + S::STG_OFF);
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, (uint32_t)S::LAND);
        bulk_g2s(smem64, G + ((size_t)tl * PL::WP + c0) * PL::H, (uint32_t)S::LAND, &bar);
    }
    mbar_wait(&bar, 0);
    const int t = threadIdx.x;
    {   // pass 1: radix C along c; butterfly (col, a, b) = thread, lanes walk col then a
        const int col = t % P, a = (t / P) % A, b = t / (P * A);
        double2 v[C];
        int n = (a * S::SA + b * S::SB) % N;
#pragma unroll
        for (int c = 0; c < C; ++c) {
            v[c] = land[n * P + col];
            n += S::SC;
            if (n >= N) n -= N;
        }
        __syncthreads();
        Dft<C, -1>::run(v);
#pragma unroll
        for (int c = 0; c < C; ++c) wk[S::w(col, a, b, c)] = v[c];
    }
    __syncthreads();
    for (int g = t; g < P * B * C; g += S::T) {   // pass 2: radix A along a
        const int col = g % P, kc = (g / P) % C, b = g / (P * C);
        double2 v[A];
#pragma unroll
        for (int a = 0; a < A; ++a) v[a] = wk[S::w(col, a, b, kc)];
        Dft<A, -1>::run(v);
#pragma unroll
        for (int a = 0; a < A; ++a) wk[S::w(col, a, b, kc)] = v[a];
    }
    __syncthreads();
    for (int g = t; g < P * A * C; g += S::T) {   // pass 3: radix B along b, CRT output
        const int col = g % P, ka = (g / P) % A, kc = g / (P * A);
        double2 v[B];
#pragma unroll
        for (int b = 0; b < B; ++b) v[b] = wk[S::w(col, ka, b, kc)];
        Dft<B, -1>::run(v);
        int k = (ka * S::EA + kc * S::EC) % N;
#pragma unroll
        for (int kb = 0; kb < B; ++kb) {
            if constexpr (UNIT_OUT) {
                const double2 x = v[kb];
                const double m2 = fma(x.x, x.x, x.y * x.y);
                const double r = m2 > 0.0 ? rsqrt(m2) * Q31_S : 0.0;
                stage[col * S::HPS + k] = make_int2(__double2int_rn(x.x * r), __double2int_rn(x.y * r));
            } else {
                out[((size_t)tl * PL::H + k) * PL::WP + c0 + col] = v[kb];
            }
            k += S::EB;
            if (k >= N) k -= N;
        }
    }
    if constexpr (UNIT_OUT) {
        fence_proxy_async();
        __syncthreads();
        if (threadIdx.x == 0) {
            int2* dst = U + ((size_t)(tile0 + tl) * PL::WP + c0) * P64::HP64;
#pragma unroll
            for (int col = 0; col < P; ++col)
                bulk_s2g(dst + (size_t)col * P64::HP64, stage + col * S::HPS,
                         (uint32_t)(sizeof(int2) * N));
            bulk_commit();
            bulk_wait_read_all();
        }
    }
}

// ------------------------------------------------------------------ D4 ----
template <class PL>
struct C2RSrcD {  // complex-to-real pre-processing of row X[0..M] into Z[0..M) (as C2RSrc)
    const double2* rows;
    const double2* twW;
    __device__ __forceinline__ double2 load(int line, int n) const {
        const double2* r = rows + (size_t)line * PL::WP;
        const double2 xn = r[n];
        const double2 xm = r[PL::M - n];
        const double2 w = __ldg(&twW[n]);
        const double2 d = make_double2(xn.x - xm.x, xn.y + xm.y);
        const double2 o = cmulc(d, w);
        return make_double2(xn.x + xm.x - o.y, xn.y - xm.y + o.x);
    }
};

struct ArgmaxDstD {  // step 5 in double: running (max |x|, smallest index at that max)
    double best_v;     // -1 before the first value
    uint32_t best_i;
    int row_base, W;
    // A whole prime-factor butterfly at once (output j at n = (C1 k1 + C2 j) mod N): its max
    // |x| by DSETP.MAX, and only when that reaches the running best (rare once a block is under
    // way) the smallest index holding it -- the same (value, index) as `store` value by value.
    static constexpr bool PFA_BATCH = true;
    template <int R1, int C1, int C2, int N>
    __device__ __forceinline__ void store_pfa(int line, int k1, const double2 (&v)[R1]) {
        double m = fmax(fabs(v[0].x), fabs(v[0].y));
#pragma unroll
        for (int j = 1; j < R1; ++j) m = fmax(m, fmax(fabs(v[j].x), fabs(v[j].y)));
        if (m >= best_v) {
            const uint32_t base = (uint32_t)(row_base + line) * W;
            uint32_t idx = 0xFFFFFFFFu, n = (uint32_t)((C1 * k1) % N);
#pragma unroll
            for (int j = 0; j < R1; ++j) {
                if (fabs(v[j].x) == m) idx = min(idx, base + 2 * n);
                if (fabs(v[j].y) == m) idx = min(idx, base + 2 * n + 1);
                n += C2;
                if (n >= (uint32_t)N) n -= N;
            }
            best_i = m > best_v ? idx : min(idx, best_i);
            best_v = m;
        }
    }
    __device__ __forceinline__ void take(double a, uint32_t idx) {
        if (a > best_v || (a == best_v && idx < best_i)) {
            best_v = a;
            best_i = idx;
        }
    }
    __device__ __forceinline__ void store(int line, int n, double2 v) {
        const uint32_t idx = (uint32_t)((row_base + line) * W + 2 * n);
        take(fabs(v.x), idx);
        take(fabs(v.y), idx + 1);
    }
};

// (v, i) beats (v2, i2): larger value, then the smaller row-major index (reading C6)
__device__ __forceinline__ void argmax_merge(double& v, uint32_t& i, double v2, uint32_t i2) {
    if (v2 > v || (v2 == v && i2 < i)) {
        v = v2;
        i = i2;
    }
}

__device__ __forceinline__ void warp_argmax(double& v, uint32_t& i) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double v2 = __shfl_xor_sync(0xFFFFFFFFu, v, o);
        const uint32_t i2 = __shfl_xor_sync(0xFFFFFFFFu, i, o);
        argmax_merge(v, i, v2, i2);
    }
}

template <class PL>
__global__ void __launch_bounds__(PL::ROW_T, 3) d4_pair_rows(const double2* __restrict__ Q,
                                                          double* __restrict__ part_v,
                                                          uint32_t* __restrict__ part_i,
                                                          int pair0,
                                                          const double2* __restrict__ tw2,
                                                          const double2* __restrict__ twW) {
    using P64 = Plan64<PL>;
    extern __shared__ __align__(128) unsigned char smem64[];
    __shared__ double rv[(PL::ROW_T + 31) / 32];
    __shared__ uint32_t ri[(PL::ROW_T + 31) / 32];
    constexpr int L = P64::ROW_L, T = P64::ROW_T;
    const int y0 = blockIdx.x * L;
    __shared__ uint64_t bar;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {   // the block's L consecutive rows of Q: one bulk copy
        mbar_arrive_expect_tx(&bar, (uint32_t)P64::ROWS_Q);
        bulk_g2s(smem64, Q + ((size_t)blockIdx.y * PL::H + y0) * PL::WP, (uint32_t)P64::ROWS_Q,
                 &bar);
    }
    mbar_wait(&bar, 0);
    C2RSrcD<PL> src{reinterpret_cast<const double2*>(smem64), twW};
    ArgmaxDstD dst{-1.0, 0xFFFFFFFFu, y0, PL::W};
    typename P64::RowX xc{reinterpret_cast<double2*>(smem64)};   // reuses the landing buffer
    using RI = typename P64::RI;
    if constexpr (RI::STAGES == 2 && gcd_c(RI::R0, RI::R1) == 1)
        FftRunPfa<typename P64::Row, +1, L, T>::template run<true>(src, xc, dst);
    else
        FftRun<typename P64::Row, +1, L, T, RowMap, false, double2>::template run<true>(src, xc, dst,
                                                                                       tw2);
    double v = dst.best_v;
    uint32_t i = dst.best_i;
    warp_argmax(v, i);
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) {
        rv[w] = v;
        ri[w] = i;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int k = 1; k < (T + 31) / 32; ++k) argmax_merge(v, i, rv[k], ri[k]);
        const size_t o = (size_t)(pair0 + blockIdx.y) * P64::NBLK + blockIdx.x;
        part_v[o] = v;
        part_i[o] = i;
    }
}

// ------------------------------------------------------------------ D4w ---
// D4 as a warp-per-row kernel (the fp32 K4w design in double): each warp walks a contiguous run
// of ROW_L-row blocks, the next row landing by bulk copy (per-warp mbarrier) as soon as stage 1
// has read the current one, with no CTA-wide barrier; the C2R pre-pass runs in place on the
// landed row, the prime-factor 29 x 24 transform on the warp (WarpFftPfa in double), and each
// stage-2 lane keeps a running (max |x|, smallest index) over the block's rows; at the block's
// end one warp reduction writes the block partial D5 reduces.  (The CTA version lost a third of
// its stall samples to the landing wait and its two barriers, ncu r02_ncu_d4.txt.)
constexpr int D4W_WARPS = 10;   // 10 x 22.4 KB of landing + exchange: one CTA per SM

template <class PL>
struct D4w {
    using RI = typename PL::RI;
    static constexpr size_t QROW = sizeof(double2) * PL::WP;          // a landed Q row
    static constexpr size_t XCH = sizeof(double2) * RI::R1 * RI::R0;   // exchange (PAD 0)
    static constexpr size_t WARP = QROW + XCH;
    static constexpr size_t OFF_WARP = 128;                            // after the mbarriers
    static constexpr size_t SMEM = OFF_WARP + D4W_WARPS * WARP;
    static constexpr bool OK = RI::STAGES == 2 && gcd_c(RI::R0, RI::R1) == 1 && RI::R0 % 2 == 1 &&
                               RI::R0 <= 32 && RI::R1 <= 32 && PL::H % PL::ROW_L == 0 &&
                               QROW % 16 == 0 && SMEM <= 227 * 1024;
};

template <int R1, int C1, int C2, int N>
struct WarpArgmaxD {   // a lane's running (max |x|, smallest index) over the rows of a block
    double best_v;
    uint32_t best_i;
    int row_base, W;
    __device__ __forceinline__ void store_pfa(int k1, const double2 (&v)[R1]) {
        double m = fmax(fabs(v[0].x), fabs(v[0].y));
#pragma unroll
        for (int j = 1; j < R1; ++j) m = fmax(m, fmax(fabs(v[j].x), fabs(v[j].y)));
        if (m >= best_v) {
            const uint32_t base = (uint32_t)row_base * W;
            uint32_t idx = 0xFFFFFFFFu, n = (uint32_t)((C1 * k1) % N);
#pragma unroll
            for (int j = 0; j < R1; ++j) {
                if (fabs(v[j].x) == m) idx = min(idx, base + 2 * n);
                if (fabs(v[j].y) == m) idx = min(idx, base + 2 * n + 1);
                n += C2;
                if (n >= (uint32_t)N) n -= N;
            }
            best_i = m > best_v ? idx : min(idx, best_i);
            best_v = m;
        }
    }
};

template <class PL>
__global__ void __launch_bounds__(32 * D4W_WARPS, 1)
    d4w_pair_rows(const double2* __restrict__ Q, double* __restrict__ part_v,
                  uint32_t* __restrict__ part_i, int pair0, int npairs,
                  const double2* __restrict__ twW) {
    using DW = D4w<PL>;
    using RI = typename PL::RI;
    constexpr int M = PL::M, H = PL::H, L = PL::ROW_L, NBLK = Plan64<PL>::NBLK;
    extern __shared__ __align__(128) unsigned char smem_d4w[];
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem_d4w) + (threadIdx.x >> 5);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* mine = smem_d4w + DW::OFF_WARP + warp * DW::WARP;
    double2* landw = reinterpret_cast<double2*>(mine);
    const WarpXchg<RI::R0, RI::R1, 0, double2> xc{reinterpret_cast<double2*>(mine + DW::QROW)};
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    __syncwarp();
    const long long nb = (long long)npairs * NBLK;
    const long long gw = (long long)blockIdx.x * D4W_WARPS + warp, nw = (long long)gridDim.x * D4W_WARPS;
    const int r0 = (int)(nb * gw / nw) * L, r1 = (int)(nb * (gw + 1) / nw) * L;
    auto issue = [&](int r) {
        mbar_arrive_expect_tx(bar, (uint32_t)DW::QROW);
        bulk_g2s(mine, Q + (size_t)r * PL::WP, (uint32_t)DW::QROW, bar);
    };
    if (lane == 0 && r0 < r1) issue(r0);
    using Pfa = WarpFftPfa<typename PL::Row, +1, double2>;
    WarpArgmaxD<RI::R1, Pfa::C1, Pfa::C2, M> acc{-1.0, 0xFFFFFFFFu, 0, PL::W};
    int k = 0;
    for (int r = r0; r < r1; ++r, ++k) {
        const int pl = r / H, y = r - pl * H;
        acc.row_base = y;
        mbar_wait(bar, k & 1);
        // C2R pre-processing in place (as K4w): Z[q] = X[q] + conj X[M-q] + i o,
        // Z[M-q] = conj(X[q] + conj X[M-q]) + i conj(o), o = (X[q] - conj X[M-q]) conj(w_W^q)
        for (int q = lane; 2 * q <= M; q += 32) {
            const double2 xn = landw[q], xm = landw[M - q];
            const double2 o = cmulc(make_double2(xn.x - xm.x, xn.y + xm.y), __ldg(&twW[q]));
            const double sx = xn.x + xm.x, dy = xn.y - xm.y;
            landw[q] = make_double2(sx - o.y, dy + o.x);
            if (q != 0 && 2 * q != M) landw[M - q] = make_double2(sx + o.y, o.x - dy);
        }
        __syncwarp();
        auto prefetch = [&]() {
            if (lane == 0 && r + 1 < r1) {
                fence_proxy_async();
                issue(r + 1);
            }
        };
        Pfa::run(landw, xc, acc, lane, prefetch);
        __syncwarp();                          // exchange free for the next row
        if ((y + 1) % L == 0) {                // block end: one partial per ROW_L rows
            double v = acc.best_v;
            uint32_t i = acc.best_i;
            warp_argmax(v, i);
            if (lane == 0) {
                const size_t o = (size_t)(pair0 + pl) * NBLK + y / L;
                part_v[o] = v;
                part_i[o] = i;
            }
            acc.best_v = -1.0;
            acc.best_i = 0xFFFFFFFFu;
        }
    }
}

// ------------------------------------------------------------------ D1w ---
// D1 as a warp-per-row kernel (the K1w design in double): the raw uint16 row lands by bulk
// copy (the next one prefetched after stage 1), the prime-factor 29 x 24 transform runs on the
// warp with its outputs left in their exchange slots (Z[q] at (q mod R0, q mod R1)), and the
// R2C post-pass writes the mirror pairs into the panel-blocked Gd.
constexpr int D1W_WARPS = 12;   // 168 registers: at most three warps per SM sub-partition

struct U16WordSrcD {   // z[n] = x[2n] + i x[2n+1] of a landed uint16 row (exact in double)
    const uint32_t* p;
    __device__ __forceinline__ double2 load(int n) const {
        const uint32_t u = p[n];
        return make_double2((double)(u & 0xFFFFu), (double)(u >> 16));
    }
};
template <class Xc, int R1>
struct PfaSlotDstD {   // a warp PFA's stage-2 outputs back into the slots they were read from
    Xc x;
    __device__ __forceinline__ void store_pfa(int k1, const double2 (&v)[R1]) const {
#pragma unroll
        for (int j = 0; j < R1; ++j) x.at(k1, j) = v[j];
    }
};

template <class PL>
struct D1w {
    using RI = typename PL::RI;
    static constexpr size_t RAWB = (size_t)PL::W * 2;                  // a raw row
    static constexpr size_t XCH = sizeof(double2) * RI::R1 * RI::R0;   // exchange (PAD 0)
    static constexpr size_t WARP = (RAWB + 15) / 16 * 16 + XCH;
    static constexpr size_t OFF_WARP = 128;
    static constexpr size_t SMEM = OFF_WARP + D1W_WARPS * WARP;
    static constexpr bool OK = D4w<PL>::OK && RAWB % 16 == 0 && SMEM <= 227 * 1024;
};

template <class PL>
__global__ void __launch_bounds__(32 * D1W_WARPS, 1)
    d1w_fwd_rows(const uint16_t* __restrict__ raw, double2* __restrict__ G, int tile0, int ntiles,
                 const double2* __restrict__ twW) {
    using DW = D1w<PL>;
    using RI = typename PL::RI;
    constexpr int M = PL::M, H = PL::H, R0 = RI::R0, R1 = RI::R1;
    extern __shared__ __align__(128) unsigned char smem_d1w[];
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem_d1w) + (threadIdx.x >> 5);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* mine = smem_d1w + DW::OFF_WARP + warp * DW::WARP;
    const uint32_t* land = reinterpret_cast<const uint32_t*>(mine);
    using Xc = WarpXchg<R0, R1, 0, double2>;
    const Xc xc{reinterpret_cast<double2*>(mine + (DW::WARP - DW::XCH))};
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    __syncwarp();
    const long long nrows = (long long)ntiles * H;
    const long long gw = (long long)blockIdx.x * D1W_WARPS + warp, nw = (long long)gridDim.x * D1W_WARPS;
    const int r0 = (int)(nrows * gw / nw), r1 = (int)(nrows * (gw + 1) / nw);
    auto issue = [&](int r) {                  // row r = tl * H + y of this chunk's tiles
        mbar_arrive_expect_tx(bar, (uint32_t)DW::RAWB);
        bulk_g2s(mine, raw + ((size_t)tile0 * H + r) * PL::W, (uint32_t)DW::RAWB, bar);
    };
    if (lane == 0 && r0 < r1) issue(r0);
    using Src = U16WordSrcD;
    using SlotDst = PfaSlotDstD<Xc, R1>;
    using Pfa = WarpFftPfa<typename PL::Row, -1, double2>;
    int k = 0;
    for (int r = r0; r < r1; ++r, ++k) {
        mbar_wait(bar, k & 1);
        auto prefetch = [&]() {
            if (lane == 0 && r + 1 < r1) {
                fence_proxy_async();
                issue(r + 1);
            }
        };
        SlotDst dst{xc};
        Pfa::run_src(Src{land}, xc, dst, lane, prefetch);
        __syncwarp();
        const int tl = r / H;
        const GRowD<PL> out{G + (size_t)tl * H * PL::WP, r - tl * H};
        for (int q = lane; q <= M / 2; q += 32) {
            const int qm = q == 0 ? 0 : M - q;
            const double2 zq = xc.at(q % R0, q % R1);
            const double2 zm = xc.at(qm % R0, qm % R1);
            const double2 E = make_double2(0.5 * (zq.x + zm.x), 0.5 * (zq.y - zm.y));
            const double2 O = make_double2(0.5 * (zq.y + zm.y), -0.5 * (zq.x - zm.x));
            const double2 wo = cmul(__ldg(&twW[q]), O);
            out[q] = make_double2(E.x + wo.x, E.y + wo.y);
            if (2 * q != M) out[M - q] = make_double2(E.x - wo.x, wo.y - E.y);
        }
        for (int q = M + 1 + lane; q < PL::WP; q += 32) out[q] = make_double2(0.0, 0.0);
        __syncwarp();                          // exchange free for the next row
    }
}

// ------------------------------------------------------------------ D5 ----
// One warp per pair: reduce the NBLK block partials and emit the K5/K6 key
// (bits(float(max)) << 32 | (2^32 - 1 - index)); the index is the exact double argmax.
__global__ void d5_argmax_keys(const double* __restrict__ part_v, const uint32_t* __restrict__ part_i,
                               unsigned long long* __restrict__ keys, int nblk, int npairs) {
    const int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int lane = threadIdx.x & 31;
    if (p >= npairs) return;   // warp-uniform
    double v = -1.0;
    uint32_t i = 0xFFFFFFFFu;
    for (int k = lane; k < nblk; k += 32)
        argmax_merge(v, i, part_v[(size_t)p * nblk + k], part_i[(size_t)p * nblk + k]);
    warp_argmax(v, i);
    if (lane == 0)
        keys[p] = v < 0.0 ? 0ull
                          : ((unsigned long long)__float_as_uint((float)v) << 32) | (0xFFFFFFFFu - i);
}

}  // namespace stitch
