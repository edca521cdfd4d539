// warp_rows.cuh — warp-per-line row kernels (K1w, K4w): no CTA-wide barriers.
//
// The row transforms (length M = W/2 = R0*R1 with R0, R1 <= 32) are small enough for one
// warp: stage 1 gives each of R1 lanes a radix-R0 butterfly, stage 2 each of R0 lanes a
// radix-R1 butterfly, with the exchange in the warp's own shared-memory slice and
// __syncwarp between the stages.  Each warp streams a contiguous range of rows: the next
// row lands by TMA bulk copy (per-warp mbarrier) as soon as stage 1 has read the current
// one.  Warps never wait for each other, so the scheduler always has independent work
// (the CTA-level versions K1p/K4p lose ~1/3 of their stall cycles at barriers).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

#include <cuda_fp16.h>

#include "async_copy.cuh"
#include "fft_engine.cuh"

namespace stitch {

// Exchange slot of element (u < R0, v < R1): v*(R0+PAD) + u; natural index n = v*R0 + u.
template <int R0, int R1, int PAD, class C = float2>
struct WarpXchg {
    C* s;
    static constexpr int SIZE = R1 * (R0 + PAD);
    __device__ __forceinline__ C& at(int u, int v) const { return s[v * (R0 + PAD) + u]; }
    __device__ __forceinline__ C& nat(int n) const {
        if constexpr (PAD == 0)
            return s[n];
        else
            return at(n % R0, n / R0);
    }
    __device__ __forceinline__ void store(int, int n, C v) const { nat(n) = v; }
};

template <class RX, int SIGN, int PAD>
struct WarpFft2;

template <int N, int R0, int R1, int SIGN, int PAD>
struct WarpFft2<Radix<N, R0, R1>, SIGN, PAD> {
    static_assert(R0 <= 32 && R1 <= 32, "warp FFT: radices must fit a warp");
    using Xc = WarpXchg<R0, R1, PAD>;
    // src.load(0, n), dst.store(0, n, v); tw2s: stage-2 twiddles [b*(R1-1) + j-1] (shared)
    template <class Src, class Dst, class Mid>
    static __device__ __forceinline__ void run(const Src& src, const Xc& xc, Dst& dst,
                                               const float2* tw2s, int lane, const Mid& mid) {
        if (lane < R1) {                       // stage 1: radix R0, butterfly b = lane
            float2 v[R0];
#pragma unroll
            for (int j = 0; j < R0; ++j) v[j] = src.load(0, lane + j * R1);
            Dft<R0, SIGN>::run(v);
#pragma unroll
            for (int j = 0; j < R0; ++j) xc.at(j, lane) = v[j];
        }
        __syncwarp();
        mid();                                 // source fully read: prefetch the next line
        if (lane < R0) {                       // stage 2: radix R1, butterfly b = lane
            float2 v[R1];
#pragma unroll
            for (int j = 0; j < R1; ++j) v[j] = xc.at(lane, j);
            const float2* tw = tw2s + lane * (R1 - 1);
#pragma unroll
            for (int j = 1; j < R1; ++j) v[j] = SIGN < 0 ? cmul(v[j], tw[j - 1]) : cmulc(v[j], tw[j - 1]);
            Dft<R1, SIGN>::run(v);
            store_butterfly<R1, R0>(dst, 0, lane, v);
        }
    }
};

// Prime-factor (Good-Thomas) variant for coprime radices (696 = 29 x 24): no twiddles between
// the stages, only index maps --
//   stage-1 input  n = (R1 a + R0 b) mod M   (a < R0: element of butterfly b < R1)
//   stage-2 output k = (C1 k1 + C2 k2) mod M, C1 = R1 (R1^-1 mod R0), C2 = R0 (R0^-1 mod R1)
// (k1 < R0: the stage-2 butterfly, k2 < R1: its output).  The input map wraps once per
// butterfly, at a lane-dependent a, so each load picks one of two base pointers; the
// destination receives whole butterflies (store_pfa) and maps indices itself.

template <class RX, int SIGN, class C = float2>
struct WarpFftPfa;

template <int N, int R0, int R1, int SIGN, class C>
struct WarpFftPfa<Radix<N, R0, R1>, SIGN, C> {
    static constexpr bool OK = gcd_c(R0, R1) == 1 && R0 <= 32 && R1 <= 32;
    static constexpr int C1 = (R1 * modinv(R1 % R0, R0)) % N;
    static constexpr int C2 = (R0 * modinv(R0 % R1, R1)) % N;
    template <class Xc, class Dst, class Mid>
    static __device__ __forceinline__ void run(const C* z, const Xc& xc, Dst& dst, int lane,
                                               const Mid& mid) {
        struct Ptr {
            const C* z;
            __device__ __forceinline__ C load(int n) const { return z[n]; }
        };
        run_src(Ptr{z}, xc, dst, lane, mid);
    }
    // the same with a source functor src.load(n) (element n of the sequence)
    template <class Src, class Xc, class Dst, class Mid>
    static __device__ __forceinline__ void run_src(const Src& src, const Xc& xc, Dst& dst,
                                                   int lane, const Mid& mid) {
        if (lane < R1) {                       // stage 1: radix R0, butterfly b = lane
            const int n1 = R0 * lane;          // n = R0 b + R1 a, minus N once it passes N
            const int aw = (N - R0 * lane + R1 - 1) / R1;
            C v[R0];
#pragma unroll
            for (int a = 0; a < R0; ++a) v[a] = src.load(n1 + a * R1 - (a < aw ? 0 : N));
            Dft<R0, SIGN>::run(v);
#pragma unroll
            for (int a = 0; a < R0; ++a) xc.at(a, lane) = v[a];
        }
        __syncwarp();
        mid();
        if (lane < R0) {                       // stage 2: radix R1, butterfly k1 = lane
            C v[R1];
#pragma unroll
            for (int j = 0; j < R1; ++j) v[j] = xc.at(lane, j);
            Dft<R1, SIGN>::run(v);
            dst.store_pfa(lane, v);
        }
    }
};

constexpr int ROWW_WARPS = 8;   // warps per CTA of the warp-per-line kernels
#ifndef ROWW_MINB1
#define ROWW_MINB1 2            // CTAs per SM the registers are budgeted for (K1w)
#endif
#ifndef ROWW_MINB4
#define ROWW_MINB4 2            // (K4w)
#endif

template <class PL>
struct RowWarp {
    using RI = typename PL::RI;
    static constexpr int PAD = (RI::R0 % 2 == 0) ? 1 : 0;        // odd stride across lanes
    using Fft = WarpFft2<typename PL::Row, -1, PAD>;
    using IFft = WarpFft2<typename PL::Row, +1, PAD>;
    static constexpr int XCH = RI::R1 * (RI::R0 + PAD);          // float2 per warp
    static constexpr int RAWB = PL::W * 2;                       // raw row bytes (K1)
    static constexpr int QROW = PL::WP * 8;                      // Q row bytes (K4)
    static constexpr size_t OFF_TW2 = 64;                        // after 8 mbarriers
    static constexpr size_t OFF_TWW = OFF_TW2 + (size_t)(PL::ROW_TW2 > 0 ? PL::ROW_TW2 : 1) * 8;
    static constexpr size_t OFF_WARP = (OFF_TWW + (size_t)(PL::M + 1) * 8 + 127) / 128 * 128;
    static constexpr size_t WARP_K1 = ((size_t)RAWB + 15) / 16 * 16 + (size_t)XCH * 8;
    static constexpr size_t SMEM_K1 = OFF_WARP + ROWW_WARPS * WARP_K1;
    // K4: the landed Q row (fp16 pairs, or float2), the C2R-processed row Z (float2), the exchange; the
    // stage-2 twiddle table only for the Stockham rows (the prime-factor rows need none); w_W
    // is read through L1
    static constexpr int QROWH = PL::WP * (PL::Q_HALF ? 4 : 8);   // a landed Q row
    static constexpr size_t ZROW = ((size_t)PL::M * 8 + 15) / 16 * 16;
    static constexpr size_t WARP_K4 = (size_t)QROWH + ZROW + (size_t)XCH * 8;
    template <bool PFA>
    static constexpr size_t OFF_WARP4 =
        (OFF_TW2 + (PFA ? 0 : (size_t)(PL::ROW_TW2 > 0 ? PL::ROW_TW2 : 1) * 8) + 127) / 128 * 128;
    template <bool PFA>
    static constexpr size_t SMEM_K4 = OFF_WARP4<PFA> + ROWW_WARPS * WARP_K4;
    static constexpr bool OK = RI::STAGES == 2 && RAWB % 16 == 0;
};

template <class PL>
__device__ __forceinline__ void rowwarp_tables(float2* tw2s, float2* twWs, const float2* tw2,
                                               const float2* twW) {
    for (int i = threadIdx.x; i < PL::ROW_TW2; i += 32 * ROWW_WARPS) tw2s[i] = __ldg(tw2 + i);
    for (int i = threadIdx.x; i <= PL::M; i += 32 * ROWW_WARPS) twWs[i] = __ldg(twW + i);
}

// ------------------------------------------------------------------ K1w ----
template <class PL>
__global__ void __launch_bounds__(32 * ROWW_WARPS, ROWW_MINB1)
    k1w_fwd_rows(const uint16_t* __restrict__ raw, float2* __restrict__ G, int tile0, int ntiles,
                 const int32_t* __restrict__ fslot, const float2* __restrict__ tw2,
                 const float2* __restrict__ twW) {
    using RW = RowWarp<PL>;
    constexpr int M = PL::M, H = PL::H;
    extern __shared__ __align__(128) unsigned char smem_w[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem_w);
    float2* tw2s = reinterpret_cast<float2*>(smem_w + RW::OFF_TW2);
    float2* twWs = reinterpret_cast<float2*>(smem_w + RW::OFF_TWW);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* mine = smem_w + RW::OFF_WARP + warp * RW::WARP_K1;
    const uint32_t* land = reinterpret_cast<const uint32_t*>(mine);
    typename RW::Fft::Xc xc{reinterpret_cast<float2*>(mine + (RW::WARP_K1 - RW::XCH * 8))};
    uint64_t* bar = &bars[warp];
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    rowwarp_tables<PL>(tw2s, twWs, tw2, twW);
    __syncthreads();                           // the only CTA-wide barrier
    const long long nrows = (long long)ntiles * H;
    const long long gw = (long long)blockIdx.x * ROWW_WARPS + warp, nw = (long long)gridDim.x * ROWW_WARPS;
    const int r0 = (int)(nrows * gw / nw), r1 = (int)(nrows * (gw + 1) / nw);
    auto issue = [&](int r) {                  // row r = tl*H + y of this chunk, tile in its slot
        const int tl = r / H;
        const size_t slot = (size_t)__ldg(fslot + tile0 + tl);
        mbar_arrive_expect_tx(bar, RW::RAWB);
        bulk_g2s(mine, raw + (slot * H + (r - tl * H)) * PL::W, RW::RAWB, bar);
    };
    if (lane == 0 && r0 < r1) issue(r0);
    int k = 0;
    for (int r = r0; r < r1; ++r, ++k) {
        mbar_wait(bar, k & 1);
        struct Src {
            const uint32_t* p;
            __device__ __forceinline__ float2 load(int, int n) const {
                const uint32_t u = p[n];
                return make_float2((float)(u & 0xFFFFu), (float)(u >> 16));
            }
        } src{land};
        auto prefetch = [&]() {
            if (lane == 0 && r + 1 < r1) {
                fence_proxy_async();
                issue(r + 1);
            }
        };
        RW::Fft::run(src, xc, xc, tw2s, lane, prefetch);   // natural-order Z back in place
        __syncwarp();
        const int tl = r / H;
        const GRow<PL> out{G + (size_t)tl * H * PL::WP, r - tl * H};   // panel-blocked (K2)
        // bin q = lane + 32k sits at &out[lane] + k * 32H (4 panels further per k), its mirror
        // M - q at &out[M - lane] - k * 32H (M is a multiple of the panel width)
        static_assert(M % PL::COL_P == 0 && 32 % PL::COL_P == 0, "panel-blocked G strides");
        constexpr int STEP = 32 / PL::COL_P * H * PL::COL_P;
        float2* pf = &out[lane];
        float2* pm = &out[M - lane];
        for (int q = lane; q <= M / 2; q += 32, pf += STEP, pm -= STEP) {
            const float2 zq = xc.nat(q);
            const float2 zm = xc.nat(q == 0 ? 0 : M - q);
            const float2 E = make_float2(0.5f * (zq.x + zm.x), 0.5f * (zq.y - zm.y));
            const float2 O = make_float2(0.5f * (zq.y + zm.y), -0.5f * (zq.x - zm.x));
            const float2 wo = cmul(twWs[q], O);
            *pf = make_float2(E.x + wo.x, E.y + wo.y);
            if (2 * q != M) *pm = make_float2(E.x - wo.x, wo.y - E.y);
        }
        for (int q = M + 1 + lane; q < PL::WP; q += 32) out[q] = make_float2(0.f, 0.f);
        __syncwarp();                          // exchange free for the next row
    }
}

// ------------------------------------------------------------------ K4w ----
// Step 5 for a warp that walks consecutive rows of one correlation surface: the running
// (max |x|, smallest index) is kept warp-uniform.  Per row, each stage-2 lane reduces its
// butterfly's outputs with FMNMX3 (two values per instruction) and one REDUX gives the row
// maximum; only when that beats the running best does a lane holding it look up its index
// (smallest among equal values, then REDUX-min over the lanes).  A later row cannot win a
// tie: its indices are larger (reading C6).  |x| >= 0, so its float bits order as unsigned.
template <int NLANES>
struct WarpArgmaxDst {
    float best_v;      // -1 before the first row
    uint32_t best_i;
    int row_base, W;
    static constexpr unsigned MASK = NLANES >= 32 ? 0xFFFFFFFFu : ((1u << NLANES) - 1u);
    static constexpr bool BATCH = true;
    template <int R, int STRIDE>
    __device__ __forceinline__ void store_batch(int line, int b, const float2 (&v)[R]) {
        float m = fmaxf(fabsf(v[0].x), fabsf(v[0].y));
#pragma unroll
        for (int j = 1; j < R; ++j) m = fmaxf(m, fmaxf(fabsf(v[j].x), fabsf(v[j].y)));
        const float M = __uint_as_float(__reduce_max_sync(MASK, __float_as_uint(m)));
        if (M > best_v) {                      // warp-uniform
            uint32_t idx = 0xFFFFFFFFu;
            if (m == M) {
                const uint32_t base = (uint32_t)((row_base + line) * W + 2 * b);
#pragma unroll
                for (int j = R - 1; j >= 0; --j) {
                    if (fabsf(v[j].y) == M) idx = base + 2 * j * STRIDE + 1;
                    if (fabsf(v[j].x) == M) idx = base + 2 * j * STRIDE;
                }
            }
            best_i = __reduce_min_sync(MASK, idx);
            best_v = M;
        }
    }
};

// K4w's argmax for the prime-factor transform: as WarpArgmaxDst, with the output index of
// element k2 of butterfly k1 given by the CRT map (looked up only when a row beats the best).
template <int NLANES, int R1, int C1, int C2, int N>
struct WarpArgmaxPfa {
    float best_v;
    uint32_t best_i;
    int row_base, W;
    static constexpr unsigned MASK = NLANES >= 32 ? 0xFFFFFFFFu : ((1u << NLANES) - 1u);
    __device__ __forceinline__ void store_pfa(int k1, const float2 (&v)[R1]) {
        float m = fmaxf(fabsf(v[0].x), fabsf(v[0].y));
#pragma unroll
        for (int j = 1; j < R1; ++j) m = fmaxf(m, fmaxf(fabsf(v[j].x), fabsf(v[j].y)));
        const float M = __uint_as_float(__reduce_max_sync(MASK, __float_as_uint(m)));
        if (M > best_v) {                      // warp-uniform
            uint32_t idx = 0xFFFFFFFFu;
            if (m == M) {
                const uint32_t base = (uint32_t)row_base * W;
                uint32_t n = (uint32_t)((C1 * k1) % N);
#pragma unroll
                for (int j = 0; j < R1; ++j) {
                    if (fabsf(v[j].x) == M) idx = min(idx, base + 2 * n);
                    if (fabsf(v[j].y) == M) idx = min(idx, base + 2 * n + 1);
                    n += C2;
                    if (n >= (uint32_t)N) n -= N;
                }
            }
            best_i = __reduce_min_sync(MASK, idx);
            best_v = M;
        }
    }
};

// Test hook (stitch_debug_surface): the same two transforms with the correlation surface
// |x| * scale stored row-major instead of reduced (best_v / best_i unused).
struct WarpSurfaceDst {
    float best_v;
    uint32_t best_i;
    int row_base, W;
    float* out;
    float scale;
    static constexpr bool BATCH = true;
    template <int R, int STRIDE>
    __device__ __forceinline__ void store_batch(int line, int b, const float2 (&v)[R]) {
        float* o = out + (size_t)(row_base + line) * W;
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const int n = b + j * STRIDE;
            o[2 * n] = fabsf(v[j].x) * scale;
            o[2 * n + 1] = fabsf(v[j].y) * scale;
        }
    }
};
template <int R1, int C1, int C2, int N>
struct WarpSurfacePfa {
    float best_v;
    uint32_t best_i;
    int row_base, W;
    float* out;
    float scale;
    __device__ __forceinline__ void store_pfa(int k1, const float2 (&v)[R1]) {
        float* o = out + (size_t)row_base * W;
        int n = (C1 * k1) % N;
#pragma unroll
        for (int j = 0; j < R1; ++j) {
            o[2 * n] = fabsf(v[j].x) * scale;
            o[2 * n + 1] = fabsf(v[j].y) * scale;
            n += C2;
            if (n >= N) n -= N;
        }
    }
};

// PFA: the prime-factor row transform (WarpFftPfa + WarpArgmaxPfa) where the radices are
// coprime; otherwise Stockham with stage-2 twiddles (WarpFft2 + WarpArgmaxDst).
// SURF: the test hook's surface output (one pair, `surf` [H][W]) instead of the argmax.
template <class PL, bool PFA = false, bool SURF = false>
__global__ void __launch_bounds__(32 * ROWW_WARPS, ROWW_MINB4)
    k4w_pair_rows(const float2* __restrict__ Qf, unsigned long long* __restrict__ keys, int pair0,
                  int npairs, const float2* __restrict__ tw2, const float2* __restrict__ twW,
                  float* __restrict__ surf = nullptr, float scale = 0.f) {
    using RW = RowWarp<PL>;
    constexpr int M = PL::M, H = PL::H;
    using QT = std::conditional_t<PL::Q_HALF, __half2, float2>;   // scaled fp16 pairs, or float2
    const QT* Q = reinterpret_cast<const QT*>(Qf);
    extern __shared__ __align__(128) unsigned char smem_w[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem_w);
    float2* tw2s = reinterpret_cast<float2*>(smem_w + RW::OFF_TW2);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* mine = smem_w + RW::template OFF_WARP4<PFA> + warp * RW::WARP_K4;
    const QT* landh = reinterpret_cast<const QT*>(mine);
    float2* zrow = reinterpret_cast<float2*>(mine + RW::QROWH);
    typename RW::IFft::Xc xc{reinterpret_cast<float2*>(mine + RW::QROWH + RW::ZROW)};
    uint64_t* bar = &bars[warp];
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    if constexpr (!PFA)
        for (int i = threadIdx.x; i < PL::ROW_TW2; i += 32 * ROWW_WARPS) tw2s[i] = __ldg(tw2 + i);
    __syncthreads();                           // the only CTA-wide barrier
    const long long nrows = (long long)npairs * H;
    const long long gw = (long long)blockIdx.x * ROWW_WARPS + warp, nw = (long long)gridDim.x * ROWW_WARPS;
    const int r0 = (int)(nrows * gw / nw), r1 = (int)(nrows * (gw + 1) / nw);
    auto issue = [&](int r) {
        mbar_arrive_expect_tx(bar, RW::QROWH);
        bulk_g2s(mine, Q + (size_t)r * PL::WP, RW::QROWH, bar);
    };
    auto flush = [&](int pair, float bv, uint32_t bi) {
        unsigned long long key =
            bv < 0.f ? 0ull : ((unsigned long long)__float_as_uint(bv) << 32) | (0xFFFFFFFFu - bi);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) key = max(key, __shfl_xor_sync(0xFFFFFFFFu, key, o));
        if (lane == 0) atomicMax(&keys[pair0 + pair], key);
    };
    if (lane == 0 && r0 < r1) issue(r0);
    using Pfa = WarpFftPfa<typename PL::Row, +1>;
    using ArgAcc = std::conditional_t<PFA,
                                      WarpArgmaxPfa<RW::RI::R0, RW::RI::R1, Pfa::C1, Pfa::C2, PL::M>,
                                      WarpArgmaxDst<RW::RI::R0>>;
    using SurfAcc = std::conditional_t<PFA, WarpSurfacePfa<RW::RI::R1, Pfa::C1, Pfa::C2, PL::M>,
                                       WarpSurfaceDst>;
    using Acc = std::conditional_t<SURF, SurfAcc, ArgAcc>;
    Acc acc = [&] {
        if constexpr (SURF) return Acc{-1.f, 0xFFFFFFFFu, 0, PL::W, surf, scale};
        else return Acc{-1.f, 0xFFFFFFFFu, 0, PL::W};
    }();
    int cur = r0 < r1 ? r0 / H : -1;
    int k = 0;
    for (int r = r0; r < r1; ++r, ++k) {
        const int pl = r / H, y = r - pl * H;
        if (pl != cur) {                       // warp-uniform
            if constexpr (!SURF) flush(cur, acc.best_v, acc.best_i);
            cur = pl;
            acc.best_v = -1.f;
            acc.best_i = 0xFFFFFFFFu;
        }
        acc.row_base = y;
        mbar_wait(bar, k & 1);
        // C2R pre-processing from the landed row into the float row Z, one mirror pair
        // (q, M-q) per lane and iteration:
        //   d = X[q] - conj X[M-q],  o = d conj(w_W^q),  Z[q] = X[q] + conj X[M-q] + i o,
        //   Z[M-q] = conj(X[q] + conj X[M-q]) + i conj(o)      (w_W^{M-q} = -conj w_W^q)
        // so Z (the length-M complex sequence whose inverse FFT interleaves the real row) is
        // ready and the landing buffer free: the next row is requested right away.
        for (int q = lane; 2 * q <= M; q += 32) {
            float2 xn, xm;
            if constexpr (PL::Q_HALF) {
                xn = __half22float2(landh[q]);
                xm = __half22float2(landh[M - q]);
            } else {
                xn = landh[q];
                xm = landh[M - q];
            }
            const float2 o = cmulc(make_float2(xn.x - xm.x, xn.y + xm.y), __ldg(&twW[q]));
            const float sx = xn.x + xm.x, dy = xn.y - xm.y;
            zrow[q] = make_float2(sx - o.y, dy + o.x);
            if (q != 0 && 2 * q != M) zrow[M - q] = make_float2(sx + o.y, o.x - dy);
        }
        __syncwarp();
        if (lane == 0 && r + 1 < r1) {
            fence_proxy_async();
            issue(r + 1);
        }
        struct Src {
            const float2* z;
            __device__ __forceinline__ float2 load(int, int n) const { return z[n]; }
        } src{zrow};
        if constexpr (PFA)
            Pfa::run(zrow, xc, acc, lane, NoMid());
        else
            RW::IFft::run(src, xc, acc, tw2s, lane, NoMid());
        __syncwarp();                          // Z and the exchange free for the next row
    }
    if constexpr (!SURF)
        if (cur >= 0) flush(cur, acc.best_v, acc.best_i);
}

}  // namespace stitch
