// pciam_kernels.cuh — the PCIAM hot path (§III, Fig. 1 steps 2-7) on sm_100a.
//
// Data layout in HBM:
//   raw   uint16 [tiles][H][W]           W contiguous (the caller's tile layout)
//   raw   uint16 [slots][H][W]           tile pixels by slot (slot = tile in the resident mode;
//                                        a recycled pool slot in the bounded mode, row f1)
//   G     float2 [chunk][WP/COL_P][H][COL_P]  row-transformed tiles of a forward chunk, in
//                                        column panels (each K2 panel one contiguous run)
//   spec  u32    [slots][WP][HP]         half spectrum kx in [0, W/2] (WP = pad16(W/2+1)),
//                                        COLUMN-major (ky contiguous, pitch HP = H rounded up to
//                                        4 mod 8 words), stored as its Q15 unit phasor F/|F|
//                                        (2 x int16), reused by <= 4 pairs: K3's
//                                        column panel of a tile is one contiguous run
//   Q     half2 / float2 [chunk][H][WP]  per-pair column-inverse intermediate (scaled fp16
//                                        pairs for the 1392x1040 plan, reading C11-Q)
//   fslot i32    [local tiles]           slot of each local tile (K1/K2 write there)
//   pairs {a, b} [pairs]                 slots of the pair's tiles (K3/K5 read there)
// (G and Q chunks are 0.38 / 0.47 GB at the default 64 / 160 chunks -- Q as scaled fp16 pairs
// for the 1392x1040 plan, Plan::Q_HALF -- and they round-trip HBM,
// DESIGN.md section 6.)
//   keys  u64    [pairs]                 packed (|c| bits << 32 | ~index) argmax per pair
//   mom   u64    [pairs][4][5]           exact integer CCF moments per candidate
//
// Kernels (one launch covers a chunk of tiles or pairs):
//   K1 fwd_rows   raw -> G      R2C along x: length-W real row as a W/2 complex FFT + post-twiddle
//                               (step 2 first half; uint16->fp32 fused into the load)
//   K2 fwd_cols   G -> spec     C2C along y on TMA-landed column panels (step 2 second half),
//                               epilogue: Q15 unit phasor
//   K3 pair_cols  2 spec -> Q   NCPS U_A conj(U_B) (exact int32) from two TMA-landed phasor panels
//                               (step 3), then the inverse C2C along y (step 4 first half)
//   K4 pair_rows  Q -> keys     C2R along x (step 4 second half) with |.| + argmax fused in the
//                               epilogue; the real correlation surface is never stored (step 5)
//   K5 ccf_mom    raw -> mom    integer moments of the 4 candidate overlaps (step 6, Fig. 3)
//   K6 finalize   mom -> pairs  CCF in fp64 from exact int128 moments, candidate selection (step 7)
#pragma once
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "async_copy.cuh"
#include "fft_engine.cuh"
#include "../../include/stitch.h"

namespace stitch {

constexpr int pad16(int x) { return (x + 15) / 16 * 16; }

// Q (the column-inverse intermediate, K3 -> K4) of the Q_HALF plans is stored as fp16 pairs
// scaled by 2^-25: |Q| <= H 32767^2 = 1.1e12 at H = 1040 becomes <= 3.3e4 (fp16 max 65504); the
// scale is exact and is carried to the reported peak height (Plan::Q_SCALE) like the Q15 one.
constexpr float Q_HALF_SCALE = 1.0f / 33554432.0f;   // 2^-25

template <class RX> struct RadixInfo;
template <int N, int R0_> struct RadixInfo<Radix<N, R0_>> {
    static constexpr int R0 = R0_, R1 = 1, STAGES = 1;
};
template <int N, int R0_, int R1_> struct RadixInfo<Radix<N, R0_, R1_>> {
    static constexpr int R0 = R0_, R1 = R1_, STAGES = 2;
};

// A compiled tile-size plan: row transform (length W/2 complex) and column
// transform (length H) radices, CTA shapes, exchange-buffer padding.
template <int W_, int H_, class RowRX, class ColRX, int ROW_L_, int ROW_T_, int COL_P_, int COL_T_,
          int ROW_PAD_, int COL_PAD_>
struct Plan {
    static constexpr int W = W_, H = H_;
    static constexpr int M = W / 2;           // complex row length
    static constexpr int WC = M + 1;          // kept bins kx in [0, M]
    static constexpr int WP = pad16(WC);      // row pitch of spectra (float2)
    // column pitch of the resident (column-major) phasor spectrum, in u32: >= H, a multiple of
    // 4 (16-byte bulk copies) and 4 mod 8, so the 8 columns of a landed panel start in 8
    // distinct 4-bank groups (conflict-free stage-1 reads)
    static constexpr int HP = H % 8 <= 4 ? H + (4 - H % 8) : H + (12 - H % 8);
    using Row = RowRX;
    using Col = ColRX;
    using RI = RadixInfo<RowRX>;
    using CI = RadixInfo<ColRX>;
    static constexpr int ROW_L = ROW_L_, ROW_T = ROW_T_;
    static constexpr int COL_P = COL_P_, COL_T = COL_T_;
    static constexpr int ROW_PAD = ROW_PAD_, COL_PAD = COL_PAD_;
    using RowX = RowXchg<RI::R0, RI::R1, ROW_PAD>;
    using ColX = ColXchg<CI::R0, CI::R1, COL_PAD, COL_P>;
    static constexpr size_t ROW_SMEM = sizeof(float2) * ROW_L * RowX::LSTRIDE;
    // column kernels: a TMA landing panel [H][COL_P] (complex, or two phasor panels), reused
    // in place as the stage exchange buffer once stage 1 has read it into registers
    // K3 lands two phasor panels [COL_P][HP] (one bulk copy each), the second 128-B aligned
    static constexpr size_t COL_PANEL_P = sizeof(uint32_t) * COL_P * HP;
    static constexpr size_t COL_PHASE_B = (COL_PANEL_P + 127) / 128 * 128;
    static constexpr size_t COL_LAND_C = sizeof(float2) * COL_P * H;
    static constexpr size_t COL_LAND_P = COL_PHASE_B + COL_PANEL_P;
    static constexpr size_t COL_LAND = COL_LAND_C > COL_LAND_P ? COL_LAND_C : COL_LAND_P;
    static constexpr size_t COL_XCH =
        CI::STAGES == 1 ? 0 : sizeof(float2) * COL_P * CI::R1 * (CI::R0 + COL_PAD);
    static constexpr size_t COL_BUF = ((COL_LAND > COL_XCH ? COL_LAND : COL_XCH) + 15) / 16 * 16;
    static constexpr int COL_TW2N = CI::R0 * (CI::R1 - 1);      // stage-2 twiddles in smem
    static constexpr size_t COL_SMEM = COL_BUF + sizeof(float2) * (COL_TW2N > 0 ? COL_TW2N : 1);
    // K2 stages its phasor panel [COL_P][HP] behind that and stores it with one bulk copy
    static constexpr size_t COL_STG_OFF = (COL_SMEM + 127) / 128 * 128;
    static constexpr size_t COL_SMEM_K2 = COL_STG_OFF + COL_PANEL_P;
    // CTAs per SM the column kernels are register-budgeted for (shared memory allows this many)
    // CTAs per SM the column kernels are built for (shared memory allows this many, <= 2:
    // the radix-40 butterfly's registers fit two 7-warp CTAs)
    static constexpr int COL_MINB_RAW = (int)((220 * 1024) / (COL_SMEM + 1024));
    static constexpr int COL_MINB = COL_MINB_RAW > 2 ? 2 : (COL_MINB_RAW < 1 ? 1 : COL_MINB_RAW);
    // stage-2 twiddle tables (w_N^{-j b}, see fft_engine.cuh)
    static constexpr int ROW_TW2 = RI::R0 * (RI::R1 - 1);
    static constexpr int COL_TW2 = CI::R0 * (CI::R1 - 1);
    // Q (K3 -> K4) as scaled fp16 pairs for the paper's large tiles (reading C11-Q: the surface
    // moves by <= ~2e-5 of its peak, 5x inside the 1e-4 near-tie margin; half the Q bytes), as
    // float2 for the small test plans, whose fewer samples leave less averaging
    static constexpr bool Q_HALF = W >= 1024;
    static constexpr double Q_SCALE = Q_HALF ? 1.0 / 33554432.0 : 1.0;
    static_assert(!Q_HALF || H * 32767.0 * 32767.0 * 1.0001 / 33554432.0 < 65504.0,
                  "scaled fp16 Q would overflow: |Q| <= H 32767^2");
    static_assert(W % 2 == 0, "W must be even");
    static_assert(Row::N == M && Col::N == H, "plan radices do not match the tile");
    static_assert(H % ROW_L == 0, "rows per CTA must divide H");
    static_assert(WP % COL_P == 0, "column panel must divide the pitch");
};

struct PairIdx {
    int32_t a, b;  // slots of A = west/north neighbour and B = tile
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

// G's panel-blocked layout: bin q of row y of a tile sits in column panel q / COL_P, whose
// H rows of COL_P bins are contiguous (K2 lands a panel with one bulk copy); a warp's 32
// consecutive bins of a row are 4 whole 64-byte runs (K1's stores stay sector-complete).
template <class PL>
struct GRow {
    float2* t;   // the tile's G block
    int y;
    __device__ __forceinline__ float2& operator[](int q) const {
        return t[((size_t)(q / PL::COL_P) * PL::H + y) * PL::COL_P + q % PL::COL_P];
    }
};

// Real-to-complex post-processing of one line (Z = the length-M complex FFT of the packed
// row, in the exchange buffer, natural order; Z[M] == Z[0]).  For q in [0, M/2]:
//   E = (Z[q] + conj Z[M-q]) / 2,  O = (Z[q] - conj Z[M-q]) / (2i)
//   X[q] = E + w_W^q O,   X[M-q] = conj(E - w_W^q O)
// (E and O of M-q are conj(E), conj(O), and w_W^{M-q} = -conj(w_W^q)), so one iteration
// writes the mirror pair; bins [M+1, WP) of the padded row are zeroed.
template <class PL, class Xc, class TwLoad>
__device__ __forceinline__ void r2c_post_line(const Xc& xc, int line, const GRow<PL>& out,
                                              const TwLoad& twq) {
    constexpr int M = PL::M;
    for (int q = threadIdx.x; q <= M / 2; q += PL::ROW_T) {
        const float2 zq = xc.nat(line, q);
        const float2 zm = xc.nat(line, q == 0 ? 0 : M - q);
        const float2 E = make_float2(0.5f * (zq.x + zm.x), 0.5f * (zq.y - zm.y));
        const float2 O = make_float2(0.5f * (zq.y + zm.y), -0.5f * (zq.x - zm.x));
        const float2 wo = cmul(twq(q), O);
        out[q] = make_float2(E.x + wo.x, E.y + wo.y);
        if (2 * q != M) out[M - q] = make_float2(E.x - wo.x, wo.y - E.y);
    }
    for (int q = M + 1 + threadIdx.x; q < PL::WP; q += PL::ROW_T) out[q] = make_float2(0.f, 0.f);
}

template <class PL>
__global__ void __launch_bounds__(PL::ROW_T) k1_fwd_rows(const uint16_t* __restrict__ raw,
                                                         float2* __restrict__ G, int tile0,
                                                         const int32_t* __restrict__ fslot,
                                                         const float2* __restrict__ tw2,
                                                         const float2* __restrict__ twW) {
    extern __shared__ float2 smem[];
    constexpr int L = PL::ROW_L, T = PL::ROW_T;
    const size_t t = (size_t)fslot[tile0 + blockIdx.y];
    const int y0 = blockIdx.x * L;
    U16RowSrc<PL> src{reinterpret_cast<const uint32_t*>(raw + (t * PL::H + y0) * PL::W)};
    typename PL::RowX xc{smem};
    // stage 2 writes Z[n] back into the slot it read it from (in place, per thread)
    FftRun<typename PL::Row, -1, L, T, RowMap>::run(src, xc, xc, tw2);
    __syncthreads();
#pragma unroll 1
    for (int line = 0; line < L; ++line)
        r2c_post_line<PL>(xc, line, GRow<PL>{G + (size_t)blockIdx.y * PL::H * PL::WP, y0 + line},
                          [&](int q) { return __ldg(&twW[q]); });
}


// ------------------------------------------------------------------ K2 ----
template <class PL>
struct PanelIOH {  // K3's output: a panel of COL_P columns of Q [H][WP] as scaled fp16 pairs
    __half2* p;
    __device__ __forceinline__ void store(int line, int n, float2 v) const {
        p[(size_t)n * PL::WP + line] = __floats2half2_rn(v.x * Q_HALF_SCALE, v.y * Q_HALF_SCALE);
    }
};

template <class PL>
struct PanelIO {  // a panel of COL_P columns of one [H][WP] complex array
    float2* p;
    __device__ __forceinline__ float2 load(int line, int n) const { return p[(size_t)n * PL::WP + line]; }
    __device__ __forceinline__ void store(int line, int n, float2 v) const { p[(size_t)n * PL::WP + line] = v; }
};

template <class PL>
struct LandSrc {  // a landed complex panel [H][COL_P] in shared memory
    const float2* s;
    __device__ __forceinline__ float2 load(int line, int n) const { return s[n * PL::COL_P + line]; }
};

// Resident spectrum code: the unit phasor F/|F| in Q15 fixed point, two signed 16-bit
// fields (bits 0-15: round(32767 Re F/|F|), bits 16-31: round(32767 Im F/|F|)).  Step 3
// needs nothing else: F_A conj(F_B) / |F_A conj(F_B)| = U_A conj(U_B) with U = F/|F|, and 0
// where F_A or F_B vanishes (reading C4): a zero F encodes as the zero phasor, so every NCPS
// product with it is exactly 0 without a flag.  Quantisation error <= 1.6e-5 per component
// (|U_q| = 1 +- 5e-5, angle +- 3e-5 rad): the correlation surface changes by a relative
// ~1e-5/sqrt(HW) at the peak, far inside the 1e-4 peak-height contract.
// Encoder (7 instructions, no atan2): r = 32767 / |v| (rsqrt, argument + 1e-36 so v = 0
// gives r finite and both fields 0); each field is rounded by the fp32 magic-number trick --
// fmaf(x, r, 1.5*2^23) holds round(x r) in two's complement in its low 16 mantissa bits --
// and the two low halves are packed with one byte permute.
__device__ __forceinline__ uint32_t phasor_q15(float2 v) {
    const float s2 = fmaf(v.x, v.x, fmaf(v.y, v.y, 1e-36f));   // floored: v = 0 -> finite r
    const float r = rsqrtf(s2) * 32767.0f;
    const float fx = fmaf(v.x, r, 12582912.0f);     // 1.5 * 2^23: ulp 1, round to nearest
    const float fy = fmaf(v.y, r, 12582912.0f);
    return __byte_perm(__float_as_uint(fx), __float_as_uint(fy), 0x5410);
}
// Decoder: the sign-extended fields (one PRMT in sign-replicate mode, one arithmetic shift)
__device__ __forceinline__ int32_t q15_lo(uint32_t w) {
    int32_t r;
    asm("prmt.b32 %0, %1, 0, 0x9910;" : "=r"(r) : "r"(w));
    return r;
}
__device__ __forceinline__ int32_t q15_hi(uint32_t w) { return (int32_t)w >> 16; }
// NCPS scale: U_A conj(U_B) in Q15 x Q15 is 32767^2 times the unit-modulus product, formed
// exactly in int32 (|.| <= |U_A| |U_B| < 1.08e9) and rounded once to fp32; the inverse
// transform is linear, so the factor is carried to the reported peak height (K6).
constexpr double NCPS_Q15_SCALE = 32767.0 * 32767.0;

template <class PL>
struct PhaseDst {  // K2 output: Q15 unit phasors of a panel [COL_P][HP] (staged in shared memory)
    uint32_t* p;
    __device__ __forceinline__ void store(int line, int n, float2 v) const {
        p[line * PL::HP + n] = phasor_q15(v);
    }
};

// L2 prefetch for the CTA `ahead` launch slots later (about one wave of resident CTAs): its
// panel is pulled from DRAM into L2 while this CTA computes, so its own TMA loads hit L2
// (the column kernels spend ~30 % of their stall samples waiting for their panel, ncu r01c).
// Returns the (panel, item) of that CTA, or item < 0 if it is past the end of the grid.
__device__ __forceinline__ void ahead_cta(int ahead, int& panel, int& item) {
    const int lin = blockIdx.y * gridDim.x + blockIdx.x + ahead;
    panel = lin % gridDim.x;
    item = lin / gridDim.x;
    if (ahead <= 0 || item >= (int)gridDim.y) item = -1;
}

// The column kernels' stage-2 twiddle table (COL_TW2N float2) joins the panel's TMA
// transaction as one bulk copy: a per-thread LDG -> STS loop here serialised an L2 round trip
// per iteration at the start of every CTA (a quarter of K3's stall samples, ncu r01).
template <class PL>
struct ColTw {
    static constexpr bool BULK = PL::COL_TW2N > 0 && (PL::COL_TW2N * 8) % 16 == 0;
    static constexpr uint32_t BYTES = BULK ? (uint32_t)(PL::COL_TW2N * 8) : 0u;
    // thread 0, inside the panel's transaction (the global table is 16-byte aligned)
    static __device__ __forceinline__ void issue(float2* tws, const float2* tw2, uint64_t* bar) {
        if constexpr (BULK) bulk_g2s(tws, tw2, BYTES, bar);
    }
    // every thread, if the table could not go by bulk copy
    static __device__ __forceinline__ void fallback(float2* tws, const float2* tw2) {
        if constexpr (!BULK)
            for (int i = threadIdx.x; i < PL::COL_TW2N; i += PL::COL_T) tws[i] = __ldg(tw2 + i);
    }
};

// K2: column FFT of a chunk of row-transformed tiles (G, complex), one column panel per CTA
// landed by one bulk copy (G is panel-blocked); writes the phase spectrum of each tile's slot
// (or, for the test hook, the complex spectrum row-major [H][WP] into `out`).  `ahead`: L2
// prefetch of the panel of the CTA that many launch slots later (one wave of resident CTAs:
// K2 7.25 -> 6.86 ms).
template <class PL, bool PHASE_OUT>
__global__ void __launch_bounds__(PL::COL_T, PL::COL_MINB)
    k2t_fwd_cols(const float2* __restrict__ G, float2* __restrict__ out,
                 uint32_t* __restrict__ spec, int tile0, const int32_t* __restrict__ fslot,
                 const float2* __restrict__ tw2, int ahead) {
    extern __shared__ __align__(128) unsigned char csmem[];
    __shared__ uint64_t bar;
    const int tl = blockIdx.y, c0 = blockIdx.x * PL::COL_P;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    float2* tws = reinterpret_cast<float2*>(csmem + PL::COL_BUF);
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, (uint32_t)PL::COL_LAND_C + ColTw<PL>::BYTES);
        bulk_g2s(csmem, G + ((size_t)tl * PL::WP + c0) * PL::H, (uint32_t)PL::COL_LAND_C, &bar);
        ColTw<PL>::issue(tws, tw2, &bar);
        int pn, it;
        ahead_cta(ahead, pn, it);
        if (it >= 0)
            bulk_prefetch_l2(G + ((size_t)it * PL::WP + pn * PL::COL_P) * PL::H,
                             (uint32_t)PL::COL_LAND_C);
    }
    ColTw<PL>::fallback(tws, tw2);
    mbar_wait(&bar, 0);
    LandSrc<PL> src{reinterpret_cast<const float2*>(csmem)};
    typename PL::ColX xc{reinterpret_cast<float2*>(csmem)};
    using Run = FftRun<typename PL::Col, -1, PL::COL_P, PL::COL_T, ColMap, true>;
    if constexpr (PHASE_OUT) {
        // the panel's 8 columns are contiguous in the column-major spectrum: staged in shared
        // memory (conflict-free: column pitch HP) and written with one bulk copy, instead of
        // 8 scattered 16-byte pieces per warp store
        uint32_t* stage = reinterpret_cast<uint32_t*>(csmem + PL::COL_STG_OFF);
        PhaseDst<PL> dst{stage};
        Run::template run<true>(src, xc, dst, tws);
        fence_proxy_async();
        __syncthreads();
        if (threadIdx.x == 0) {
            bulk_s2g(spec + ((size_t)fslot[tile0 + tl] * PL::WP + c0) * PL::HP, stage,
                     (uint32_t)PL::COL_PANEL_P);
            bulk_commit();
            bulk_wait_read_all();
        }
    } else {
        PanelIO<PL> dst{out + (size_t)tl * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tws);
    }
}

// ------------------------------------------------------------------ K3 ----
template <class PL>
struct NcpsPhaseSrc {  // step 3 from two landed phasor panels: U_A conj(U_B) (x 32767^2)
    const uint32_t* a;
    const uint32_t* b;
    __device__ __forceinline__ float2 load(int line, int n) const {
        const uint32_t ua = a[line * PL::HP + n], ub = b[line * PL::HP + n];
        const int32_t ax = q15_lo(ua), ay = q15_hi(ua), bx = q15_lo(ub), by = q15_hi(ub);
        return make_float2((float)(ax * bx + ay * by), (float)(ay * bx - ax * by));
    }
};

template <class PL>
__global__ void __launch_bounds__(PL::COL_T, PL::COL_MINB)
    k3t_pair_cols(const uint32_t* __restrict__ spec, float2* __restrict__ Q,
                  const PairIdx* __restrict__ pairs, int pair0, const float2* __restrict__ tw2) {
    extern __shared__ __align__(128) unsigned char csmem[];
    __shared__ uint64_t bar;
    const PairIdx pr = pairs[pair0 + blockIdx.y];
    const int c0 = blockIdx.x * PL::COL_P;
    uint32_t* la = reinterpret_cast<uint32_t*>(csmem);
    uint32_t* lb = reinterpret_cast<uint32_t*>(csmem + PL::COL_PHASE_B);
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    float2* tws = reinterpret_cast<float2*>(csmem + PL::COL_BUF);
    if (threadIdx.x == 0) {   // each tile's panel is one contiguous run: one bulk copy each
        constexpr uint32_t PB = (uint32_t)PL::COL_PANEL_P;
        mbar_arrive_expect_tx(&bar, 2 * PB + ColTw<PL>::BYTES);
        bulk_g2s(la, spec + ((size_t)pr.a * PL::WP + c0) * PL::HP, PB, &bar);
        bulk_g2s(lb, spec + ((size_t)pr.b * PL::WP + c0) * PL::HP, PB, &bar);
        ColTw<PL>::issue(tws, tw2, &bar);
    }
    ColTw<PL>::fallback(tws, tw2);
    mbar_wait(&bar, 0);
    NcpsPhaseSrc<PL> src{la, lb};
    typename PL::ColX xc{reinterpret_cast<float2*>(csmem)};
    using Run = FftRun<typename PL::Col, +1, PL::COL_P, PL::COL_T, ColMap, true>;
    if constexpr (PL::Q_HALF) {
        PanelIOH<PL> dst{reinterpret_cast<__half2*>(Q) + (size_t)blockIdx.y * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tws);
    } else {
        PanelIO<PL> dst{Q + (size_t)blockIdx.y * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tws);
    }
}

// Column lengths with a three-factor prime-factor (Good-Thomas) split into pairwise coprime
// radices that have codelets (1040 = 16 x 5 x 13): the fp64 three-pass column kernels (D2, D3)
// need no twiddles and hold at most a 16-point butterfly in registers.
template <int H> struct Pfa3 {   // no three-factor split with codelets: two-stage kernels run
    static constexpr bool OK = false;
    static constexpr int A = 1, B = 1, C = 1;
};
template <> struct Pfa3<1040> {
    static constexpr bool OK = true;
    static constexpr int A = 16, B = 5, C = 13;
};


// ------------------------------------------------------------------ K4 ----
template <class PL>
struct C2RSrc {  // complex-to-real pre-processing of row X[0..M] into Z[0..M)
    const float2* rows;    // Q rows (the CTA row kernels serve the small plans: float2 Q)
    const float2* twW;
    __device__ __forceinline__ float2 load(int line, int n) const {
        static_assert(!PL::Q_HALF, "fp16 Q is read by K4w only");
        const float2* r = rows + (size_t)line * PL::WP;
        const float2 xn = r[n];
        const float2 xm = r[PL::M - n];
        // E = X[n] + conj X[M-n];  O = (X[n] - conj X[M-n]) e^{+2 pi i n / W};  Z = E + i O
        const float2 w = __ldg(&twW[n]);
        const float2 d = make_float2(xn.x - xm.x, xn.y + xm.y);
        const float2 o = cmulc(d, w);
        return make_float2(xn.x + xm.x - o.y, xn.y - xm.y + o.x);
    }
};

struct ArgmaxDst {  // step 5: running max of |x| with its row-major index, never stored
    float best_v;      // largest |x| seen by this thread (>= 0; -1 before the first value)
    uint32_t best_i;   // its row-major index y*W + x (smallest index among equal values)
    int row_base;      // y0 of the CTA's first line
    int W;
    // Every thread stores its values in increasing index order (one butterfly per line and
    // thread in the row plans: n = b + j*R0 with j increasing), so a strict '>' keeps the
    // smallest index among equal values; across threads the packed key decides (C6).
    __device__ __forceinline__ void take(float a, uint32_t idx) {
        if (a > best_v) {
            best_v = a;
            best_i = idx;
        }
    }
    __device__ __forceinline__ void store(int line, int n, float2 v) {
        const uint32_t idx = (uint32_t)((row_base + line) * W + 2 * n);
        take(fabsf(v.x), idx);       // x[2n]
        take(fabsf(v.y), idx + 1);   // x[2n+1]
    }
    // A whole butterfly (elements b + j*STRIDE): its max |x| by FMNMX (one instruction per
    // value instead of compare + two selects), and only when that reaches the running best
    // (rare once a line is under way) the smallest index holding it.  Same result as `store`
    // value by value: the best value, ties to the smallest index (reading C6).
    static constexpr bool BATCH = true;
    template <int R, int STRIDE>
    __device__ __forceinline__ void store_batch(int line, int b, const float2 (&v)[R]) {
        float m = fmaxf(fabsf(v[0].x), fabsf(v[0].y));
#pragma unroll
        for (int j = 1; j < R; ++j) m = fmaxf(m, fmaxf(fabsf(v[j].x), fabsf(v[j].y)));
        if (m >= best_v) {
            const uint32_t base = (uint32_t)((row_base + line) * W + 2 * b);
            uint32_t idx = 0xFFFFFFFFu;
#pragma unroll
            for (int j = R - 1; j >= 0; --j) {   // ends on the smallest index holding m
                if (fabsf(v[j].y) == m) idx = base + 2 * j * STRIDE + 1;
                if (fabsf(v[j].x) == m) idx = base + 2 * j * STRIDE;
            }
            if (m > best_v || idx < best_i) best_i = idx;
            best_v = m;
        }
    }
    // packed key: larger |x| wins, then the smaller index (reading C6)
    __device__ __forceinline__ unsigned long long key() const {
        if (best_v < 0.f) return 0ull;
        return ((unsigned long long)__float_as_uint(best_v) << 32) | (0xFFFFFFFFu - best_i);
    }
};

template <int T>
__device__ __forceinline__ unsigned long long block_max_u64(unsigned long long v) {
    __shared__ unsigned long long red[(T + 31) / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xFFFFFFFFu, v, o));
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) red[w] = v;
    __syncthreads();
    if (threadIdx.x < 32) {
        v = threadIdx.x < (T + 31) / 32 ? red[threadIdx.x] : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xFFFFFFFFu, v, o));
    }
    return v;
}

// Test hook (stitch_debug_surface): the correlation surface |x| * scale stored row-major
// [H][W] instead of reduced (the same transform, so the same values the argmax sees).
struct SurfaceDst {
    float* out;
    int row_base, W;
    float scale;
    __device__ __forceinline__ void store(int line, int n, float2 v) const {
        float* o = out + (size_t)(row_base + line) * W + 2 * n;
        o[0] = fabsf(v.x) * scale;
        o[1] = fabsf(v.y) * scale;
    }
};

// CTA row kernel (plans whose row transform is not a two-stage warp FFT: 48x40, 58x26).
// SURF: the test hook's surface output instead of the argmax.
template <class PL, bool SURF = false>
__global__ void __launch_bounds__(PL::ROW_T) k4_pair_rows(const float2* __restrict__ Q,
                                                          unsigned long long* __restrict__ keys,
                                                          int pair0,
                                                          const float2* __restrict__ tw2,
                                                          const float2* __restrict__ twW,
                                                          float* __restrict__ surf = nullptr,
                                                          float scale = 0.f) {
    extern __shared__ float2 smem[];
    constexpr int L = PL::ROW_L, T = PL::ROW_T;
    const int y0 = blockIdx.x * L;
    C2RSrc<PL> src{Q + ((size_t)blockIdx.y * PL::H + y0) * PL::WP, twW};
    typename PL::RowX xc{smem};
    if constexpr (SURF) {
        SurfaceDst dst{surf, y0, PL::W, scale};
        FftRun<typename PL::Row, +1, L, T, RowMap>::run(src, xc, dst, tw2);
    } else {
        ArgmaxDst dst{-1.f, 0xFFFFFFFFu, y0, PL::W};
        FftRun<typename PL::Row, +1, L, T, RowMap>::run(src, xc, dst, tw2);
        const unsigned long long best = block_max_u64<T>(dst.key());
        if (threadIdx.x == 0) atomicMax(&keys[pair0 + blockIdx.y], best);
    }
}

}  // namespace stitch
#include "warp_rows.cuh"
namespace stitch {

// ------------------------------------------------------------------ K5 ----
// Candidate overlaps of pair p (Fig. 2 l.8-11 unified, Fig. 3): candidate (dx, dy) has
// region a = A[dy:H, dx:W], b = B[0:H-dy, 0:W-dx].  c1 = (x, y) and c2 = (W-x, y) share
// their rows (dy = y: A rows y.., B rows 0..H-y-1), and so do c3 = (x, H-y) and
// c4 = (W-x, H-y) (dy = H-y).  Row group g (0: c1/c2, 1: c3/c4) is cut into blocks of
// CCF_ROWS rows; a CTA stages CCF_BATCH rows of A and B at a time in shared memory (TMA bulk
// copies, double-buffered: each tile row is read once for both candidates) and one warp
// takes one staged row, pairing every B pixel b = B[i][j] with both of its partners
//   candidate dx = x   : a = A[dy+i][x + j],      j <  W - x
//   candidate dx = W-x : a = A[dy+i][W - x + j],  j <  x
// two pixels per 32-bit shared load (an odd offset dx is realigned with one funnel shift),
// accumulating the exact integer moments Sa, Sb, Saa, Sbb, Sab (u32 sums, u64 wide MADs).
constexpr int CCF_ROWS = 64;   // rows of one group per CTA
constexpr int CCF_BATCH = 4;   // rows staged in shared memory at a time (one warp per row)
constexpr int CCF_T = 32 * CCF_BATCH;
constexpr int CCF_PAD = 16;    // bytes after each staging buffer (the realigned loads of an
                               // odd dx read one pixel past the row's end, never used)

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
    return v;
}

struct Moments {  // exact per-lane totals
    unsigned long long sa = 0, sb = 0, saa = 0, sbb = 0, sab = 0;
    __device__ __forceinline__ void add(uint32_t a, uint32_t b) {
        sa += a;
        sb += b;
        saa += (unsigned long long)a * a;
        sbb += (unsigned long long)b * b;
        sab += (unsigned long long)a * b;
    }
};

// Packed-pixel moments with 16x8-bit integer dot products (IDP.2A): for words wa = (a0, a1),
// wb = (b0, b1) of two 16-bit pixels each, one byte permute gives wb' = (b0 lo byte, b1 lo
// byte, b0 hi byte, b1 hi byte), and dp2a_lo(wa, wb') + 256 dp2a_hi(wa, wb') = a0 b0 + a1 b1
// exactly, so Saa, Sbb, Sab take two dot products each per pixel pair of words and Sa, Sb one
// (against the byte vector (1, 1)), with no unpacking: 2 PRMT + 8 IDP per two pixel pairs
// instead of 4 unpacks, 6 wide multiplies and 8 adds (the u64 accumulation made the ALU pipe
// K5's bottleneck, ncu).  Each u32 sum grows by < 2 * 65535 * 256 = 2^25 per call, so it is
// flushed into the exact u64 totals at most every 127 calls (flush_rows()).
struct MomentsPk {
    uint32_t sa = 0, sb = 0, saa_l = 0, saa_h = 0, sbb_l = 0, sbb_h = 0, sab_l = 0, sab_h = 0;
    __device__ __forceinline__ void add2(uint32_t wa, uint32_t wb) {
        const uint32_t pa = __byte_perm(wa, 0, 0x3120), pb = __byte_perm(wb, 0, 0x3120);
        sa = __dp2a_lo(wa, 0x0101u, sa);
        sb = __dp2a_lo(wb, 0x0101u, sb);
        saa_l = __dp2a_lo(wa, pa, saa_l);
        saa_h = __dp2a_hi(wa, pa, saa_h);
        sbb_l = __dp2a_lo(wb, pb, sbb_l);
        sbb_h = __dp2a_hi(wb, pb, sbb_h);
        sab_l = __dp2a_lo(wa, pb, sab_l);
        sab_h = __dp2a_hi(wa, pb, sab_h);
    }
    __device__ __forceinline__ void flush(Moments& m) {
        m.sa += sa;
        m.sb += sb;
        m.saa += saa_l + ((unsigned long long)saa_h << 8);
        m.sbb += sbb_l + ((unsigned long long)sbb_h << 8);
        m.sab += sab_l + ((unsigned long long)sab_h << 8);
        *this = MomentsPk();
    }
};
// rows a warp may accumulate between flushes: a row gives one candidate set at most
// ceil(W/2 / 32) + 1 calls (the +1: the odd-width tail is added to the u64 totals directly)
template <int W>
struct CcfFlush {
    static constexpr int CALLS = (W / 2 + 31) / 32;
    static constexpr int ROWS = 127 / CALLS > 0 ? 127 / CALLS : 1;
};

// Moments of one candidate over one staged row: a = ar[off + j], b = br[j], j < w; lane l
// takes the pixel pairs (2q, 2q+1), q = l + 32k; an odd w leaves pixel w-1 to lane 0.
template <bool ODD>
__device__ __forceinline__ void row_moments_pk(MomentsPk& m, Moments& mt, const uint16_t* ar,
                                               const uint16_t* br, int off, int w, int lane) {
    const uint32_t* b32 = reinterpret_cast<const uint32_t*>(br);
    const uint32_t* a32 = reinterpret_cast<const uint32_t*>(ar + off - (ODD ? 1 : 0));
    const int npk = w >> 1;
#pragma unroll 4
    for (int q = lane; q < npk; q += 32) {
        uint32_t wa;
        if constexpr (ODD) wa = __funnelshift_r(a32[q], a32[q + 1], 16);
        else wa = a32[q];
        m.add2(wa, b32[q]);
    }
    if ((w & 1) && lane == 0) mt.add(ar[off + w - 1], br[w - 1]);
}

template <int W, int H>
__global__ void __launch_bounds__(CCF_T) k5_ccf_moments(const uint16_t* __restrict__ raw,
                                                        const PairIdx* __restrict__ pairs,
                                                        const unsigned long long* __restrict__ keys,
                                                        unsigned long long* __restrict__ mom,
                                                        int pair0) {
    static_assert(W % 2 == 0, "packed pixel pairs need an even row length");
    constexpr bool BULK = (W * 2) % 16 == 0;   // rows 16-byte aligned: TMA bulk copies
    constexpr int BUFS = BULK ? 2 : 1;
    constexpr int BUFB = (2 * CCF_BATCH * W * 2 + CCF_PAD + 15) / 16 * 16;   // bytes per buffer
    extern __shared__ __align__(16) unsigned char ccf_smem[];
    __shared__ unsigned long long red[10][CCF_T / 32];
    __shared__ uint64_t bar[2];
    const int p = pair0 + blockIdx.y;
    const PairIdx pr = pairs[p];
    const uint32_t lo = 0xFFFFFFFFu - (uint32_t)(keys[p] & 0xFFFFFFFFull);
    const int x = (int)(lo % (uint32_t)W), y = (int)(lo / (uint32_t)W);
    const int nb0 = (H - y + CCF_ROWS - 1) / CCF_ROWS;
    int g, i0, hg;
    if ((int)blockIdx.x < nb0) { g = 0; i0 = blockIdx.x * CCF_ROWS; hg = H - y; }
    else { g = 1; i0 = (blockIdx.x - nb0) * CCF_ROWS; hg = y; }
    if (i0 >= hg) return;                      // block-uniform
    const int dy = g ? H - y : y;
    const int rows_total = min(CCF_ROWS, hg - i0);
    const int nbatch = (rows_total + CCF_BATCH - 1) / CCF_BATCH;
    const uint16_t* A = raw + (size_t)pr.a * H * W + (size_t)(dy + i0) * W;
    const uint16_t* B = raw + (size_t)pr.b * H * W + (size_t)i0 * W;
    auto bufA = [&](int buf) { return reinterpret_cast<uint16_t*>(ccf_smem + buf * BUFB); };
    auto bufB = [&](int buf) { return bufA(buf) + CCF_BATCH * W; };
    auto issue = [&](int bi) {  // TMA bulk copy of batch bi (A rows and B rows) into buffer bi&1
        const int rows = min(CCF_BATCH, rows_total - bi * CCF_BATCH);
        const uint32_t bytes = (uint32_t)(rows * W * 2);
        uint64_t* br = &bar[bi & 1];
        mbar_arrive_expect_tx(br, 2 * bytes);
        bulk_g2s(bufA(bi & 1), A + (size_t)bi * CCF_BATCH * W, bytes, br);
        bulk_g2s(bufB(bi & 1), B + (size_t)bi * CCF_BATCH * W, bytes, br);
    };
    if constexpr (BULK) {
        if (threadIdx.x == 0) {
            mbar_init(&bar[0], 1);
            mbar_init(&bar[1], 1);
            fence_mbar_init();
        }
        __syncthreads();
        if (threadIdx.x == 0) issue(0);
    }
    const int w0 = W - x, lane = threadIdx.x & 31, rrow = threadIdx.x >> 5;
    const bool odd = x & 1;                    // dx = x and dx = W - x have the same parity
    Moments m0, m1;                            // exact totals, candidates dx = x and W - x
    MomentsPk p0, p1;                          // running packed sums
    constexpr int FLUSH = CcfFlush<W>::ROWS;
    for (int bi = 0; bi < nbatch; ++bi) {
        const int rows = min(CCF_BATCH, rows_total - bi * CCF_BATCH);
        const int buf = bi % BUFS;
        if constexpr (BULK) {
            // prefetch the next batch into the other buffer (freed by the barrier that
            // ended batch bi-1), then wait for this one
            if (threadIdx.x == 0 && bi + 1 < nbatch) {
                fence_proxy_async();
                issue(bi + 1);
            }
            mbar_wait(&bar[buf], (bi >> 1) & 1);
        } else {                               // rows not 16-byte aligned: plain staging
            const int n = rows * W;
            for (int q = threadIdx.x; q < n; q += CCF_T) {
                bufA(0)[q] = __ldg(A + (size_t)bi * CCF_BATCH * W + q);
                bufB(0)[q] = __ldg(B + (size_t)bi * CCF_BATCH * W + q);
            }
            __syncthreads();
        }
        if (rrow < rows) {                     // warp-uniform
            const uint16_t* ar = bufA(buf) + rrow * W;
            const uint16_t* br = bufB(buf) + rrow * W;
            if (odd) {
                row_moments_pk<true>(p0, m0, ar, br, x, w0, lane);    // candidate dx = x
                row_moments_pk<true>(p1, m1, ar, br, w0, x, lane);    // candidate dx = W - x
            } else {
                row_moments_pk<false>(p0, m0, ar, br, x, w0, lane);
                row_moments_pk<false>(p1, m1, ar, br, w0, x, lane);
            }
            if (bi % FLUSH == FLUSH - 1) {
                p0.flush(m0);
                p1.flush(m1);
            }
        }
        __syncthreads();                       // buffer free for batch bi+2
    }
    p0.flush(m0);
    p1.flush(m1);
    unsigned long long v[10] = {m0.sa, m0.sb, m0.saa, m0.sbb, m0.sab,
                                m1.sa, m1.sb, m1.saa, m1.sbb, m1.sab};
    const int warp = threadIdx.x >> 5;
#pragma unroll
    for (int q = 0; q < 10; ++q) {
        v[q] = warp_sum_u64(v[q]);
        if (lane == 0) red[q][warp] = v[q];
    }
    __syncthreads();
    if (threadIdx.x < 10) {
        unsigned long long s = 0;
#pragma unroll
        for (int w = 0; w < CCF_T / 32; ++w) s += red[threadIdx.x][w];
        const int c = 2 * g + threadIdx.x / 5;  // candidate index 0..3 (c1..c4)
        atomicAdd(&mom[((size_t)p * 4 + c) * 5 + threadIdx.x % 5], s);
    }
}

inline size_t k5_smem_bytes(int W) {
    const size_t bufb = ((size_t)2 * CCF_BATCH * W * 2 + CCF_PAD + 15) / 16 * 16;
    return (size_t)((W * 2) % 16 == 0 ? 2 : 1) * bufb;
}
inline int k5_grid_x(int H) { return H / CCF_ROWS + 2; }

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
                            stitch_pair* __restrict__ out, int H, int W, int npairs,
                            double peak_div) {
    const int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= npairs) return;
    const unsigned long long key = keys[p];
    const uint32_t lo = 0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFull);
    const int x = (int)(lo % (uint32_t)W), y = (int)(lo / (uint32_t)W);
    stitch_pair r;
    r.peak_x = x;
    r.peak_y = y;
    // peak_div = W*H (fp64 path), W*H*32767^2 (fp32 path: Q15 phasor NCPS, see phasor_q15)
    r.peak = (float)((double)__uint_as_float((uint32_t)(key >> 32)) / peak_div);
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
