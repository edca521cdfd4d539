// stitch_api.cu — host side of the C ABI declared in include/stitch.h.
//
// Owns the device memory plan, the pair list (Fig. 4 order), the
// launch schedule of K1..K6 (pciam_kernels.cuh) and the copy-in / copy-out.
// The runtime is deliberately small: one stream, chunked launches sized so the
// per-chunk intermediates (K1->K2 spectra, K3->K4 Q) stay in the 126 MB L2.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <new>
#include <string>
#include <type_traits>
#include <vector>

#include "../../include/stitch.h"
#include "pciam_kernels.cuh"
#include "pciam_fp64.cuh"
#include "col_groups.cuh"

using namespace stitch;

namespace {

// ------------------------------------------------------------ plan table ---
// Compiled tile-size plans (Radix lists: the row transform is W/2 complex).
//            W     H     row radices          column radices      rowL rowT colP colT rowPad colPad
using P1392 = Plan<1392, 1040, Radix<696, 29, 24>, Radix<1040, 40, 26>, 4, 128, 8, 208, 0, 1>;
using P256 = Plan<256, 192, Radix<128, 16, 8>, Radix<192, 16, 12>, 8, 128, 8, 128, 1, 1>;
using P48 = Plan<48, 40, Radix<24, 24>, Radix<40, 40>, 8, 32, 8, 32, 0, 0>;
using P58 = Plan<58, 26, Radix<29, 29>, Radix<26, 26>, 2, 32, 8, 32, 0, 0>;

// "Quad" column plans: the same transforms on 4-column panels, run by the persistent column
// kernels with three CTAs per SM, each prefetching its next panel by TMA while it computes
// (the one-panel-per-CTA kernels spend ~30 % of their stall samples waiting for their panel,
// ncu r01c).  void: no quad variant for that plan.
template <class PL> struct QuadOf { using type = void; };
template <> struct QuadOf<P1392> {
    using type = Plan<1392, 1040, Radix<696, 29, 24>, Radix<1040, 40, 26>, 4, 128, 4, 160, 0, 1>;
};
template <> struct QuadOf<P256> {
    using type = Plan<256, 192, Radix<128, 16, 8>, Radix<192, 16, 12>, 8, 128, 4, 64, 1, 1>;
};
constexpr int QUAD_MINB = 3;

struct PlanOps {
    int W, H, M, WC, WP, row_l, col_p;
    int row_r0, row_r1, col_r0, col_r1;  // stage radices (r1 = 1: single stage)
    cudaError_t (*setup)(int* grid_k1p, int* grid_k4p, int* grid_k1w, int* grid_k4w);
    void (*k1p)(const uint16_t*, float2*, int, int, const float2*, const float2*, int, cudaStream_t);
    void (*k4p)(const float2*, unsigned long long*, int, int, const float2*, const float2*, int,
                cudaStream_t);
    void (*k5)(const uint16_t*, const PairIdx*, const unsigned long long*, unsigned long long*, int,
               int, cudaStream_t);
    void (*k2p)(const CUtensorMap&, float2*, uint32_t*, int, int, const float2*, bool, int,
                cudaStream_t);
    void (*k3p)(const CUtensorMap&, float2*, const PairIdx*, int, int, const float2*, int,
                cudaStream_t);
    void (*k1w)(const uint16_t*, float2*, int, int, const float2*, const float2*, int, cudaStream_t);
    void (*k4w)(const float2*, unsigned long long*, int, int, const float2*, const float2*, int,
                cudaStream_t);
    void (*k1)(const uint16_t*, float2*, int, int, const float2*, const float2*, cudaStream_t);
    void (*k2)(const CUtensorMap&, float2*, uint32_t*, int, int, const float2*, bool, int,
               cudaStream_t);
    void (*k3)(const CUtensorMap&, float2*, const PairIdx*, int, int, const float2*, int,
               cudaStream_t);
    void (*k4)(const float2*, unsigned long long*, int, int, const float2*, const float2*,
               cudaStream_t);
    // two-group column kernels (K2g/K3g); setup_g returns the grid (0: none for this plan)
    cudaError_t (*setup_g)(int* grid);
    void (*k2g)(const CUtensorMap&, uint32_t*, int, int, const float2*, int, cudaStream_t);
    void (*k3g)(const CUtensorMap&, float2*, const PairIdx*, int, int, const float2*, int,
                cudaStream_t);
    // quad column plans (col_p_q = 0: none); setup returns the persistent grid
    int col_p_q;
    cudaError_t (*setup_q)(int* grid);
    void (*k2q)(const CUtensorMap&, float2*, uint32_t*, int, int, const float2*, int, cudaStream_t);
    void (*k3q)(const CUtensorMap&, float2*, const PairIdx*, int, int, const float2*, int,
                cudaStream_t);
    // fp64 path (f2, pciam_fp64.cuh)
    int nblk64, colp64;
    cudaError_t (*d_setup)();
    void (*d1)(const uint16_t*, double2*, int, int, const double2*, const double2*, cudaStream_t);
    void (*d2)(double2*, double2*, int, int, const double2*, bool, cudaStream_t);
    void (*d3)(const double2*, double2*, const PairIdx*, int, int, const double2*, cudaStream_t);
    void (*d4)(const double2*, double*, uint32_t*, int, int, const double2*, const double2*,
               cudaStream_t);
};

template <class K>
cudaError_t max_smem(K* kernel, size_t bytes) {
    cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)bytes);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                (int)cudaSharedmemCarveoutMaxShared);
}

// K4w runs the prime-factor row transform where the radices are coprime, unless STITCH_PFA=0
inline bool pfa_enabled() {   // read per launch (launch sequences are captured once per ctx)
    const char* env = std::getenv("STITCH_PFA");
    return !(env && env[0] == '0');
}
template <class PL>
constexpr bool k4_pfa_ok() {
    if constexpr (RowWarp<PL>::OK) return RowWarp<PL>::RI::STAGES == 2 && WarpFftPfa<typename PL::Row, 1>::OK && RowWarp<PL>::PAD == 0;
    else return false;
}
template <class PL>
cudaError_t plan_setup(int* grid_k1p, int* grid_k4p, int* grid_k1w, int* grid_k4w) {
    cudaError_t e;
    *grid_k1w = *grid_k4w = 0;
    using RP = RowPersist<PL>;
    int dev = 0, sms = 0, nb = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
        return e;
    *grid_k1p = 0;
    if (RP::K1_BULK) {
        if ((e = max_smem(k1p_fwd_rows<PL>, RP::SMEM_K1)) != cudaSuccess) return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k1p_fwd_rows<PL>, PL::ROW_T,
                                                                RP::SMEM_K1)) != cudaSuccess)
            return e;
        *grid_k1p = nb * sms;
    }
    if ((e = max_smem(k4p_pair_rows<PL>, RP::SMEM_K4)) != cudaSuccess) return e;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k4p_pair_rows<PL>, PL::ROW_T,
                                                            RP::SMEM_K4)) != cudaSuccess)
        return e;
    *grid_k4p = nb * sms;
    if ((e = max_smem(k5_ccf_moments<PL::W, PL::H>, k5_smem_bytes(PL::W))) != cudaSuccess) return e;
    if ((e = max_smem(k2p_fwd_cols<PL, true>, PL::COLP_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(k2p_fwd_cols<PL, false>, PL::COLP_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(k3p_pair_cols<PL>, PL::COLP_SMEM)) != cudaSuccess) return e;
    if constexpr (RowWarp<PL>::OK) {
        using RW = RowWarp<PL>;
        if ((e = max_smem(k1w_fwd_rows<PL>, RW::SMEM_K1)) != cudaSuccess) return e;
        if ((e = max_smem(k4w_pair_rows<PL>, RW::SMEM_K4)) != cudaSuccess) return e;
        if constexpr (k4_pfa_ok<PL>())
            if ((e = max_smem(k4w_pair_rows<PL, true>, RW::SMEM_K4)) != cudaSuccess) return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k1w_fwd_rows<PL>,
                                                                32 * ROWW_WARPS, RW::SMEM_K1)) !=
            cudaSuccess)
            return e;
        *grid_k1w = nb * sms;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k4w_pair_rows<PL>,
                                                                32 * ROWW_WARPS, RW::SMEM_K4)) !=
            cudaSuccess)
            return e;
        *grid_k4w = nb * sms;
    }
    if ((e = max_smem(k1_fwd_rows<PL>, PL::ROW_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(k4_pair_rows<PL>, PL::ROW_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(k2t_fwd_cols<PL, true>, PL::COL_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(k2t_fwd_cols<PL, false>, PL::COL_SMEM)) != cudaSuccess) return e;
    return max_smem(k3t_pair_cols<PL>, PL::COL_SMEM);
}

template <class PL>
void launch_k1(const uint16_t* raw, float2* G, int t0, int nt, const float2* twM,
               const float2* twW, cudaStream_t s) {
    k1_fwd_rows<PL><<<dim3(PL::H / PL::ROW_L, nt), PL::ROW_T, PL::ROW_SMEM, s>>>(raw, G, t0,
                                                                                 twM, twW);
}
template <class PL>
void launch_k2(const CUtensorMap& tmG, float2* G, uint32_t* spec, int t0, int nt, const float2* tw2,
               bool phase_out, int ahead, cudaStream_t s) {
    const dim3 grid(PL::WP / PL::COL_P, nt);
    if (phase_out)
        k2t_fwd_cols<PL, true><<<grid, PL::COL_T, PL::COL_SMEM, s>>>(tmG, G, spec, t0, tw2, ahead);
    else
        k2t_fwd_cols<PL, false><<<grid, PL::COL_T, PL::COL_SMEM, s>>>(tmG, G, spec, t0, tw2, 0);
}
template <class PL>
void launch_k3(const CUtensorMap& tmS, float2* Q, const PairIdx* pairs, int p0, int np,
               const float2* tw2, int ahead, cudaStream_t s) {
    k3t_pair_cols<PL><<<dim3(PL::WP / PL::COL_P, np), PL::COL_T, PL::COL_SMEM, s>>>(
        tmS, Q, pairs, p0, tw2, ahead);
}
template <class PL>
void launch_k4(const float2* Q, unsigned long long* keys, int p0, int np, const float2* twM,
               const float2* twW, cudaStream_t s) {
    k4_pair_rows<PL><<<dim3(PL::H / PL::ROW_L, np), PL::ROW_T, PL::ROW_SMEM, s>>>(Q, keys, p0,
                                                                                  twM, twW);
}

template <class PL>
void launch_k1p(const uint16_t* raw, float2* G, int t0, int nt, const float2* tw2,
                const float2* twW, int grid, cudaStream_t s) {
    const int nblk = nt * (PL::H / PL::ROW_L);
    k1p_fwd_rows<PL><<<grid < nblk ? grid : nblk, PL::ROW_T, RowPersist<PL>::SMEM_K1, s>>>(
        raw, G, t0, nt, tw2, twW);
}
template <class PL>
void launch_k4p(const float2* Q, unsigned long long* keys, int p0, int np, const float2* tw2,
                const float2* twW, int grid, cudaStream_t s) {
    const int nblk = np * (PL::H / PL::ROW_L);
    k4p_pair_rows<PL><<<grid < nblk ? grid : nblk, PL::ROW_T, RowPersist<PL>::SMEM_K4, s>>>(
        Q, keys, p0, np, tw2, twW);
}

template <class PL>
void launch_k2p(const CUtensorMap& tmG, float2* G, uint32_t* spec, int t0, int nt,
                const float2* tw2, bool phase_out, int grid, cudaStream_t s) {
    const int items = nt * (PL::WP / PL::COL_P);
    const int gx = grid < items ? grid : items;
    if (phase_out)
        k2p_fwd_cols<PL, true><<<gx, PL::COL_T, PL::COLP_SMEM, s>>>(tmG, G, spec, t0, nt, tw2);
    else
        k2p_fwd_cols<PL, false><<<gx, PL::COL_T, PL::COLP_SMEM, s>>>(tmG, G, spec, t0, nt, tw2);
}
template <class PL>
void launch_k3p(const CUtensorMap& tmS, float2* Q, const PairIdx* pairs, int p0, int np,
                const float2* tw2, int grid, cudaStream_t s) {
    const int items = np * (PL::WP / PL::COL_P);
    const int gx = grid < items ? grid : items;
    k3p_pair_cols<PL><<<gx, PL::COL_T, PL::COLP_SMEM, s>>>(tmS, Q, pairs, p0, np, tw2);
}

template <class PL>
void launch_k1w(const uint16_t* raw, float2* G, int t0, int nt, const float2* tw2,
                const float2* twW, int grid, cudaStream_t s) {
    if constexpr (RowWarp<PL>::OK) {
        const int warps = (nt * PL::H + 0) / 1;
        const int need = (warps + ROWW_WARPS - 1) / ROWW_WARPS;
        k1w_fwd_rows<PL><<<grid < need ? grid : need, 32 * ROWW_WARPS, RowWarp<PL>::SMEM_K1, s>>>(
            raw, G, t0, nt, tw2, twW);
    }
}
template <class PL>
void launch_k4w(const float2* Q, unsigned long long* keys, int p0, int np, const float2* tw2,
                const float2* twW, int grid, cudaStream_t s) {
    if constexpr (k4_pfa_ok<PL>()) {
        if (pfa_enabled()) {
            const int need = (np * PL::H + ROWW_WARPS - 1) / ROWW_WARPS;
            k4w_pair_rows<PL, true><<<grid < need ? grid : need, 32 * ROWW_WARPS,
                                      RowWarp<PL>::SMEM_K4, s>>>(Q, keys, p0, np, tw2, twW);
            return;
        }
    }
    if constexpr (RowWarp<PL>::OK) {
        const int need = (np * PL::H + ROWW_WARPS - 1) / ROWW_WARPS;
        k4w_pair_rows<PL><<<grid < need ? grid : need, 32 * ROWW_WARPS, RowWarp<PL>::SMEM_K4, s>>>(
            Q, keys, p0, np, tw2, twW);
    }
}

template <class PL>
void launch_k5(const uint16_t* raw, const PairIdx* pairs, const unsigned long long* keys,
               unsigned long long* mom, int p0, int np, cudaStream_t s) {
    k5_ccf_moments<PL::W, PL::H><<<dim3(k5_grid_x(PL::H), np), CCF_T, k5_smem_bytes(PL::W), s>>>(
        raw, pairs, keys, mom, p0);
}

// ---- two-group column kernels
template <class PL>
cudaError_t setup_g(int* grid) {
    *grid = 0;
    using CG = ColGroups<PL>;
    if constexpr (CG::OK) {
        cudaError_t e;
        int dev = 0, sms = 0, nb2 = 0, nb3 = 0;
        if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
        if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
            return e;
        if ((e = max_smem(k2g_fwd_cols<PL>, CG::SMEM)) != cudaSuccess) return e;
        if ((e = max_smem(k3g_pair_cols<PL>, CG::SMEM)) != cudaSuccess) return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb2, k2g_fwd_cols<PL>, CG::NT,
                                                                CG::SMEM)) != cudaSuccess)
            return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb3, k3g_pair_cols<PL>, CG::NT,
                                                                CG::SMEM)) != cudaSuccess)
            return e;
        *grid = std::min(nb2, nb3) * sms;
    }
    return cudaSuccess;
}
template <class PL>
void launch_k2g(const CUtensorMap& tmG, uint32_t* spec, int t0, int nt, const float2* tw2,
                int grid, cudaStream_t s) {
    using CG = ColGroups<PL>;
    if constexpr (CG::OK) {
        const int items = nt * (PL::WP / PL::COL_P);
        k2g_fwd_cols<PL><<<grid < items ? grid : items, CG::NT, CG::SMEM, s>>>(tmG, spec, t0, nt,
                                                                              tw2);
    }
}
template <class PL>
void launch_k3g(const CUtensorMap& tmS, float2* Q, const PairIdx* pairs, int p0, int np,
                const float2* tw2, int grid, cudaStream_t s) {
    using CG = ColGroups<PL>;
    if constexpr (CG::OK) {
        const int items = np * (PL::WP / PL::COL_P);
        k3g_pair_cols<PL><<<grid < items ? grid : items, CG::NT, CG::SMEM, s>>>(tmS, Q, pairs, p0,
                                                                               np, tw2);
    }
}

// ---- quad column plans
template <class PL>
cudaError_t setup_q(int* grid) {
    *grid = 0;
    using Q = typename QuadOf<PL>::type;
    if constexpr (!std::is_void<Q>::value) {
        cudaError_t e;
        int dev = 0, sms = 0, nb2 = 0, nb3 = 0;
        if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
        if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
            return e;
        auto k2 = k2p_fwd_cols<Q, true, QUAD_MINB, true>;
        auto k3 = k3p_pair_cols<Q, QUAD_MINB, true>;
        if ((e = max_smem(k2, Q::COLP_TOFF)) != cudaSuccess) return e;
        if ((e = max_smem(k3, Q::COLP_TOFF)) != cudaSuccess) return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb2, k2, Q::COL_T, Q::COLP_TOFF)) !=
            cudaSuccess)
            return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb3, k3, Q::COL_T, Q::COLP_TOFF)) !=
            cudaSuccess)
            return e;
        *grid = std::min(nb2, nb3) * sms;
    }
    return cudaSuccess;
}
template <class PL>
void launch_k2q(const CUtensorMap& tmG, float2* G, uint32_t* spec, int t0, int nt,
                const float2* tw2, int grid, cudaStream_t s) {
    using Q = typename QuadOf<PL>::type;
    if constexpr (!std::is_void<Q>::value) {
        const int items = nt * (Q::WP / Q::COL_P);
        k2p_fwd_cols<Q, true, QUAD_MINB, true><<<grid < items ? grid : items, Q::COL_T,
                                                 Q::COLP_TOFF, s>>>(tmG, G, spec, t0, nt, tw2);
    }
}
template <class PL>
void launch_k3q(const CUtensorMap& tmS, float2* Q_, const PairIdx* pairs, int p0, int np,
                const float2* tw2, int grid, cudaStream_t s) {
    using Q = typename QuadOf<PL>::type;
    if constexpr (!std::is_void<Q>::value) {
        const int items = np * (Q::WP / Q::COL_P);
        k3p_pair_cols<Q, QUAD_MINB, true><<<grid < items ? grid : items, Q::COL_T, Q::COLP_TOFF,
                                            s>>>(tmS, Q_, pairs, p0, np, tw2);
    }
}
template <class PL>
constexpr int quad_col_p() {
    using Q = typename QuadOf<PL>::type;
    if constexpr (std::is_void<Q>::value) return 0; else return Q::COL_P;
}

// ---- fp64 path launchers (f2)
template <class PL>
cudaError_t d_setup() {
    using P64 = Plan64<PL>;
    cudaError_t e;
    if ((e = max_smem(d1_fwd_rows<PL>, P64::ROW_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(d4_pair_rows<PL>, P64::ROW_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(d2_fwd_cols<PL, true>, P64::COL_SMEM)) != cudaSuccess) return e;
    if ((e = max_smem(d2_fwd_cols<PL, false>, P64::COL_SMEM)) != cudaSuccess) return e;
    return max_smem(d3_pair_cols<PL>, P64::COL_SMEM);
}
template <class PL>
void launch_d1(const uint16_t* raw, double2* G, int t0, int nt, const double2* tw2,
               const double2* twW, cudaStream_t s) {
    using P64 = Plan64<PL>;
    d1_fwd_rows<PL><<<dim3(P64::NBLK, nt), P64::ROW_T, P64::ROW_SMEM, s>>>(raw, G, t0, tw2, twW);
}
template <class PL>
void launch_d2(double2* G, double2* U, int t0, int nt, const double2* tw2, bool unit_out,
               cudaStream_t s) {
    using P64 = Plan64<PL>;
    const dim3 grid(PL::WP / P64::COL_P, nt);
    if (unit_out)
        d2_fwd_cols<PL, true><<<grid, P64::COL_T, P64::COL_SMEM, s>>>(G, U, t0, tw2);
    else
        d2_fwd_cols<PL, false><<<grid, P64::COL_T, P64::COL_SMEM, s>>>(G, U, t0, tw2);
}
template <class PL>
void launch_d3(const double2* U, double2* Q, const PairIdx* pairs, int p0, int np,
               const double2* tw2, cudaStream_t s) {
    using P64 = Plan64<PL>;
    d3_pair_cols<PL><<<dim3(PL::WP / P64::COL_P, np), P64::COL_T, P64::COL_SMEM, s>>>(U, Q, pairs,
                                                                                      p0, tw2);
}
template <class PL>
void launch_d4(const double2* Q, double* pv, uint32_t* pi, int p0, int np, const double2* tw2,
               const double2* twW, cudaStream_t s) {
    using P64 = Plan64<PL>;
    d4_pair_rows<PL><<<dim3(P64::NBLK, np), P64::ROW_T, P64::ROW_SMEM, s>>>(Q, pv, pi, p0, tw2,
                                                                            twW);
}

template <class PL>
PlanOps make_ops() {
    return PlanOps{PL::W,       PL::H,         PL::M,          PL::WC,        PL::WP,
                   PL::ROW_L,   PL::COL_P,     PL::RI::R0,     PL::RI::R1,    PL::CI::R0,
                   PL::CI::R1,  plan_setup<PL>, launch_k1p<PL>, launch_k4p<PL>, launch_k5<PL>,
                   launch_k2p<PL>, launch_k3p<PL>, launch_k1w<PL>, launch_k4w<PL>, launch_k1<PL>,
                   launch_k2<PL>, launch_k3<PL>, launch_k4<PL>, setup_g<PL>, launch_k2g<PL>,
                   launch_k3g<PL>, quad_col_p<PL>(), setup_q<PL>,
                   launch_k2q<PL>, launch_k3q<PL>, Plan64<PL>::NBLK,
                   Plan64<PL>::COL_P, d_setup<PL>, launch_d1<PL>, launch_d2<PL>, launch_d3<PL>,
                   launch_d4<PL>};
}

const PlanOps* find_plan(int W, int H) {
    static const PlanOps ops[] = {make_ops<P1392>(), make_ops<P256>(), make_ops<P48>(),
                                  make_ops<P58>()};
    for (const auto& o : ops)
        if (o.W == W && o.H == H) return &o;
    return nullptr;
}

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

// Dual pair schedule (STITCH_DUAL=1): K3 and K4 on separate streams with two Q slots, and K4's
// persistent grid limited to STITCH_DUAL_K4 CTAs per SM (default 1), so a K4 chunk and the next
// chunk's K3 share every SM: the issue-bound row kernel fills the column kernel's TMA waits.
int dual_pairs_env() {
    const char* e = std::getenv("STITCH_DUAL");
    return e && e[0] == '1';
}

// twiddle tables: row stage-2 [r0*(r1-1)], column stage-2 [c0*(c1-1)], R2C/C2R w_W [W]
// (slot counts rounded up to even, so every table starts 16-byte aligned for bulk copies)
size_t tw_row(const PlanOps* o) { return ((size_t)o->row_r0 * (o->row_r1 - 1) + 1) & ~(size_t)1; }
size_t tw_col(const PlanOps* o) { return ((size_t)o->col_r0 * (o->col_r1 - 1) + 1) & ~(size_t)1; }
size_t tw_count(const PlanOps* o) { return tw_row(o) + tw_col(o) + o->W + 2; }

struct Layout {
    int h_begin, t_begin, t_end, nlocal;
    int64_t npairs;
    int chunk_pairs, chunk_tiles;
    int prec;   // 0 fp32, 1 fp64 (f2)
    int q_slots;  // pair-chunk intermediates: 2 = K3(c+1) may run beside K4(c) (dual schedule)
    size_t off_raw, off_spec, off_g, off_q, off_pairs, off_keys, off_mom, off_res, off_tw,
        off_part, total;
};

stitch_status make_layout(const stitch_config* c, const PlanOps* ops, Layout* L) {
    const int n = c->grid_rows, m = c->grid_cols;
    const int64_t nt = (int64_t)n * m;
    L->t_begin = c->tile_begin;
    L->t_end = c->tile_end ? c->tile_end : (int)nt;
    if (L->t_begin < 0 || L->t_end > nt || L->t_begin >= L->t_end) return STITCH_ERR_INVALID_ARG;
    L->h_begin = L->t_begin - m > 0 ? L->t_begin - m : 0;
    L->nlocal = L->t_end - L->h_begin;
    int64_t np = 0;
    for (int t = L->t_begin; t < L->t_end; ++t) np += (t % m >= 1) + (t / m >= 1);
    L->npairs = np;
    if (c->precision != 0 && c->precision != 1) return STITCH_ERR_INVALID_ARG;
    L->prec = c->precision;
    // fp64 chunks of 8 keep the 94 MB intermediate (8 x H x WP x 16 B at 1392x1040) in L2
    L->chunk_pairs = c->chunk_pairs > 0 ? c->chunk_pairs : (L->prec ? 8 : 160);
    L->chunk_tiles = c->chunk_tiles > 0 ? c->chunk_tiles : (L->prec ? 8 : 64);
    if (L->chunk_pairs > 65535 || L->chunk_tiles > 65535) return STITCH_ERR_INVALID_ARG;
    const size_t H = ops->H, W = ops->W, WP = ops->WP;
    // resident spectrum: u32 Q15 unit phasor (fp32) or double2 unit phasor (fp64)
    const size_t spec_el = L->prec ? sizeof(double2) : sizeof(uint32_t);
    const size_t cplx = L->prec ? sizeof(double2) : sizeof(float2);
    size_t o = 0;
    L->off_raw = o;   o += align256((size_t)L->nlocal * H * W * sizeof(uint16_t));
    L->off_spec = o;  o += align256((size_t)L->nlocal * H * WP * spec_el);
    L->off_g = o;     o += align256((size_t)L->chunk_tiles * H * WP * cplx);
    L->q_slots = (!L->prec && dual_pairs_env()) ? 2 : 1;
    L->off_q = o;     o += align256((size_t)L->q_slots * L->chunk_pairs * H * WP * cplx);
    L->off_pairs = o; o += align256((size_t)(np > 0 ? np : 1) * sizeof(PairIdx));
    L->off_keys = o;  o += align256((size_t)(np > 0 ? np : 1) * sizeof(unsigned long long));
    L->off_mom = o;   o += align256((size_t)(np > 0 ? np : 1) * 20 * sizeof(unsigned long long));
    L->off_res = o;   o += align256((size_t)(np > 0 ? np : 1) * sizeof(stitch_pair));
    L->off_tw = o;    o += align256((size_t)(tw_count(ops)) * cplx);
    L->off_part = o;  // fp64 argmax partials: double [pairs][nblk] then u32 [pairs][nblk]
    if (L->prec) o += align256((size_t)(np > 0 ? np : 1) * ops->nblk64 * (8 + 4));
    L->total = o;
    return STITCH_OK;
}

stitch_status check_config(const stitch_config* c, const PlanOps** ops) {
    if (!c) return STITCH_ERR_INVALID_ARG;
    if (c->grid_rows < 1 || c->grid_cols < 1 || c->tile_width < 2 || c->tile_height < 1)
        return STITCH_ERR_INVALID_ARG;
    if ((int64_t)c->grid_rows * c->grid_cols > (1 << 30)) return STITCH_ERR_INVALID_ARG;
    *ops = find_plan(c->tile_width, c->tile_height);
    if (!*ops) return STITCH_ERR_UNSUPPORTED;
    if ((int64_t)c->tile_width * c->tile_height > 0x7FFFFFFF) return STITCH_ERR_UNSUPPORTED;
    return STITCH_OK;
}

}  // namespace

struct stitch_ctx {
    stitch_config cfg;
    const PlanOps* ops;
    Layout L;
    int n, m, H, W;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    char* mem = nullptr;
    bool own_mem = false;
    uint16_t* raw;
    uint32_t* spec;                   // resident Q15 phasor spectra [nlocal][H][WP]
    float2 *G, *Q, *twM, *twH, *twW;  // chunk intermediates, twiddles
    float2* Q2 = nullptr;             // second pair-chunk slot (dual schedule)
    int grid_k4w_dual = 0;            // K4w grid beside K3 (dual schedule)
    cudaStream_t s_pair4 = nullptr;   // K4 stream (dual schedule)
    std::vector<cudaEvent_t> ev_k3;   // per pair chunk: its Q is complete (dual schedule)
    int prec = 0;                     // 1: fp64 path (f2): the buffers below are used instead
    double2 *Gd = nullptr, *Qd = nullptr, *Ud = nullptr;   // Ud: resident unit phasors
    double2 *twMd = nullptr, *twHd = nullptr, *twWd = nullptr;
    double* part_v = nullptr;         // fp64 argmax partials [pairs][nblk64]
    uint32_t* part_i = nullptr;
    CUtensorMap tmG, tmS;             // TMA descriptors of G (complex) and spec (Q15 phasors)
    CUtensorMap tmG4, tmS4;           // the same with the quad plans' 4-column boxes
    int grid_colq = 0;                // quad persistent column kernels (0: not used)
    int grid_colg = 0;                // two-group column kernels (0: not used)
    int col_ahead = 0;                // K2 L2 prefetch distance in CTAs (0: off)
    int col_ahead3 = 0;               // K3 L2 prefetch distance in CTAs (0: off)
    PairIdx* pairs;
    unsigned long long *keys, *mom;
    stitch_pair* res;
    std::vector<int32_t> pair_tile;   // global tile index (B) of each pair
    std::vector<int8_t> pair_kind;    // 0 west, 1 north
    std::vector<stitch_pair> res_h;
    bool loaded = false, computed = false;
    int64_t launches = 0;
    int grid_k1p = 0, grid_k4p = 0;   // persistent-kernel grids (0: use the non-persistent kernel)
    int grid_colp = 0;                // persistent column kernels (K2p/K3p): one CTA per SM
    int grid_k1w = 0, grid_k4w = 0;   // warp-per-line row kernels (0: not used)
    // CUDA graphs of the launch sequences (captured on first use on an internal stream,
    // replayed on the caller's stream): one graph launch per step instead of ~700 launches
    bool use_graph = true;
    cudaStream_t cap_stream = nullptr;
    struct GraphRec {
        cudaGraphExec_t exec;
        int64_t launches;
    };
    std::map<uint64_t, GraphRec> graphs;
    // concurrent schedule (timing off): forward chunks, pair chunks and CCF chunks on three
    // internal streams joined by events, so compute-bound and memory-bound kernels overlap
    bool concurrent = true;
    cudaStream_t s_fwd = nullptr, s_pair = nullptr, s_ccf = nullptr, s_h2d = nullptr;
    std::vector<cudaEvent_t> ev_h2d;          // per forward chunk: its tiles have landed
    std::vector<cudaEvent_t> ev_fwd, ev_k4;   // per forward chunk / per pair chunk
    cudaEvent_t ev_fork = nullptr, ev_join[3] = {nullptr, nullptr, nullptr};
    std::vector<int> pair_need;               // forward chunk completing each pair chunk's tiles
    int timing = 0;  // 0 off, 1 per-stage events, 2 per-stage + per-launch events,
                     // 3 timeline of the concurrent schedule (events around every launch)
    struct TlRec {
        int8_t kid, stream;
        cudaEvent_t a, b;
    };
    std::vector<TlRec> tl;             // timing 3: one record per launch
    std::vector<cudaEvent_t> tl_pool;  // reusable events
    size_t tl_used = 0;
    cudaEvent_t tl_origin = nullptr;
    std::vector<float> tl_ms;          // [2 * records]: start, end relative to the fork
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
    float ms[4] = {0, 0, 0, 0};
    std::vector<cudaEvent_t> kev;     // per-launch events (timing == 2)
    std::vector<int8_t> kkind;        // kernel id of each recorded launch
    float kms[6] = {0, 0, 0, 0, 0, 0};
    int64_t kcount[6] = {0, 0, 0, 0, 0, 0};
    std::string err;
};

// Timeline (timing mode 3): an event pair around a launch on stream `s` (index si).
static cudaError_t tl_event(stitch_ctx* ctx, cudaEvent_t* out) {
    if (ctx->tl_used == ctx->tl_pool.size()) {
        cudaEvent_t e;
        cudaError_t r = cudaEventCreate(&e);
        if (r != cudaSuccess) return r;
        ctx->tl_pool.push_back(e);
    }
    *out = ctx->tl_pool[ctx->tl_used++];
    return cudaSuccess;
}
template <class F>
static cudaError_t tl_wrap(stitch_ctx* ctx, cudaStream_t s, int si, int kid, F launch) {
    if (ctx->timing != 3) {
        launch();
        return cudaSuccess;
    }
    stitch_ctx::TlRec r{(int8_t)kid, (int8_t)si, nullptr, nullptr};
    cudaError_t e;
    if ((e = tl_event(ctx, &r.a)) != cudaSuccess || (e = tl_event(ctx, &r.b)) != cudaSuccess) return e;
    if ((e = cudaEventRecord(r.a, s)) != cudaSuccess) return e;
    launch();
    if ((e = cudaEventRecord(r.b, s)) != cudaSuccess) return e;
    ctx->tl.push_back(r);
    return cudaSuccess;
}

// Per-launch event (timing mode 2): kid 0..5 = K1..K6.
static cudaError_t mark(stitch_ctx* ctx, int kid) {
    if (ctx->timing < 2) return cudaSuccess;
    const size_t i = ctx->kkind.size();
    if (i + 1 >= ctx->kev.size()) {
        const size_t old = ctx->kev.size();
        ctx->kev.resize(old ? old * 2 : 1024, nullptr);
        for (size_t j = old; j < ctx->kev.size(); ++j) {
            cudaError_t e = cudaEventCreate(&ctx->kev[j]);
            if (e != cudaSuccess) return e;
        }
    }
    ctx->kkind.push_back((int8_t)kid);
    return cudaEventRecord(ctx->kev[i + 1], ctx->stream);
}

static stitch_status fail(stitch_ctx* ctx, stitch_status s, const std::string& msg) {
    if (ctx) ctx->err = msg;
    return s;
}

static stitch_status cuda_fail(stitch_ctx* ctx, cudaError_t e, const char* where) {
    return fail(ctx, e == cudaErrorMemoryAllocation ? STITCH_ERR_OUT_OF_MEMORY : STITCH_ERR_CUDA,
                std::string(where) + ": " + cudaGetErrorString(e));
}

#define CK(call, where)                                   \
    do {                                                  \
        cudaError_t e_ = (call);                          \
        if (e_ != cudaSuccess) return cuda_fail(ctx, e_, where); \
    } while (0)

extern "C" {

const char* stitch_status_string(stitch_status s) {
    switch (s) {
        case STITCH_OK: return "ok";
        case STITCH_ERR_INVALID_ARG: return "invalid argument";
        case STITCH_ERR_UNSUPPORTED: return "unsupported tile size";
        case STITCH_ERR_OUT_OF_MEMORY: return "out of device memory";
        case STITCH_ERR_CUDA: return "CUDA error";
        case STITCH_ERR_STATE: return "invalid call order";
    }
    return "unknown status";
}

stitch_status stitch_workspace_size(const stitch_config* cfg, size_t* bytes) {
    const PlanOps* ops;
    if (!bytes) return STITCH_ERR_INVALID_ARG;
    stitch_status s = check_config(cfg, &ops);
    if (s != STITCH_OK) return s;
    Layout L;
    if ((s = make_layout(cfg, ops, &L)) != STITCH_OK) return s;
    *bytes = L.total;
    return STITCH_OK;
}

stitch_status stitch_pair_count(const stitch_config* cfg, int64_t* count) {
    const PlanOps* ops;
    if (!count) return STITCH_ERR_INVALID_ARG;
    stitch_status s = check_config(cfg, &ops);
    if (s != STITCH_OK) return s;
    Layout L;
    if ((s = make_layout(cfg, ops, &L)) != STITCH_OK) return s;
    *count = L.npairs;
    return STITCH_OK;
}

void stitch_destroy(stitch_ctx* ctx) {
    if (!ctx) return;
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    for (auto& e : ctx->ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->kev)
        if (e) cudaEventDestroy(e);
    for (auto& g : ctx->graphs) cudaGraphExecDestroy(g.second.exec);
    if (ctx->cap_stream) cudaStreamDestroy(ctx->cap_stream);
    for (auto& e : ctx->ev_fwd)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->ev_k4)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->ev_h2d)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->ev_k3)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->tl_pool)
        if (e) cudaEventDestroy(e);
    if (ctx->s_pair4) cudaStreamDestroy(ctx->s_pair4);
    if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
    for (auto& e : ctx->ev_join)
        if (e) cudaEventDestroy(e);
    for (cudaStream_t st : {ctx->s_fwd, ctx->s_pair, ctx->s_ccf, ctx->s_h2d})
        if (st) cudaStreamDestroy(st);
    if (ctx->own_mem && ctx->mem) cudaFree(ctx->mem);
    if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
    delete ctx;
}

stitch_status stitch_init(const stitch_config* cfg, stitch_ctx** out) {
    if (!out) return STITCH_ERR_INVALID_ARG;
    *out = nullptr;
    const PlanOps* ops;
    stitch_status s = check_config(cfg, &ops);
    if (s != STITCH_OK) return s;
    Layout L;
    if ((s = make_layout(cfg, ops, &L)) != STITCH_OK) return s;
    if (cfg->workspace && cfg->workspace_bytes < L.total) return STITCH_ERR_INVALID_ARG;
    if (cfg->workspace && (reinterpret_cast<uintptr_t>(cfg->workspace) & 255))
        return STITCH_ERR_INVALID_ARG;

    stitch_ctx* ctx = new (std::nothrow) stitch_ctx();
    if (!ctx) return STITCH_ERR_OUT_OF_MEMORY;
    ctx->cfg = *cfg;
    ctx->ops = ops;
    ctx->L = L;
    ctx->n = cfg->grid_rows;
    ctx->m = cfg->grid_cols;
    ctx->H = ops->H;
    ctx->W = ops->W;
    auto bail = [&](stitch_status st) {
        stitch_destroy(ctx);
        return st;
    };
    cudaError_t e = cudaSetDevice(cfg->device);
    if (e != cudaSuccess) return bail(STITCH_ERR_CUDA);
    if ((e = ops->setup(&ctx->grid_k1p, &ctx->grid_k4p, &ctx->grid_k1w, &ctx->grid_k4w)) !=
        cudaSuccess)
        return bail(STITCH_ERR_CUDA);
    ctx->prec = L.prec;
    if (ctx->prec && (e = ops->d_setup()) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    {
        const char* wenv = std::getenv("STITCH_ROWWARP");   // STITCH_ROWWARP=0: CTA row kernels
        if (wenv && wenv[0] == '0') ctx->grid_k1w = ctx->grid_k4w = 0;
    }
    {
        // column-kernel variant: one CTA per panel (default: several CTAs per SM overlap each
        // other's TMA waits) or persistent with TMA prefetch (STITCH_COL_PERSIST=1; one CTA
        // per SM, measured slower on B200: fewer resident warps)
        const char* env = std::getenv("STITCH_COL_PERSIST");
        int sms = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cfg->device);
        ctx->grid_colp = (env && env[0] == '1') ? sms : 0;
        // K2 / K3: L2 prefetch of the panels of the CTA one wave ahead (STITCH_L2PF /
        // STITCH_L2PF3 = <CTAs>, 0 = off).  Measured: K2 7.25 -> 6.85 ms at one wave (2 CTAs
        // x SMs); K3 slower (11.18 -> 11.53 ms: its prefetch needs the next pair's tile
        // indices, a dependent global load in the prologue), so off for K3 by default.
        {
            const char* pf = std::getenv("STITCH_L2PF");
            ctx->col_ahead = pf ? std::atoi(pf) : 2 * sms;
            const char* pf3 = std::getenv("STITCH_L2PF3");
            ctx->col_ahead3 = pf3 ? std::atoi(pf3) : 0;
        }
        // two-group persistent column kernels (STITCH_COLG=1)
        {
            const char* genv2 = std::getenv("STITCH_COLG");
            if (!ctx->prec && genv2 && genv2[0] == '1')
                if ((e = ops->setup_g(&ctx->grid_colg)) != cudaSuccess) return bail(STITCH_ERR_CUDA);
        }
        // quad persistent column kernels (STITCH_COLQ=1; measured slower on B200, ncu r01q:
        // the panel prefetch removes the TMA wait (30 % -> 3 % of K3's stall samples) but the
        // 104-of-160-thread stage 1 leaves 22 % at barriers and the L1 twiddle loads another
        // ~20 %: K3 11.2 -> 15.6 ms per step)
        const char* qenv = std::getenv("STITCH_COLQ");
        if (!ctx->prec && ops->col_p_q > 0 && qenv && qenv[0] == '1') {
            if ((e = ops->setup_q(&ctx->grid_colq)) != cudaSuccess) return bail(STITCH_ERR_CUDA);
        }
        const char* genv = std::getenv("STITCH_GRAPH");   // STITCH_GRAPH=0: direct launches
        ctx->use_graph = !(genv && genv[0] == '0');
        const char* cenv = std::getenv("STITCH_CONCURRENT");  // STITCH_CONCURRENT=0: one stream
        ctx->concurrent = !(cenv && cenv[0] == '0') && !ctx->prec;
        if (ctx->concurrent) {
            for (cudaStream_t* st : {&ctx->s_fwd, &ctx->s_pair, &ctx->s_ccf, &ctx->s_h2d})
                if (cudaStreamCreateWithFlags(st, cudaStreamNonBlocking) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
            const int nf = (L.nlocal + L.chunk_tiles - 1) / L.chunk_tiles;
            const int nc = (int)((L.npairs + L.chunk_pairs - 1) / L.chunk_pairs);
            ctx->ev_fwd.assign(nf, nullptr);
            ctx->ev_h2d.assign(nf, nullptr);
            ctx->ev_k4.assign(nc, nullptr);
            for (auto& e : ctx->ev_h2d)
                if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
            if (L.q_slots == 2 && ctx->grid_k4w > 0) {
                if (cudaStreamCreateWithFlags(&ctx->s_pair4, cudaStreamNonBlocking) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
                ctx->ev_k3.assign(nc, nullptr);
                for (auto& e : ctx->ev_k3)
                    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                        return bail(STITCH_ERR_CUDA);
                const char* ke = std::getenv("STITCH_DUAL_K4");
                const int per_sm = ke ? std::max(1, std::atoi(ke)) : 1;
                int sms = 0;
                cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cfg->device);
                ctx->grid_k4w_dual = std::min(ctx->grid_k4w, per_sm * sms);
            }
            for (auto& e : ctx->ev_fwd)
                if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
            for (auto& e : ctx->ev_k4)
                if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
            if (cudaEventCreateWithFlags(&ctx->ev_fork, cudaEventDisableTiming) != cudaSuccess)
                return bail(STITCH_ERR_CUDA);
            for (auto& e : ctx->ev_join)
                if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                    return bail(STITCH_ERR_CUDA);
        }
        if (ctx->use_graph &&
            cudaStreamCreateWithFlags(&ctx->cap_stream, cudaStreamNonBlocking) != cudaSuccess)
            return bail(STITCH_ERR_CUDA);
    }

    if (cfg->stream) {
        ctx->stream = (cudaStream_t)cfg->stream;
    } else {
        if (cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking) != cudaSuccess)
            return bail(STITCH_ERR_CUDA);
        ctx->own_stream = true;
    }
    if (cfg->workspace) {
        ctx->mem = (char*)cfg->workspace;
    } else {
        e = cudaMalloc(&ctx->mem, L.total);
        if (e != cudaSuccess)
            return bail(e == cudaErrorMemoryAllocation ? STITCH_ERR_OUT_OF_MEMORY : STITCH_ERR_CUDA);
        ctx->own_mem = true;
    }
    char* b = ctx->mem;
    ctx->raw = (uint16_t*)(b + L.off_raw);
    ctx->spec = (uint32_t*)(b + L.off_spec);
    ctx->G = (float2*)(b + L.off_g);
    ctx->Q = (float2*)(b + L.off_q);
    if (L.q_slots == 2) ctx->Q2 = ctx->Q + (size_t)L.chunk_pairs * ops->H * ops->WP;
    ctx->pairs = (PairIdx*)(b + L.off_pairs);
    ctx->keys = (unsigned long long*)(b + L.off_keys);
    ctx->mom = (unsigned long long*)(b + L.off_mom);
    ctx->res = (stitch_pair*)(b + L.off_res);
    ctx->twM = (float2*)(b + L.off_tw);
    ctx->twH = ctx->twM + tw_row(ops);
    ctx->twW = ctx->twH + tw_col(ops);
    if (ctx->prec) {
        ctx->Ud = (double2*)(b + L.off_spec);
        ctx->Gd = (double2*)(b + L.off_g);
        ctx->Qd = (double2*)(b + L.off_q);
        ctx->twMd = (double2*)(b + L.off_tw);
        ctx->twHd = ctx->twMd + tw_row(ops);
        ctx->twWd = ctx->twHd + tw_col(ops);
        const size_t np1 = (size_t)(L.npairs > 0 ? L.npairs : 1) * ops->nblk64;
        ctx->part_v = (double*)(b + L.off_part);
        ctx->part_i = (uint32_t*)(b + L.off_part + np1 * sizeof(double));
    }

    // TMA descriptors (driver entry point through the runtime; no libcuda link needed);
    // the fp64 path uses plain loads
    if (!ctx->prec) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) !=
                cudaSuccess || !fn)
            return bail(STITCH_ERR_CUDA);
        auto encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
        const cuuint32_t boxh = (cuuint32_t)(ops->H / ((ops->H + 255) / 256));
        const cuuint32_t estr[2] = {1, 1};
        // G: complex chunk [chunk_tiles*H][WP] as floats; spec: u32 Q15 phasors [nlocal*H][WP]
        auto encode_pair = [&](CUtensorMap* mg, CUtensorMap* ms, int colp) {
            const cuuint64_t gd[2] = {(cuuint64_t)2 * ops->WP, (cuuint64_t)L.chunk_tiles * ops->H};
            const cuuint64_t gs[1] = {(cuuint64_t)ops->WP * 8};
            const cuuint32_t gb[2] = {(cuuint32_t)2 * colp, boxh};
            const cuuint64_t sd[2] = {(cuuint64_t)ops->WP, (cuuint64_t)L.nlocal * ops->H};
            const cuuint64_t ss[1] = {(cuuint64_t)ops->WP * 4};
            const cuuint32_t sb[2] = {(cuuint32_t)colp, boxh};
            return encode(mg, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, ctx->G, gd, gs, gb, estr,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS &&
                   encode(ms, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, ctx->spec, sd, ss, sb, estr,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
        };
        if (!encode_pair(&ctx->tmG, &ctx->tmS, ops->col_p)) return bail(STITCH_ERR_CUDA);
        if (ctx->grid_colq > 0 && !encode_pair(&ctx->tmG4, &ctx->tmS4, ops->col_p_q))
            return bail(STITCH_ERR_CUDA);
    }

    // Twiddles w_N^e = exp(-2 pi i e / N), computed in double, rounded once.
    //   stage-2 tables: tw2[b*(r1-1) + j-1] = w_N^{j b}, b < r0, 1 <= j < r1 (fft_engine.cuh)
    std::vector<float2> tw(tw_count(ops));
    auto w = [](long e, long N) {
        const double a = -2.0 * M_PI * (double)(e % N) / (double)N;
        return make_float2((float)std::cos(a), (float)std::sin(a));
    };
    auto fill2 = [&](float2* dst, int r0, int r1) {
        const int N = r0 * r1;
        for (int bb = 0; bb < r0; ++bb)
            for (int j = 1; j < r1; ++j) dst[(size_t)bb * (r1 - 1) + j - 1] = w((long)j * bb, N);
    };
    fill2(tw.data(), ops->row_r0, ops->row_r1);
    fill2(tw.data() + tw_row(ops), ops->col_r0, ops->col_r1);
    for (int k = 0; k < ops->W; ++k) tw[tw_row(ops) + tw_col(ops) + k] = w(k, ops->W);

    // Pair list: every owned tile's west and north pair, as (neighbour, tile) (Fig. 4).
    // Processing order (results do not depend on it): tiles in bands of PAIR_BAND tile
    // rows, column-major inside a band, so a tile's spectrum and raw pixels are reused by
    // its <= 4 pairs while still in L2 (the paper's traversal-order idea).
    // 4 rows: a tile's west-pair reuse 8 pairs (~90 MB of panels and Q) after its first use
    // stays in the 126 MB L2 (bands of 1-8 measured: 3-4 best, K3 10.81 -> 10.63 ms), and the
    // first pair chunk waits for 4 tile rows of forward transforms instead of 8.
    // STITCH_PAIR_BAND overrides (experiments).
    int PAIR_BAND = 4;
    if (const char* benv = std::getenv("STITCH_PAIR_BAND")) PAIR_BAND = std::max(1, std::atoi(benv));
    std::vector<int> order;
    order.reserve((size_t)(L.t_end - L.t_begin));
    for (int t = L.t_begin; t < L.t_end; ++t) order.push_back(t);
    const int mm = ctx->m;
    std::stable_sort(order.begin(), order.end(), [mm, PAIR_BAND](int a, int b) {
        const int ra = a / mm, rb = b / mm, ba = ra / PAIR_BAND, bb = rb / PAIR_BAND;
        if (ba != bb) return ba < bb;
        if (a % mm != b % mm) return a % mm < b % mm;
        return ra < rb;
    });
    std::vector<PairIdx> pl;
    pl.reserve((size_t)L.npairs);
    for (const int t : order) {
        const int r = t / ctx->m, c = t % ctx->m;
        if (c >= 1) {
            pl.push_back(PairIdx{t - 1 - L.h_begin, t - L.h_begin});
            ctx->pair_tile.push_back(t);
            ctx->pair_kind.push_back(0);
        }
        if (r >= 1) {
            pl.push_back(PairIdx{t - ctx->m - L.h_begin, t - L.h_begin});
            ctx->pair_tile.push_back(t);
            ctx->pair_kind.push_back(1);
        }
    }
    ctx->res_h.resize((size_t)L.npairs);
    // forward chunk that completes every tile a pair chunk reads (concurrent schedule)
    for (int64_t p0 = 0; p0 < L.npairs; p0 += L.chunk_pairs) {
        int mx = 0;
        for (int64_t p = p0; p < L.npairs && p < p0 + L.chunk_pairs; ++p)
            mx = std::max(mx, std::max(pl[(size_t)p].a, pl[(size_t)p].b));
        ctx->pair_need.push_back(mx / L.chunk_tiles);
    }
    // fp64 twiddles: the same tables, rounded once to double
    std::vector<double2> twd;
    if (ctx->prec) {
        twd.resize(tw_count(ops));
        auto wd = [](long e2, long N) {
            const double a = -2.0 * M_PI * (double)(e2 % N) / (double)N;
            return make_double2(std::cos(a), std::sin(a));
        };
        auto fill2d = [&](double2* dst, int r0, int r1) {
            const int N = r0 * r1;
            for (int bb = 0; bb < r0; ++bb)
                for (int j = 1; j < r1; ++j) dst[(size_t)bb * (r1 - 1) + j - 1] = wd((long)j * bb, N);
        };
        fill2d(twd.data(), ops->row_r0, ops->row_r1);
        fill2d(twd.data() + tw_row(ops), ops->col_r0, ops->col_r1);
        for (int k = 0; k < ops->W; ++k) twd[tw_row(ops) + tw_col(ops) + k] = wd(k, ops->W);
        if ((e = cudaMemcpyAsync(ctx->twMd, twd.data(), twd.size() * sizeof(double2),
                                 cudaMemcpyHostToDevice, ctx->stream)) != cudaSuccess)
            return bail(STITCH_ERR_CUDA);
    } else if ((e = cudaMemcpyAsync(ctx->twM, tw.data(), tw.size() * sizeof(float2),
                                    cudaMemcpyHostToDevice, ctx->stream)) != cudaSuccess)
        return bail(STITCH_ERR_CUDA);
    if (!pl.empty() &&
        (e = cudaMemcpyAsync(ctx->pairs, pl.data(), pl.size() * sizeof(PairIdx),
                             cudaMemcpyHostToDevice, ctx->stream)) != cudaSuccess)
        return bail(STITCH_ERR_CUDA);
    for (auto& ev : ctx->ev)
        if (cudaEventCreate(&ev) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    if ((e = cudaStreamSynchronize(ctx->stream)) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    *out = ctx;
    return STITCH_OK;
}

static stitch_status load_common(stitch_ctx* ctx, const uint16_t* src, size_t n_bytes,
                                 cudaMemcpyKind kind) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!src) return fail(ctx, STITCH_ERR_INVALID_ARG, "null grid pointer");
    const size_t tile = (size_t)ctx->H * ctx->W;
    if (n_bytes != (size_t)ctx->n * ctx->m * tile * sizeof(uint16_t))
        return fail(ctx, STITCH_ERR_INVALID_ARG, "n_bytes != n*m*H*W*2");
    CK(cudaMemcpyAsync(ctx->raw, src + (size_t)ctx->L.h_begin * tile,
                       (size_t)ctx->L.nlocal * tile * sizeof(uint16_t), kind, ctx->stream),
       "load grid");
    ctx->loaded = true;
    ctx->computed = false;
    return STITCH_OK;
}

stitch_status stitch_load_tiles(stitch_ctx* ctx, const uint16_t* tiles, int32_t first_tile,
                                int32_t count, int32_t on_device) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!tiles) return fail(ctx, STITCH_ERR_INVALID_ARG, "null tiles pointer");
    if (first_tile > ctx->L.h_begin || first_tile + (int64_t)count < ctx->L.t_end || first_tile < 0)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range does not cover [halo_begin, tile_end)");
    const size_t tile = (size_t)ctx->H * ctx->W;
    CK(cudaMemcpyAsync(ctx->raw, tiles + (size_t)(ctx->L.h_begin - first_tile) * tile,
                       (size_t)ctx->L.nlocal * tile * sizeof(uint16_t),
                       on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, ctx->stream),
       "load tiles");
    ctx->loaded = true;
    ctx->computed = false;
    return STITCH_OK;
}

stitch_status stitch_resident_range(stitch_ctx* ctx, int32_t* halo_begin, int32_t* tile_begin,
                                    int32_t* tile_end) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (halo_begin) *halo_begin = ctx->L.h_begin;
    if (tile_begin) *tile_begin = ctx->L.t_begin;
    if (tile_end) *tile_end = ctx->L.t_end;
    return STITCH_OK;
}

stitch_status stitch_load_grid(stitch_ctx* ctx, const uint16_t* host_grid, size_t n_bytes) {
    return load_common(ctx, host_grid, n_bytes, cudaMemcpyHostToDevice);
}

stitch_status stitch_load_grid_device(stitch_ctx* ctx, const uint16_t* dev_grid, size_t n_bytes) {
    return load_common(ctx, dev_grid, n_bytes, cudaMemcpyDeviceToDevice);
}

// K6's divisor of the argmax value: max|c| / (W H) (C5); the fp32 path's NCPS carries the
// Q15 phasor scale 32767^2 (pciam_kernels.cuh, phasor_q15).
static double k6_peak_div(const stitch_ctx* ctx) {
    const double wh = (double)ctx->W * (double)ctx->H;
    return ctx->prec ? wh : wh * NCPS_Q15_SCALE;
}

// Row kernels: warp-per-line (K1w/K4w) where the plan allows, else
// persistent CTA rows (K1p/K4p), else one CTA per row block (K1/K4).
static void launch_k1_any(stitch_ctx* ctx, int t0, int nt, cudaStream_t s) {
    const PlanOps* o = ctx->ops;
    if (ctx->grid_k1w > 0)
        o->k1w(ctx->raw, ctx->G, t0, nt, ctx->twM, ctx->twW, ctx->grid_k1w, s);
    else if (ctx->grid_k1p > 0)
        o->k1p(ctx->raw, ctx->G, t0, nt, ctx->twM, ctx->twW, ctx->grid_k1p, s);
    else
        o->k1(ctx->raw, ctx->G, t0, nt, ctx->twM, ctx->twW, s);
}
static void launch_k4_any(stitch_ctx* ctx, int p0, int np, cudaStream_t s,
                          const float2* Qp = nullptr, int grid_w = 0) {
    const PlanOps* o = ctx->ops;
    const float2* q = Qp ? Qp : ctx->Q;
    if (ctx->grid_k4w > 0)
        o->k4w(q, ctx->keys, p0, np, ctx->twM, ctx->twW, grid_w > 0 ? grid_w : ctx->grid_k4w, s);
    else if (ctx->grid_k4p > 0)
        o->k4p(q, ctx->keys, p0, np, ctx->twM, ctx->twW, ctx->grid_k4p, s);
    else
        o->k4(q, ctx->keys, p0, np, ctx->twM, ctx->twW, s);
}

// Column kernels: quad persistent (3 CTAs/SM, TMA prefetch) where available, else the
// persistent single-CTA variant if requested, else one CTA per panel.
static void launch_k2_any(stitch_ctx* ctx, int t0, int nt, cudaStream_t s) {
    const PlanOps* o = ctx->ops;
    if (ctx->grid_colg > 0)
        o->k2g(ctx->tmG, ctx->spec, t0, nt, ctx->twH, ctx->grid_colg, s);
    else if (ctx->grid_colq > 0)
        o->k2q(ctx->tmG4, ctx->G, ctx->spec, t0, nt, ctx->twH, ctx->grid_colq, s);
    else if (ctx->grid_colp > 0)
        o->k2p(ctx->tmG, ctx->G, ctx->spec, t0, nt, ctx->twH, true, ctx->grid_colp, s);
    else
        o->k2(ctx->tmG, ctx->G, ctx->spec, t0, nt, ctx->twH, true, ctx->col_ahead, s);
}
static void launch_k3_any(stitch_ctx* ctx, int p0, int np, cudaStream_t s,
                          float2* Qp = nullptr) {
    const PlanOps* o = ctx->ops;
    float2* q = Qp ? Qp : ctx->Q;
    if (ctx->grid_colg > 0)
        o->k3g(ctx->tmS, q, ctx->pairs, p0, np, ctx->twH, ctx->grid_colg, s);
    else if (ctx->grid_colq > 0)
        o->k3q(ctx->tmS4, q, ctx->pairs, p0, np, ctx->twH, ctx->grid_colq, s);
    else if (ctx->grid_colp > 0)
        o->k3p(ctx->tmS, q, ctx->pairs, p0, np, ctx->twH, ctx->grid_colp, s);
    else
        o->k3(ctx->tmS, q, ctx->pairs, p0, np, ctx->twH, ctx->col_ahead3, s);
}

// Forward transforms (K1 + K2) of the resident tiles with local indices [lt0, lt0 + count).
static stitch_status forward_impl(stitch_ctx* ctx, int lt0, int count) {
    const PlanOps* o = ctx->ops;
    const int ct = ctx->L.chunk_tiles;
    for (int t0 = lt0; t0 < lt0 + count; t0 += ct) {
        const int nt = lt0 + count - t0 < ct ? lt0 + count - t0 : ct;
        if (ctx->prec) {   // fp64 path (f2): D1, D2
            o->d1(ctx->raw, ctx->Gd, t0, nt, ctx->twMd, ctx->twWd, ctx->stream);
            CK(mark(ctx, 0), "event");
            o->d2(ctx->Gd, ctx->Ud, t0, nt, ctx->twHd, true, ctx->stream);
            CK(mark(ctx, 1), "event");
            ctx->launches += 2;
            continue;
        }
        launch_k1_any(ctx, t0, nt, ctx->stream);
        CK(mark(ctx, 0), "event");
        launch_k2_any(ctx, t0, nt, ctx->stream);
        CK(mark(ctx, 1), "event");
        ctx->launches += 2;
    }
    CK(cudaGetLastError(), "forward launch");
    return STITCH_OK;
}

// Steps 3-7 (K3..K6) for every pair of the range; spectra must be resident.
static stitch_status pairs_impl(stitch_ctx* ctx) {
    const PlanOps* o = ctx->ops;
    cudaStream_t s = ctx->stream;
    const int64_t np = ctx->L.npairs;
    if (np > 0) {
        CK(cudaMemsetAsync(ctx->keys, 0, (size_t)np * sizeof(unsigned long long), s), "memset");
        CK(cudaMemsetAsync(ctx->mom, 0, (size_t)np * 20 * sizeof(unsigned long long), s), "memset");
        if (ctx->timing >= 2) CK(mark(ctx, -1), "event");
        const int cp = ctx->L.chunk_pairs;
        for (int64_t p0 = 0; p0 < np; p0 += cp) {
            const int npc = (int)(np - p0 < cp ? np - p0 : cp);
            if (ctx->prec) {   // fp64 path (f2): D3, D4 (block argmax partials)
                o->d3(ctx->Ud, ctx->Qd, ctx->pairs, (int)p0, npc, ctx->twHd, s);
                CK(mark(ctx, 2), "event");
                o->d4(ctx->Qd, ctx->part_v, ctx->part_i, (int)p0, npc, ctx->twMd, ctx->twWd, s);
                CK(mark(ctx, 3), "event");
                ctx->launches += 2;
                continue;
            }
            launch_k3_any(ctx, (int)p0, npc, s);
            CK(mark(ctx, 2), "event");
            launch_k4_any(ctx, (int)p0, npc, s);
            CK(mark(ctx, 3), "event");
            ctx->launches += 2;
        }
        if (ctx->prec) {   // D5: per-pair reduction of the partials into the K5/K6 key
            d5_argmax_keys<<<(unsigned)((np + 7) / 8), 256, 0, s>>>(ctx->part_v, ctx->part_i,
                                                                   ctx->keys, o->nblk64, (int)np);
            CK(mark(ctx, 3), "event");
            ctx->launches += 1;
        }
        CK(cudaGetLastError(), "pair launch");
    }
    if (ctx->timing) CK(cudaEventRecord(ctx->ev[2], s), "event");
    if (np > 0) {
        for (int64_t p0 = 0; p0 < np; p0 += 65535) {
            const int npc = (int)(np - p0 < 65535 ? np - p0 : 65535);
            o->k5(ctx->raw, ctx->pairs, ctx->keys, ctx->mom, (int)p0, npc, s);
            CK(mark(ctx, 4), "event");
            ctx->launches += 1;
        }
        k6_finalize<<<(unsigned)((np + 127) / 128), 128, 0, s>>>(ctx->keys, ctx->mom, ctx->res,
                                                                 ctx->H, ctx->W, (int)np,
                                                                 k6_peak_div(ctx));
        CK(mark(ctx, 5), "event");
        ctx->launches += 1;
        CK(cudaGetLastError(), "ccf launch");
    }
    if (ctx->timing) CK(cudaEventRecord(ctx->ev[3], s), "event");
    ctx->computed = true;
    return STITCH_OK;
}

// Start of a step: reset launch counters and (timing modes) record the start events.
static stitch_status step_begin(stitch_ctx* ctx) {
    cudaStream_t s = ctx->stream;
    ctx->launches = 0;
    ctx->kkind.clear();
    ctx->computed = false;
    if (ctx->timing >= 2) {
        if (ctx->kev.empty()) {
            ctx->kev.resize(1024, nullptr);
            for (auto& e : ctx->kev) CK(cudaEventCreate(&e), "event create");
        }
        CK(cudaEventRecord(ctx->kev[0], s), "event");
    }
    if (ctx->timing) CK(cudaEventRecord(ctx->ev[0], s), "event");
    return STITCH_OK;
}

// Enqueue `body` (which launches on ctx->stream) directly, or -- graph mode, no event
// timing -- as a CUDA graph captured once per key on the internal capture stream and
// replayed on the caller's stream.  Every launch parameter (pointers, tensor maps, chunk
// schedule) is fixed per context, so a replay is exactly the captured sequence.
// Whole step on three streams (timing off): s_fwd runs the forward chunks (K1, K2) and
// records an event per chunk; s_pair runs the pair chunks (K3, K4), each waiting for the
// forward chunk that completes the tiles it reads; s_ccf runs K5 per pair chunk behind
// its K4, then K6.  Buffers G (s_fwd) and Q (s_pair) are only touched by one stream.
// host_src (optional): the caller's host copy of the resident tiles [h_begin, t_end); each
// forward chunk's tiles are copied on a fourth stream just before that chunk's K1, so the
// H2D of later chunks overlaps the transforms and pairs of earlier ones (step 1 pipelined
// with steps 2-7, as the paper's read/copier stages feed its GPU stages).
// forward = false: steps 3-7 only (the split multi-GPU step: spectra already resident).
static stitch_status compute_concurrent(stitch_ctx* ctx, const uint16_t* host_src = nullptr,
                                        bool forward = true) {
    const PlanOps* o = ctx->ops;
    cudaStream_t m = ctx->stream;
    const int64_t np = ctx->L.npairs;
    const int nl = ctx->L.nlocal, ct = ctx->L.chunk_tiles, cp = ctx->L.chunk_pairs;
    if (np > 0) {
        CK(cudaMemsetAsync(ctx->keys, 0, (size_t)np * sizeof(unsigned long long), m), "memset");
        CK(cudaMemsetAsync(ctx->mom, 0, (size_t)np * 20 * sizeof(unsigned long long), m), "memset");
    }
    if (ctx->timing == 3) {
        ctx->tl.clear();
        ctx->tl_used = 0;
        CK(tl_event(ctx, &ctx->tl_origin), "event");
        CK(cudaEventRecord(ctx->tl_origin, m), "event");
    }
    CK(cudaEventRecord(ctx->ev_fork, m), "fork");
    for (cudaStream_t st : {ctx->s_fwd, ctx->s_pair, ctx->s_ccf, ctx->s_h2d, ctx->s_pair4})
        if (st) CK(cudaStreamWaitEvent(st, ctx->ev_fork, 0), "fork wait");
    cudaStream_t sf = ctx->s_fwd, sp = ctx->s_pair, sk = ctx->s_ccf;
    const size_t tile_px = (size_t)ctx->H * ctx->W;
    for (int f = 0, t0 = 0; forward && t0 < nl; ++f, t0 += ct) {
        const int nt = nl - t0 < ct ? nl - t0 : ct;
        if (host_src) {
            CK(cudaMemcpyAsync(ctx->raw + (size_t)t0 * tile_px, host_src + (size_t)t0 * tile_px,
                               (size_t)nt * tile_px * sizeof(uint16_t), cudaMemcpyHostToDevice,
                               ctx->s_h2d),
               "chunk H2D");
            CK(cudaEventRecord(ctx->ev_h2d[f], ctx->s_h2d), "event");
            CK(cudaStreamWaitEvent(sf, ctx->ev_h2d[f], 0), "wait H2D");
        }
        CK(tl_wrap(ctx, sf, 0, 0, [&] { launch_k1_any(ctx, t0, nt, sf); }), "timeline");
        CK(tl_wrap(ctx, sf, 0, 1, [&] { launch_k2_any(ctx, t0, nt, sf); }), "timeline");
        CK(cudaEventRecord(ctx->ev_fwd[f], sf), "event");
        ctx->launches += 2;
    }
    int waited = -1;
    for (int c = 0; (int64_t)c * cp < np; ++c) {
        const int64_t p0 = (int64_t)c * cp;
        const int npc = (int)(np - p0 < cp ? np - p0 : cp);
        const int need = ctx->pair_need[c];
        if (forward && need > waited) {
            CK(cudaStreamWaitEvent(sp, ctx->ev_fwd[need], 0), "wait forward");
            waited = need;
        }
        if (ctx->s_pair4) {   // dual schedule: slot c&1, K3 and K4 on their own streams
            float2* q = (c & 1) ? ctx->Q2 : ctx->Q;
            if (c >= 2) CK(cudaStreamWaitEvent(sp, ctx->ev_k4[c - 2], 0), "wait slot");
            launch_k3_any(ctx, (int)p0, npc, sp, q);
            CK(cudaEventRecord(ctx->ev_k3[c], sp), "event");
            CK(cudaStreamWaitEvent(ctx->s_pair4, ctx->ev_k3[c], 0), "wait k3");
            launch_k4_any(ctx, (int)p0, npc, ctx->s_pair4, q, ctx->grid_k4w_dual);
            CK(cudaEventRecord(ctx->ev_k4[c], ctx->s_pair4), "event");
        } else {
            CK(tl_wrap(ctx, sp, 1, 2, [&] { launch_k3_any(ctx, (int)p0, npc, sp); }), "timeline");
            CK(tl_wrap(ctx, sp, 1, 3, [&] { launch_k4_any(ctx, (int)p0, npc, sp); }), "timeline");
            CK(cudaEventRecord(ctx->ev_k4[c], sp), "event");
        }
        CK(cudaStreamWaitEvent(sk, ctx->ev_k4[c], 0), "wait k4");
        CK(tl_wrap(ctx, sk, 2, 4, [&] {
               o->k5(ctx->raw, ctx->pairs, ctx->keys, ctx->mom, (int)p0, npc, sk);
           }), "timeline");
        ctx->launches += 3;
    }
    if (np > 0) {
        CK(tl_wrap(ctx, sk, 2, 5, [&] {
               k6_finalize<<<(unsigned)((np + 127) / 128), 128, 0, sk>>>(
                   ctx->keys, ctx->mom, ctx->res, ctx->H, ctx->W, (int)np, k6_peak_div(ctx));
           }), "timeline");
        ctx->launches += 1;
    }
    CK(cudaGetLastError(), "concurrent launch");
    // (s_h2d's last copy is ordered before the last K1 on s_fwd, and every K4 on s_pair4 before
    // a K5 on s_ccf, so joining s_fwd, s_pair and s_ccf covers all streams)
    cudaStream_t ss[3] = {sf, sp, sk};
    for (int i = 0; i < 3; ++i) {
        CK(cudaEventRecord(ctx->ev_join[i], ss[i]), "join");
        CK(cudaStreamWaitEvent(m, ctx->ev_join[i], 0), "join wait");
    }
    ctx->computed = true;
    return STITCH_OK;
}

extern "C++" {
template <class F>
static stitch_status run_graphed(stitch_ctx* ctx, uint64_t key, F body) {
    if (ctx->timing || !ctx->use_graph) return body();
    auto it = ctx->graphs.find(key);
    if (it == ctx->graphs.end()) {
        cudaStream_t user = ctx->stream;
        const int64_t l0 = ctx->launches;
        ctx->stream = ctx->cap_stream;
        cudaError_t e = cudaStreamBeginCapture(ctx->cap_stream, cudaStreamCaptureModeThreadLocal);
        if (e != cudaSuccess) {
            ctx->stream = user;
            return cuda_fail(ctx, e, "begin capture");
        }
        stitch_status st = body();
        cudaGraph_t g = nullptr;
        e = cudaStreamEndCapture(ctx->cap_stream, &g);
        ctx->stream = user;
        if (st != STITCH_OK) {
            if (g) cudaGraphDestroy(g);
            return st;
        }
        if (e != cudaSuccess) return cuda_fail(ctx, e, "end capture");
        cudaGraphExec_t ex = nullptr;
        e = cudaGraphInstantiate(&ex, g, 0);
        cudaGraphDestroy(g);
        if (e != cudaSuccess) return cuda_fail(ctx, e, "graph instantiate");
        it = ctx->graphs.emplace(key, stitch_ctx::GraphRec{ex, ctx->launches - l0}).first;
        ctx->launches = l0;
    }
    CK(cudaGraphLaunch(it->second.exec, ctx->stream), "graph launch");
    ctx->launches += it->second.launches;
    return STITCH_OK;
}
}  // extern "C++" 

stitch_status stitch_forward_async(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "forward before load");
    return stitch_forward_range_async(ctx, ctx->L.h_begin, ctx->L.nlocal);
}

stitch_status stitch_forward_range_async(stitch_ctx* ctx, int32_t first_tile, int32_t count) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "forward before load");
    if (count < 0 || first_tile < ctx->L.h_begin || first_tile + (int64_t)count > ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range not resident");
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    const uint64_t key = (2ull << 60) | ((uint64_t)(uint32_t)first_tile << 30) | (uint32_t)count;
    st = run_graphed(ctx, key, [&]() { return forward_impl(ctx, first_tile - ctx->L.h_begin, count); });
    if (st == STITCH_OK && ctx->timing) CK(cudaEventRecord(ctx->ev[1], ctx->stream), "event");
    return st;
}

stitch_status stitch_pairs_async(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "pairs before load");
    stitch_status st = run_graphed(ctx, 3ull << 60, [&]() {
        // K5 on its own stream beside the K3/K4 chunks, as in the whole step
        if (ctx->concurrent && !ctx->timing) return compute_concurrent(ctx, nullptr, false);
        return pairs_impl(ctx);
    });
    if (st == STITCH_OK) ctx->computed = true;
    return st;
}

stitch_status stitch_compute_translations_async(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "compute before load");
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    st = run_graphed(ctx, 1ull << 60, [&]() {
        if (ctx->concurrent && (!ctx->timing || ctx->timing == 3)) return compute_concurrent(ctx);
        stitch_status s2 = forward_impl(ctx, 0, ctx->L.nlocal);
        if (s2 != STITCH_OK) return s2;
        if (ctx->timing) CK(cudaEventRecord(ctx->ev[1], ctx->stream), "event");
        return pairs_impl(ctx);
    });
    if (st == STITCH_OK) ctx->computed = true;
    return st;
}

stitch_status stitch_compute_translations_from_host_async(stitch_ctx* ctx, const uint16_t* tiles,
                                                         int32_t first_tile, int32_t count) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!tiles) return fail(ctx, STITCH_ERR_INVALID_ARG, "null tiles pointer");
    if (first_tile > ctx->L.h_begin || first_tile + (int64_t)count < ctx->L.t_end || first_tile < 0)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range does not cover [halo_begin, tile_end)");
    const uint16_t* src = tiles + (size_t)(ctx->L.h_begin - first_tile) * ctx->H * ctx->W;
    cudaPointerAttributes pa;
    const bool pinned = cudaPointerGetAttributes(&pa, tiles) == cudaSuccess &&
                        pa.type == cudaMemoryTypeHost;
    cudaGetLastError();   // clear a pointer-query error on pageable memory
    if (!ctx->concurrent || ctx->timing || !pinned) {   // no pipelining: load, then the step
        stitch_status st = stitch_load_tiles(ctx, tiles, first_tile, count, 0);
        if (st != STITCH_OK) return st;
        return stitch_compute_translations_async(ctx);
    }
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    ctx->loaded = true;
    // one captured graph per host buffer address (the copies' source is baked into it)
    const uint64_t key = (4ull << 60) ^ (uint64_t)reinterpret_cast<uintptr_t>(src);
    st = run_graphed(ctx, key, [&]() { return compute_concurrent(ctx, src); });
    if (st == STITCH_OK) ctx->computed = true;
    return st;
}

stitch_status stitch_spectra_range(stitch_ctx* ctx, int32_t first_tile, int32_t count,
                                   void** dev_ptr, size_t* bytes) {
    if (!ctx || !dev_ptr || !bytes) return STITCH_ERR_INVALID_ARG;
    if (count < 0 || first_tile < ctx->L.h_begin || first_tile + (int64_t)count > ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range not resident");
    const size_t per =
        (size_t)ctx->H * ctx->ops->WP * (ctx->prec ? sizeof(double2) : sizeof(uint32_t));
    *dev_ptr = reinterpret_cast<char*>(ctx->spec) + (size_t)(first_tile - ctx->L.h_begin) * per;
    *bytes = (size_t)count * per;
    return STITCH_OK;
}

static cudaError_t collect_timings(stitch_ctx* ctx) {
    cudaError_t e = cudaSuccess;
    if (ctx->timing == 3) {
        ctx->tl_ms.assign(2 * ctx->tl.size(), 0.f);
        for (size_t i = 0; i < ctx->tl.size(); ++i) {
            if ((e = cudaEventElapsedTime(&ctx->tl_ms[2 * i], ctx->tl_origin, ctx->tl[i].a)) !=
                    cudaSuccess ||
                (e = cudaEventElapsedTime(&ctx->tl_ms[2 * i + 1], ctx->tl_origin, ctx->tl[i].b)) !=
                    cudaSuccess)
                return e;
        }
        return cudaSuccess;
    }
    if (ctx->timing) {
        for (int i = 0; i < 3; ++i)
            if ((e = cudaEventElapsedTime(&ctx->ms[i], ctx->ev[i], ctx->ev[i + 1])) != cudaSuccess)
                return e;
        if ((e = cudaEventElapsedTime(&ctx->ms[3], ctx->ev[0], ctx->ev[3])) != cudaSuccess) return e;
    }
    if (ctx->timing >= 2) {
        for (int k = 0; k < 6; ++k) { ctx->kms[k] = 0.f; ctx->kcount[k] = 0; }
        for (size_t i = 0; i < ctx->kkind.size(); ++i) {
            float t = 0.f;
            if ((e = cudaEventElapsedTime(&t, ctx->kev[i], ctx->kev[i + 1])) != cudaSuccess) return e;
            const int k = ctx->kkind[i];
            if (k >= 0) { ctx->kms[k] += t; ctx->kcount[k] += 1; }
        }
    }
    return cudaSuccess;
}

stitch_status stitch_get_translations(stitch_ctx* ctx, stitch_pair* west, stitch_pair* north) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!west || !north) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output array");
    if (!ctx->computed) return fail(ctx, STITCH_ERR_STATE, "no computed translations");
    const int64_t np = ctx->L.npairs;
    if (np > 0)
        CK(cudaMemcpyAsync(ctx->res_h.data(), ctx->res, (size_t)np * sizeof(stitch_pair),
                           cudaMemcpyDeviceToHost, ctx->stream),
           "copy results");
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    CK(collect_timings(ctx), "event timing");
    stitch_pair absent;
    std::memset(&absent, 0, sizeof(absent));
    absent.ccf = NAN;
    for (int k = 0; k < 4; ++k) absent.ccf_k[k] = NAN;
    for (int t = ctx->L.t_begin; t < ctx->L.t_end; ++t) {
        west[t] = absent;
        north[t] = absent;
    }
    for (int64_t p = 0; p < np; ++p) {
        stitch_pair* dst = ctx->pair_kind[p] == 0 ? west : north;
        dst[ctx->pair_tile[p]] = ctx->res_h[p];
    }
    return STITCH_OK;
}

stitch_status stitch_compute_translations(stitch_ctx* ctx, stitch_pair* west, stitch_pair* north) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!west || !north) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output array");
    stitch_status s = stitch_compute_translations_async(ctx);
    if (s != STITCH_OK) return s;
    return stitch_get_translations(ctx, west, north);
}

stitch_status stitch_debug_spectrum(stitch_ctx* ctx, int32_t tile, float* host_out) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!host_out) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output");
    if (tile < ctx->L.h_begin || tile >= ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile not resident");
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "spectrum before load");
    if (ctx->prec) return fail(ctx, STITCH_ERR_STATE, "fp64 context: use stitch_debug_spectrum_f64");
    // The resident store keeps Q15 unit phasors; recompute the complex spectrum of this tile
    // with the same K1 + K2 kernels into the chunk buffer G (slot 0) and copy it out.
    const int lt = tile - ctx->L.h_begin;
    const PlanOps* o = ctx->ops;
    launch_k1_any(ctx, lt, 1, ctx->stream);
    o->k2(ctx->tmG, ctx->G, ctx->spec, lt, 1, ctx->twH, false, 0, ctx->stream);
    CK(cudaGetLastError(), "spectrum launch");
    CK(cudaMemcpy2DAsync(host_out, ctx->ops->WC * sizeof(float2), ctx->G,
                         ctx->ops->WP * sizeof(float2), ctx->ops->WC * sizeof(float2), ctx->H,
                         cudaMemcpyDeviceToHost, ctx->stream),
       "copy spectrum");
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    return STITCH_OK;
}

stitch_status stitch_debug_spectrum_f64(stitch_ctx* ctx, int32_t tile, double* host_out) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!host_out) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output");
    if (!ctx->prec) return fail(ctx, STITCH_ERR_STATE, "fp32 context: use stitch_debug_spectrum");
    if (tile < ctx->L.h_begin || tile >= ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile not resident");
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "spectrum before load");
    // the resident store keeps unit phasors: recompute this tile's complex spectrum with the
    // same D1 + D2 kernels into chunk slot 0 of Gd (D2 writing complex values in place)
    const int lt = tile - ctx->L.h_begin;
    const PlanOps* o = ctx->ops;
    o->d1(ctx->raw, ctx->Gd, lt, 1, ctx->twMd, ctx->twWd, ctx->stream);
    o->d2(ctx->Gd, ctx->Ud, lt, 1, ctx->twHd, false, ctx->stream);
    CK(cudaGetLastError(), "spectrum launch");
    CK(cudaMemcpy2DAsync(host_out, ctx->ops->WC * sizeof(double2), ctx->Gd,
                         ctx->ops->WP * sizeof(double2), ctx->ops->WC * sizeof(double2), ctx->H,
                         cudaMemcpyDeviceToHost, ctx->stream),
       "copy spectrum");
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    return STITCH_OK;
}

stitch_status stitch_synchronize(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    if (ctx->computed) CK(collect_timings(ctx), "event timing");
    return STITCH_OK;
}

stitch_status stitch_kernel_timings(stitch_ctx* ctx, float* ms6, int64_t* launches6) {
    if (!ctx || !ms6 || !launches6) return STITCH_ERR_INVALID_ARG;
    for (int k = 0; k < 6; ++k) {
        ms6[k] = ctx->kms[k];
        launches6[k] = ctx->kcount[k];
    }
    return STITCH_OK;
}

stitch_status stitch_last_counts(stitch_ctx* ctx, int64_t* launches, int64_t* forward_ffts,
                                 int64_t* pairs) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (launches) *launches = ctx->launches;
    if (forward_ffts) *forward_ffts = ctx->L.nlocal;
    if (pairs) *pairs = ctx->L.npairs;
    return STITCH_OK;
}

stitch_status stitch_last_timings(stitch_ctx* ctx, float* ms4) {
    if (!ctx || !ms4) return STITCH_ERR_INVALID_ARG;
    for (int i = 0; i < 4; ++i) ms4[i] = ctx->ms[i];
    return STITCH_OK;
}

stitch_status stitch_set_timing(stitch_ctx* ctx, int enabled) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (enabled < 0 || enabled > 3) return fail(ctx, STITCH_ERR_INVALID_ARG, "timing mode 0..3");
    ctx->timing = enabled;
    return STITCH_OK;
}

stitch_status stitch_timeline(stitch_ctx* ctx, int32_t* kernel, int32_t* stream, float* start_ms,
                              float* end_ms, int64_t capacity, int64_t* count) {
    if (!ctx || !count) return STITCH_ERR_INVALID_ARG;
    *count = (int64_t)ctx->tl.size();
    if (ctx->tl_ms.size() != 2 * ctx->tl.size())
        return fail(ctx, STITCH_ERR_STATE, "no collected timeline (timing 3, then synchronize)");
    for (int64_t i = 0; i < *count && i < capacity; ++i) {
        if (kernel) kernel[i] = ctx->tl[i].kid;
        if (stream) stream[i] = ctx->tl[i].stream;
        if (start_ms) start_ms[i] = ctx->tl_ms[2 * i];
        if (end_ms) end_ms[i] = ctx->tl_ms[2 * i + 1];
    }
    return STITCH_OK;
}

const char* stitch_last_error(stitch_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

}  // extern "C"
