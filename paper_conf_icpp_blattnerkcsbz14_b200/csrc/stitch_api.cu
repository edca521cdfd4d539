// stitch_api.cu — host side of the C ABI declared in include/stitch.h.
//
// Owns the device memory plan, the step schedule and the copy-in / copy-out:
//   * plan table: the compiled FFT plans per tile size (radices, CTA shapes);
//   * layout: raw pixels and Q15 phasor spectra by SLOT (slot = local tile in the resident
//     mode; a recycled pool slot in the bounded mode), the forward-chunk G
//     and pair-chunk Q intermediates (0.38 / 0.47 GB at the default 64 / 160 chunks: they
//     round-trip HBM), the pair list (Fig. 4), argmax keys, CCF moments, results;
//   * schedule: a static list of forward chunks (K1 + K2, an H2D copy first when the tiles come
//     from the host) and pair chunks (K3 + K4, then K5), decided at stitch_init and enqueued on
//     internal streams (forward, pairs, CCF, H2D) joined by events, captured once into a CUDA
//     graph and replayed on the caller's stream.  In the bounded mode the list interleaves the
//     two kinds so that slots are recycled by reference count (the paper's pool);
//   * multi-rank: an optional in-library NCCL halo exchange (libnccl.so.2 loaded at run time) on
//     its own stream, overlapped with the interior pairs.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>   // types only: the functions are resolved with dlsym (no link-time NCCL)
#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: a no-op unless a tool (ncu / nsys) attaches

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <deque>
#include <map>
#include <mutex>
#include <new>
#include <set>
#include <string>
#include <type_traits>
#include <vector>

#include "../../include/stitch.h"
#include "pciam_kernels.cuh"
#include "pciam_fp64.cuh"

using namespace stitch;

namespace {

// ------------------------------------------------------------ plan table ---
// Compiled tile-size plans (the row transform is the W/2-point complex FFT of a real row).
//            W     H     row radices          column radices      rowL rowT colP colT rowPad colPad
using P1392 = Plan<1392, 1040, Radix<696, 29, 24>, Radix<1040, 40, 26>, 4, 128, 8, 208, 0, 1>;
using P256 = Plan<256, 192, Radix<128, 16, 8>, Radix<192, 16, 12>, 8, 128, 8, 128, 1, 1>;
using P48 = Plan<48, 40, Radix<24, 24>, Radix<40, 40>, 8, 32, 8, 32, 0, 0>;
using P58 = Plan<58, 26, Radix<29, 29>, Radix<26, 26>, 2, 32, 8, 32, 0, 0>;

// Tile rows per band of the resident pair order (a tile's spectrum and
// pixels are reused by its <= 4 pairs while still in L2; bands of 1-8 measured, 3-4 best).
constexpr int PAIR_BAND = 4;

struct PlanOps {
    int W, H, M, WC, WP, HP, HP64, col_p;
    int row_r0, row_r1, col_r0, col_r1;   // stage radices (r1 = 1: single stage)
    cudaError_t (*setup)(int* grid_k1, int* grid_k4);
    void (*k1)(const uint16_t*, float2*, int, int, const int32_t*, const float2*, const float2*,
               int, cudaStream_t);
    void (*k2)(const float2*, float2*, uint32_t*, int, int, const int32_t*, const float2*, bool,
               int, cudaStream_t);
    void (*k3)(const uint32_t*, float2*, const PairIdx*, int, int, const float2*, cudaStream_t);
    void (*k4)(const float2*, unsigned long long*, int, int, const float2*, const float2*, int,
               cudaStream_t);
    void (*k4s)(const float2*, float*, float, const float2*, const float2*, int, cudaStream_t);
    void (*k5)(const uint16_t*, const PairIdx*, const unsigned long long*, unsigned long long*, int,
               int, cudaStream_t);
    // fp64 path (f2, pciam_fp64.cuh)
    int nblk64;
    double q_scale;   // the scale K3 applies to Q (carried to the reported peak height)
    cudaError_t (*d_setup)();
    void (*d1)(const uint16_t*, double2*, int, int, const double2*, const double2*, cudaStream_t);
    void (*d2)(const double2*, int2*, double2*, int, int, const double2*, bool, cudaStream_t);
    void (*d3)(const int2*, double2*, const PairIdx*, int, int, const double2*, cudaStream_t);
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

// K4w runs the prime-factor (Good-Thomas) row transform where the two radices are coprime
// (696 = 29 x 24), Stockham with stage-2 twiddles otherwise (128 = 16 x 8).
template <class PL>
constexpr bool k4_pfa_ok() {
    if constexpr (RowWarp<PL>::OK)
        return RowWarp<PL>::RI::STAGES == 2 && WarpFftPfa<typename PL::Row, 1>::OK &&
               RowWarp<PL>::PAD == 0;
    else
        return false;
}

#define CKE(x)                                     \
    do {                                           \
        cudaError_t e_ = (x);                      \
        if (e_ != cudaSuccess) return e_;          \
    } while (0)

template <class PL>
cudaError_t plan_setup(int* grid_k1, int* grid_k4) {
    *grid_k1 = *grid_k4 = 0;
    int dev = 0, sms = 0, nb = 0;
    CKE(cudaGetDevice(&dev));
    CKE(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    CKE(max_smem(k5_ccf_moments<PL::W, PL::H>, k5_smem_bytes(PL::W)));
    CKE(max_smem(k2t_fwd_cols<PL, true>, PL::COL_SMEM_K2));
    CKE(max_smem(k2t_fwd_cols<PL, false>, PL::COL_SMEM));
    CKE(max_smem(k3t_pair_cols<PL>, PL::COL_SMEM));
    if constexpr (RowWarp<PL>::OK) {
        using RW = RowWarp<PL>;
        constexpr bool PFA = k4_pfa_ok<PL>();
        CKE(max_smem(k1w_fwd_rows<PL>, RW::SMEM_K1));
        CKE(max_smem(k4w_pair_rows<PL, PFA>, RW::template SMEM_K4<PFA>));
        CKE(max_smem(k4w_pair_rows<PL, PFA, true>, RW::template SMEM_K4<PFA>));
        CKE(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k1w_fwd_rows<PL>, 32 * ROWW_WARPS,
                                                          RW::SMEM_K1));
        *grid_k1 = nb * sms;
        CKE(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k4w_pair_rows<PL, PFA>,
                                                          32 * ROWW_WARPS,
                                                          RW::template SMEM_K4<PFA>));
        *grid_k4 = nb * sms;
    } else {
        CKE(max_smem(k1_fwd_rows<PL>, PL::ROW_SMEM));
        CKE(max_smem(k4_pair_rows<PL>, PL::ROW_SMEM));
        CKE(max_smem(k4_pair_rows<PL, true>, PL::ROW_SMEM));
    }
    return cudaSuccess;
}

// K1: warp-per-row persistent kernel (K1w) where the plan's row transform is a two-stage warp
// FFT; one CTA per row block otherwise (the small test plans).
template <class PL>
void launch_k1(const uint16_t* raw, float2* G, int t0, int nt, const int32_t* fslot,
               const float2* tw2, const float2* twW, int grid, cudaStream_t s) {
    if constexpr (RowWarp<PL>::OK) {
        const int need = (nt * PL::H + ROWW_WARPS - 1) / ROWW_WARPS;
        k1w_fwd_rows<PL><<<grid < need ? grid : need, 32 * ROWW_WARPS, RowWarp<PL>::SMEM_K1, s>>>(
            raw, G, t0, nt, fslot, tw2, twW);
    } else {
        k1_fwd_rows<PL><<<dim3(PL::H / PL::ROW_L, nt), PL::ROW_T, PL::ROW_SMEM, s>>>(
            raw, G, t0, fslot, tw2, twW);
    }
}
template <class PL>
void launch_k2(const float2* G, float2* out, uint32_t* spec, int t0, int nt, const int32_t* fslot,
               const float2* tw2, bool phase_out, int ahead, cudaStream_t s) {
    const dim3 grid(PL::WP / PL::COL_P, nt);
    if (phase_out)
        k2t_fwd_cols<PL, true><<<grid, PL::COL_T, PL::COL_SMEM_K2, s>>>(G, out, spec, t0, fslot,
                                                                        tw2, ahead);
    else
        k2t_fwd_cols<PL, false><<<grid, PL::COL_T, PL::COL_SMEM, s>>>(G, out, spec, t0, fslot, tw2,
                                                                      0);
}
template <class PL>
void launch_k3(const uint32_t* spec, float2* Q, const PairIdx* pairs, int p0, int np,
               const float2* tw2, cudaStream_t s) {
    k3t_pair_cols<PL><<<dim3(PL::WP / PL::COL_P, np), PL::COL_T, PL::COL_SMEM, s>>>(spec, Q, pairs,
                                                                                   p0, tw2);
}
template <class PL>
void launch_k4(const float2* Q, unsigned long long* keys, int p0, int np, const float2* tw2,
               const float2* twW, int grid, cudaStream_t s) {
    if constexpr (RowWarp<PL>::OK) {
        const int need = (np * PL::H + ROWW_WARPS - 1) / ROWW_WARPS;
        k4w_pair_rows<PL, k4_pfa_ok<PL>()><<<grid < need ? grid : need, 32 * ROWW_WARPS,
                                             RowWarp<PL>::template SMEM_K4<k4_pfa_ok<PL>()>, s>>>(
            Q, keys, p0, np, tw2, twW);
    } else {
        k4_pair_rows<PL><<<dim3(PL::H / PL::ROW_L, np), PL::ROW_T, PL::ROW_SMEM, s>>>(Q, keys, p0,
                                                                                      tw2, twW);
    }
}
template <class PL>
void launch_k4s(const float2* Q, float* surf, float scale, const float2* tw2, const float2* twW,
                int grid, cudaStream_t s) {
    if constexpr (RowWarp<PL>::OK) {
        const int need = (PL::H + ROWW_WARPS - 1) / ROWW_WARPS;
        k4w_pair_rows<PL, k4_pfa_ok<PL>(), true><<<grid < need ? grid : need, 32 * ROWW_WARPS,
                                                   RowWarp<PL>::template SMEM_K4<k4_pfa_ok<PL>()>, s>>>(
            Q, nullptr, 0, 1, tw2, twW, surf, scale);
    } else {
        k4_pair_rows<PL, true><<<dim3(PL::H / PL::ROW_L, 1), PL::ROW_T, PL::ROW_SMEM, s>>>(
            Q, nullptr, 0, tw2, twW, surf, scale);
    }
}
template <class PL>
void launch_k5(const uint16_t* raw, const PairIdx* pairs, const unsigned long long* keys,
               unsigned long long* mom, int p0, int np, cudaStream_t s) {
    k5_ccf_moments<PL::W, PL::H><<<dim3(k5_grid_x(PL::H), np), CCF_T, k5_smem_bytes(PL::W), s>>>(
        raw, pairs, keys, mom, p0);
}

// ---- fp64 path launchers (f2)
template <class PL>
cudaError_t d_setup() {
    using P64 = Plan64<PL>;
    CKE(max_smem(d1_fwd_rows<PL>, P64::ROW_SMEM));
    if constexpr (D1w<PL>::OK) CKE(max_smem(d1w_fwd_rows<PL>, D1w<PL>::SMEM));
    CKE(max_smem(d4_pair_rows<PL>, P64::D4_SMEM));
    if constexpr (D4w<PL>::OK) CKE(max_smem(d4w_pair_rows<PL>, D4w<PL>::SMEM));
    CKE(max_smem(d2_fwd_cols<PL, true>, P64::D2_SMEM));
    CKE(max_smem(d2_fwd_cols<PL, false>, P64::D2_SMEM));
    if constexpr (D3P<PL>::F::OK) {
        CKE(max_smem(d3p_pair_cols<PL>, D3P<PL>::SMEM));
        CKE(max_smem(d2p_fwd_cols<PL, true>, D2P<PL>::SMEM));
        CKE(max_smem(d2p_fwd_cols<PL, false>, D2P<PL>::SMEM));
    }
    return max_smem(d3_pair_cols<PL>, P64::D3_SMEM);
}
template <class PL>
void launch_d1(const uint16_t* raw, double2* G, int t0, int nt, const double2* tw2,
               const double2* twW, cudaStream_t s) {
    using P64 = Plan64<PL>;
    if constexpr (D1w<PL>::OK) {   // warp per row, one CTA per SM
        static int sms = 0;
        if (!sms) {
            int dev = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        }
        const int need = (int)(((long long)nt * PL::H + D1W_WARPS - 1) / D1W_WARPS);
        d1w_fwd_rows<PL><<<need < sms ? need : sms, 32 * D1W_WARPS, D1w<PL>::SMEM, s>>>(
            raw, G, t0, nt, twW);
        return;
    }
    d1_fwd_rows<PL><<<dim3(P64::NBLK, nt), P64::ROW_T, P64::ROW_SMEM, s>>>(raw, G, t0, tw2, twW);
}
template <class PL>
void launch_d2(const double2* G, int2* U, double2* out, int t0, int nt, const double2* tw2,
               bool unit_out, cudaStream_t s) {
    using P64 = Plan64<PL>;
    const dim3 grid(PL::WP / P64::COL_P, nt);
    if constexpr (D2P<PL>::F::OK) {   // three-factor prime-factor columns (1040 = 16 x 5 x 13)
        using S2 = D2P<PL>;
        if (unit_out)
            d2p_fwd_cols<PL, true><<<grid, S2::T, S2::SMEM, s>>>(G, U, out, t0);
        else
            d2p_fwd_cols<PL, false><<<grid, S2::T, S2::SMEM, s>>>(G, U, out, t0);
        return;
    }
    if (unit_out)
        d2_fwd_cols<PL, true><<<grid, P64::COL_T, P64::D2_SMEM, s>>>(G, U, out, t0, tw2);
    else
        d2_fwd_cols<PL, false><<<grid, P64::COL_T, P64::D2_SMEM, s>>>(G, U, out, t0, tw2);
}
template <class PL>
void launch_d3(const int2* U, double2* Q, const PairIdx* pairs, int p0, int np,
               const double2* tw2, cudaStream_t s) {
    using P64 = Plan64<PL>;
    if constexpr (D3P<PL>::F::OK) {   // three-factor prime-factor columns (1040 = 16 x 5 x 13)
        using S3 = D3P<PL>;
        d3p_pair_cols<PL><<<dim3(PL::WP / S3::P, np), S3::T, S3::SMEM, s>>>(U, Q, pairs, p0);
        return;
    }
    d3_pair_cols<PL><<<dim3(PL::WP / P64::COL_P3, np), P64::COL_T3, P64::D3_SMEM, s>>>(U, Q, pairs,
                                                                                      p0, tw2);
}
template <class PL>
void launch_d4(const double2* Q, double* pv, uint32_t* pi, int p0, int np, const double2* tw2,
               const double2* twW, cudaStream_t s) {
    using P64 = Plan64<PL>;
    if constexpr (D4w<PL>::OK) {   // warp per row, one CTA per SM
        static int sms = 0;
        if (!sms) {
            int dev = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        }
        const int need = (int)(((long long)np * P64::NBLK + D4W_WARPS - 1) / D4W_WARPS);
        d4w_pair_rows<PL><<<need < sms ? need : sms, 32 * D4W_WARPS, D4w<PL>::SMEM, s>>>(
            Q, pv, pi, p0, np, twW);
        return;
    }
    d4_pair_rows<PL><<<dim3(P64::NBLK, np), P64::ROW_T, P64::D4_SMEM, s>>>(Q, pv, pi, p0, tw2,
                                                                            twW);
}

template <class PL>
PlanOps make_ops() {
    PlanOps o;
    o.W = PL::W; o.H = PL::H; o.M = PL::M; o.WC = PL::WC; o.WP = PL::WP; o.HP = PL::HP; o.HP64 = Plan64<PL>::HP64;
    o.col_p = PL::COL_P;
    o.q_scale = PL::Q_SCALE;
    o.row_r0 = PL::RI::R0; o.row_r1 = PL::RI::R1; o.col_r0 = PL::CI::R0; o.col_r1 = PL::CI::R1;
    o.setup = plan_setup<PL>;
    o.k1 = launch_k1<PL>; o.k2 = launch_k2<PL>; o.k3 = launch_k3<PL>; o.k4 = launch_k4<PL>;
    o.k4s = launch_k4s<PL>; o.k5 = launch_k5<PL>;
    o.nblk64 = Plan64<PL>::NBLK;
    o.d_setup = d_setup<PL>;
    o.d1 = launch_d1<PL>; o.d2 = launch_d2<PL>; o.d3 = launch_d3<PL>; o.d4 = launch_d4<PL>;
    return o;
}

const PlanOps* find_plan(int W, int H) {
    static const PlanOps ops[] = {make_ops<P1392>(), make_ops<P256>(), make_ops<P48>(),
                                  make_ops<P58>()};
    for (const auto& o : ops)
        if (o.W == W && o.H == H) return &o;
    return nullptr;
}

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

// twiddle tables: row stage-2 [r0*(r1-1)], column stage-2 [c0*(c1-1)], R2C/C2R w_W [W]
// (slot counts rounded up to even, so every table starts 16-byte aligned for bulk copies)
size_t tw_row(const PlanOps* o) { return ((size_t)o->row_r0 * (o->row_r1 - 1) + 1) & ~(size_t)1; }
size_t tw_col(const PlanOps* o) { return ((size_t)o->col_r0 * (o->col_r1 - 1) + 1) & ~(size_t)1; }
size_t tw_count(const PlanOps* o) { return tw_row(o) + tw_col(o) + o->W + 2; }

// ------------------------------------------------------------- NCCL ----
// Loaded at run time (the one torch ships is already in the process when torch is; else the
// system's), so the library has no link-time NCCL dependency and single-GPU use needs none.
struct NcclApi {
    bool ok = false;
    std::string err;
    ncclResult_t (*get_unique_id)(ncclUniqueId*) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    ncclResult_t (*send)(const void*, size_t, ncclDataType_t, int, ncclComm_t,
                         cudaStream_t) = nullptr;
    ncclResult_t (*recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*group_start)() = nullptr;
    ncclResult_t (*group_end)() = nullptr;
    const char* (*error_string)(ncclResult_t) = nullptr;
};

const NcclApi& nccl() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char* d = dlerror();
            api.err = std::string("cannot load libnccl.so.2: ") + (d ? d : "?");
            return;
        }
        auto sym = [&](const char* n) { return dlsym(h, n); };
        api.get_unique_id = reinterpret_cast<decltype(api.get_unique_id)>(sym("ncclGetUniqueId"));
        api.comm_init_rank = reinterpret_cast<decltype(api.comm_init_rank)>(sym("ncclCommInitRank"));
        api.comm_destroy = reinterpret_cast<decltype(api.comm_destroy)>(sym("ncclCommDestroy"));
        api.send = reinterpret_cast<decltype(api.send)>(sym("ncclSend"));
        api.recv = reinterpret_cast<decltype(api.recv)>(sym("ncclRecv"));
        api.group_start = reinterpret_cast<decltype(api.group_start)>(sym("ncclGroupStart"));
        api.group_end = reinterpret_cast<decltype(api.group_end)>(sym("ncclGroupEnd"));
        api.error_string = reinterpret_cast<decltype(api.error_string)>(sym("ncclGetErrorString"));
        api.ok = api.get_unique_id && api.comm_init_rank && api.comm_destroy && api.send &&
                 api.recv && api.group_start && api.group_end && api.error_string;
        if (!api.ok) api.err = "libnccl.so.2 lacks a required symbol";
    });
    return api;
}

// ------------------------------------------------------------- layout ----
struct Layout {
    int h_begin, t_begin, t_end, nlocal;
    int nslots;          // tile slots (raw + spectrum): nlocal, or the pool size (bounded mode)
    int64_t npairs;
    int chunk_pairs, chunk_tiles;
    int prec;            // 0 fp32, 1 fp64 (f2)
    int pool;            // bounded mode (row f1)
    int world, rank;
    bool exchange;       // in-library NCCL halo exchange
    size_t spec_tile_bytes;   // one slot's spectrum
    size_t off_raw, off_spec, off_g, off_q, off_pairs, off_keys, off_mom, off_res, off_tw,
        off_part, off_fslot, total;
};

// Balanced row-band partition: rank k of R owns [k nt/R, (k+1) nt/R).
void band_of(int64_t nt, int rank, int world, int* b, int* e) {
    *b = (int)(nt * rank / world);
    *e = (int)(nt * (rank + 1) / world);
}

// Every halo lies in the previous rank's band (all bands but the last hold >= one tile row).
bool exchange_feasible(int64_t nt, int m, int world) {
    if (world < 2) return false;
    for (int k = 0; k + 1 < world; ++k) {
        int b, e;
        band_of(nt, k, world, &b, &e);
        if (e - b < m) return false;
    }
    return true;
}

stitch_status make_layout(const stitch_config* c, const PlanOps* ops, Layout* L) {
    const int n = c->grid_rows, m = c->grid_cols;
    const int64_t nt = (int64_t)n * m;
    L->world = c->world_size > 1 ? c->world_size : 1;
    L->rank = L->world > 1 ? c->rank : 0;
    if (L->world > 1 && (c->rank < 0 || c->rank >= c->world_size || nt < c->world_size))
        return STITCH_ERR_INVALID_ARG;
    L->t_begin = c->tile_begin;
    L->t_end = c->tile_end ? c->tile_end : (int)nt;
    if (L->world > 1 && c->tile_begin == 0 && c->tile_end == 0)
        band_of(nt, L->rank, L->world, &L->t_begin, &L->t_end);
    if (L->t_begin < 0 || L->t_end > nt || L->t_begin >= L->t_end) return STITCH_ERR_INVALID_ARG;
    L->exchange = false;
    if (c->nccl_id) {
        // the library owns the partition when it owns the exchange
        if (L->world < 2 || c->tile_begin != 0 || c->tile_end != 0) return STITCH_ERR_INVALID_ARG;
        if (c->precision != 0) return STITCH_ERR_UNSUPPORTED;   // the exchange moves Q15 spectra
        L->exchange = exchange_feasible(nt, m, L->world);
    }
    L->h_begin = L->t_begin - m > 0 ? L->t_begin - m : 0;
    L->nlocal = L->t_end - L->h_begin;
    int64_t np = 0;
    for (int t = L->t_begin; t < L->t_end; ++t) np += (t % m >= 1) + (t / m >= 1);
    L->npairs = np;
    if (c->precision != 0 && c->precision != 1) return STITCH_ERR_INVALID_ARG;
    L->prec = c->precision;
    if (c->pool_tiles < 0) return STITCH_ERR_INVALID_ARG;
    L->pool = c->pool_tiles > 0;
    if (L->pool && (L->prec || c->nccl_id)) return STITCH_ERR_UNSUPPORTED;
    L->nslots = L->pool ? std::min(c->pool_tiles, L->nlocal) : L->nlocal;
    // default chunks (both precisions): 160 pairs / 64 tiles -- the intermediates round-trip
    // HBM either way, and larger launches lose less to their tail wave (fp64 sweep: 8/8 75.7 ms,
    // 32/16 68.5 ms, 160/64 67.8 ms per 42x59 step, DESIGN.md variant 40)
    // bounded mode: chunks of about an eighth of the pool (and ~3 pairs per tile), so slots
    // turn over while the H2D stream runs ahead (pool 160 at 42x59: 20 / 60 -> 132 ms end to
    // end, PCIe-bound like the resident mode; 40 / 160: 154 ms)
    const int ct_pool = std::max(1, std::min(64, L->nslots / 8));
    L->chunk_tiles = c->chunk_tiles > 0 ? c->chunk_tiles : (L->pool ? ct_pool : 64);
    L->chunk_pairs = c->chunk_pairs > 0 ? c->chunk_pairs
                                        : (L->pool ? std::min(160, 3 * L->chunk_tiles) : 160);
    if (L->chunk_pairs > 65535 || L->chunk_tiles > 65535) return STITCH_ERR_INVALID_ARG;
    const size_t H = ops->H, W = ops->W, WP = ops->WP;
    // spectrum by slot: u32 Q15 unit phasor [WP][HP] (fp32) or double2 unit phasor [H][WP] (fp64)
    L->spec_tile_bytes = L->prec ? (size_t)ops->HP64 * WP * sizeof(int2)
                                 : (size_t)ops->HP * WP * sizeof(uint32_t);
    const size_t cplx = L->prec ? sizeof(double2) : sizeof(float2);
    const size_t np1 = (size_t)(np > 0 ? np : 1);
    size_t o = 0;
    L->off_raw = o;   o += align256((size_t)L->nslots * H * W * sizeof(uint16_t));
    L->off_spec = o;  o += align256((size_t)L->nslots * L->spec_tile_bytes);
    L->off_g = o;     o += align256((size_t)L->chunk_tiles * H * WP * cplx);
    L->off_q = o;     o += align256((size_t)L->chunk_pairs * H * WP * cplx);
    L->off_pairs = o; o += align256(np1 * sizeof(PairIdx));
    L->off_keys = o;  o += align256(np1 * sizeof(unsigned long long));
    L->off_mom = o;   o += align256(np1 * 20 * sizeof(unsigned long long));
    L->off_res = o;   o += align256(np1 * sizeof(stitch_pair));
    L->off_tw = o;    o += align256((size_t)(tw_count(ops)) * cplx);
    L->off_fslot = o; o += align256((size_t)L->nlocal * sizeof(int32_t));
    L->off_part = o;  // fp64 argmax partials: double [pairs][nblk] then u32 [pairs][nblk]
    if (L->prec) o += align256(np1 * ops->nblk64 * (8 + 4));
    L->total = o;
    return STITCH_OK;
}

stitch_status check_config(const stitch_config* c, const PlanOps** ops) {
    if (!c) return STITCH_ERR_INVALID_ARG;
    if (c->grid_rows < 1 || c->grid_cols < 1 || c->tile_width < 2 || c->tile_height < 1)
        return STITCH_ERR_INVALID_ARG;
    if ((int64_t)c->grid_rows * c->grid_cols > (1 << 30)) return STITCH_ERR_INVALID_ARG;
    if (c->flags & ~(uint32_t)(STITCH_FLAG_NO_GRAPH | STITCH_FLAG_SERIAL))
        return STITCH_ERR_INVALID_ARG;
    *ops = find_plan(c->tile_width, c->tile_height);
    if (!*ops) return STITCH_ERR_UNSUPPORTED;
    return STITCH_OK;
}

// Makes `dev` current for the lifetime of the guard and restores the caller's device.
struct DevGuard {
    int old = -1;
    bool changed = false;
    cudaError_t err = cudaSuccess;
    explicit DevGuard(int dev) {
        if ((err = cudaGetDevice(&old)) != cudaSuccess) return;
        if (old != dev) {
            err = cudaSetDevice(dev);
            changed = err == cudaSuccess;
        }
    }
    ~DevGuard() {
        if (changed) cudaSetDevice(old);
    }
};

// ----------------------------------------------------------- schedule ----
struct FwdChunk {
    int t0, nt;          // local tiles [t0, t0 + nt)
    int wait_pair = -1;  // bounded mode: pair chunk whose K5 frees the last slot this chunk takes
    int wait_fwd = -1;   // bounded mode: forward chunk whose K1 last read a slot this chunk takes
};
struct PairChunk {
    int64_t p0;
    int np;
    int need;            // forward chunk (index in the step list) completing its tiles; -1: none
    bool boundary;       // reads a halo spectrum received from rank-1
};
struct Op {
    enum Kind : int8_t { FWD, PAIR, EXCH } kind;
    int idx;
};

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
    uint32_t* spec;                   // Q15 phasor spectra by slot [nslots][H][WP]
    float2 *G, *Q, *twM, *twH, *twW;  // chunk intermediates, twiddles
    int32_t* fslot;                   // slot of each local tile
    int prec = 0;                     // 1: fp64 path (f2): the buffers below are used instead
    double2 *Gd = nullptr, *Qd = nullptr;
    int2* Ud = nullptr;               // resident Q31 unit phasors (fp64 path)
    double2 *twMd = nullptr, *twHd = nullptr, *twWd = nullptr;
    double* part_v = nullptr;         // fp64 argmax partials [pairs][nblk64]
    uint32_t* part_i = nullptr;
    int grid_k1 = 0, grid_k4 = 0;     // persistent grids of the warp row kernels (0: CTA kernels)
    int col_ahead = 0;                // K2 L2 prefetch distance in CTAs (one wave)
    PairIdx* pairs;
    unsigned long long *keys, *mom;
    stitch_pair* res;
    std::vector<PairIdx> pairs_h;
    std::vector<int32_t> pair_tile;   // global tile index (B) of each pair
    std::vector<int8_t> pair_kind;    // 0 west, 1 north
    std::vector<int32_t> fslot_h;
    std::vector<stitch_pair> res_h;
    // static schedule (stitch_init)
    std::vector<FwdChunk> fwd;
    std::vector<PairChunk> pch;
    std::vector<Op> ops_step;         // the whole step in enqueue order
    int64_t n_interior = 0;           // pairs [0, n_interior) need no halo spectrum
    int c_boundary = 0;               // first pair chunk of the boundary pairs
    // NCCL halo exchange (L.exchange)
    ncclComm_t comm = nullptr;
    int send_lt = 0, send_cnt = 0, recv_lt = 0, recv_cnt = 0;   // local tile ranges
    bool loaded = false, computed = false;
    int64_t launches = 0;
    bool use_graph = true, concurrent = true;
    cudaStream_t cap_stream = nullptr;
    struct GraphRec {
        cudaGraphExec_t exec = nullptr;
        cudaGraph_t graph = nullptr;
        int64_t launches = 0;
        const char* src = nullptr;    // host source baked into the H2D nodes (nullptr: none)
        std::vector<cudaGraphNode_t> h2d;
        std::vector<cudaMemcpy3DParms> h2d_p;
    };
    std::map<uint64_t, GraphRec> graphs;
    cudaStream_t s_fwd = nullptr, s_pair = nullptr, s_ccf = nullptr, s_h2d = nullptr,
                 s_comm = nullptr;
    std::vector<cudaEvent_t> ev_h2d, ev_fwd, ev_k4, ev_k5;
    cudaEvent_t ev_halo = nullptr, ev_fork = nullptr;
    cudaEvent_t ev_join[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
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

// Per-launch event (timing mode 2): kid 0..5 = K1..K6 (-1: not a kernel).
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

static stitch_status nccl_fail(stitch_ctx* ctx, ncclResult_t r, const char* where) {
    const NcclApi& api = nccl();
    return fail(ctx, STITCH_ERR_NCCL,
                std::string(where) + ": " + (api.error_string ? api.error_string(r) : "nccl error"));
}

#define CK(call, where)                                          \
    do {                                                         \
        cudaError_t e_ = (call);                                 \
        if (e_ != cudaSuccess) return cuda_fail(ctx, e_, where); \
    } while (0)

// Tracing: every device-touching entry point is an NVTX range named after
// it, so a profiler can scope captures to a call (ncu --nvtx --nvtx-include "stitch_.../").
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

#define GUARD(ctx)                                                          \
    NvtxRange nvtx_(__func__);                                              \
    DevGuard guard_((ctx)->cfg.device);                                     \
    if (guard_.err != cudaSuccess) return cuda_fail(ctx, guard_.err, "set device")

// ------------------------------------------------ schedule construction ----
// Resident mode: forward chunks in tile order; pairs in bands of PAIR_BAND tile rows
// (column-major inside a band), interior pairs first, then the boundary pairs (tile A in the
// halo, which an NCCL exchange may still be delivering); every pair chunk waits for the
// forward chunk that completes its tiles.
static void build_resident(stitch_ctx* ctx) {
    const Layout& L = ctx->L;
    const int m = ctx->m, hb = L.h_begin, tbl = L.t_begin - hb;
    const int ct = L.chunk_tiles, cp = L.chunk_pairs;
    ctx->fslot_h.resize(L.nlocal);
    for (int i = 0; i < L.nlocal; ++i) ctx->fslot_h[i] = i;
    // the step's forward chunks: every local tile, or only the owned ones when the halo's
    // spectra arrive by NCCL
    const int f0 = L.exchange ? tbl : 0;
    std::vector<int> chunk_of(L.nlocal, -1);
    for (int t0 = f0; t0 < L.nlocal; t0 += ct) {
        const int nt = std::min(ct, L.nlocal - t0);
        for (int i = 0; i < nt; ++i) chunk_of[t0 + i] = (int)ctx->fwd.size();
        ctx->fwd.push_back(FwdChunk{t0, nt});
    }
    std::vector<int> order;
    for (int t = L.t_begin; t < L.t_end; ++t) order.push_back(t);
    std::stable_sort(order.begin(), order.end(), [m](int a, int b) {
        const int ra = a / m, rb = b / m, ba = ra / PAIR_BAND, bb = rb / PAIR_BAND;
        if (ba != bb) return ba < bb;
        if (a % m != b % m) return a % m < b % m;
        return ra < rb;
    });
    struct P { int a, b, t; int8_t kind; };
    std::vector<P> inner, bound;
    for (const int t : order) {
        const int r = t / m, c = t % m;
        if (c >= 1) (t - 1 >= L.t_begin ? inner : bound).push_back(P{t - 1 - hb, t - hb, t, 0});
        if (r >= 1) (t - m >= L.t_begin ? inner : bound).push_back(P{t - m - hb, t - hb, t, 1});
    }
    ctx->n_interior = (int64_t)inner.size();
    auto emit = [&](const std::vector<P>& v, bool boundary) {
        for (size_t i = 0; i < v.size(); i += (size_t)cp) {
            PairChunk pc{(int64_t)ctx->pairs_h.size(), (int)std::min(v.size() - i, (size_t)cp), -1,
                         boundary};
            for (size_t j = i; j < i + (size_t)pc.np; ++j) {
                const P& q = v[j];
                ctx->pairs_h.push_back(PairIdx{q.a, q.b});
                ctx->pair_tile.push_back(q.t);
                ctx->pair_kind.push_back(q.kind);
                pc.need = std::max(pc.need, std::max(chunk_of[q.a], chunk_of[q.b]));
            }
            ctx->pch.push_back(pc);
        }
    };
    emit(inner, false);
    ctx->c_boundary = (int)ctx->pch.size();
    emit(bound, true);
    for (int f = 0; f < (int)ctx->fwd.size(); ++f) ctx->ops_step.push_back(Op{Op::FWD, f});
    if (L.exchange) ctx->ops_step.push_back(Op{Op::EXCH, 0});
    for (int c = 0; c < (int)ctx->pch.size(); ++c) ctx->ops_step.push_back(Op{Op::PAIR, c});
}

// Bounded mode (row f1; the paper's pool of reusable buffers with per-tile reference counts,
// P:L1082-1110): tiles are transformed in row-major forward chunks into free slots of a
// fixed pool; each tile's count starts at the number of pairs that read it (<= 4: west, east,
// north, south, Fig. 4) and drops as pair chunks are scheduled; a slot whose count reaches 0
// is free again once that pair chunk's K5 (the last reader of its pixels and, through the
// K3 -> K4 -> K5 chain, of its spectrum) has finished -- the forward chunk that takes it
// next waits for that event.  Pairs are scheduled as soon as both tiles are ready, in chunks
// of up to chunk_pairs, earlier when the pool runs dry.  The simulation runs once, here, so
// the step is a static interleaving of forward and pair chunks (graph-capturable).
static bool build_pooled(stitch_ctx* ctx, std::string* why) {
    const Layout& L = ctx->L;
    const int m = ctx->m, hb = L.h_begin, nl = L.nlocal;
    const int ct = L.chunk_tiles, cp = L.chunk_pairs;
    std::vector<int> refs(nl, 0);
    for (int t = L.t_begin; t < L.t_end; ++t) {
        const int lt = t - hb;
        if (t % m >= 1) { ++refs[lt]; ++refs[lt - 1]; }
        if (t / m >= 1) { ++refs[lt]; ++refs[lt - m]; }
    }
    ctx->fslot_h.assign(nl, -1);
    std::set<int> free_slots;
    for (int s = 0; s < L.nslots; ++s) free_slots.insert(s);
    std::vector<int> tag_pair(L.nslots, -1), tag_fwd(L.nslots, -1);
    struct P { int a, b, t; int8_t kind; };   // local tiles
    std::deque<P> pending;
    int cur_f = -1, next_slot = 0;
    auto release = [&](int lt, int tp, int tf) {
        const int s = ctx->fslot_h[lt];
        tag_pair[s] = tp;
        tag_fwd[s] = tf;
        free_slots.insert(s);
    };
    auto emit_pairs = [&](int k) {
        const int c = (int)ctx->pch.size();
        ctx->pch.push_back(PairChunk{(int64_t)ctx->pairs_h.size(), k, cur_f, false});
        ctx->ops_step.push_back(Op{Op::PAIR, c});
        for (int i = 0; i < k; ++i) {
            const P q = pending.front();
            pending.pop_front();
            ctx->pairs_h.push_back(PairIdx{ctx->fslot_h[q.a], ctx->fslot_h[q.b]});
            ctx->pair_tile.push_back(q.t);
            ctx->pair_kind.push_back(q.kind);
            for (const int lt : {q.a, q.b})
                if (--refs[lt] == 0) release(lt, c, -1);
        }
    };
    for (int t0 = 0; t0 < nl; t0 += ct) {
        const int nt = std::min(ct, nl - t0);
        while ((int)free_slots.size() < nt) {
            if (pending.empty()) {
                *why = "pool_tiles too small for the grid: every slot holds a tile still awaiting a "
                       "pair (need about one tile row + one forward chunk of slots)";
                return false;
            }
            emit_pairs(std::min((int)pending.size(), cp));
        }
        FwdChunk fc{t0, nt};
        for (int i = 0; i < nt; ++i) {
            // next fit around the ring: slots are freed roughly in the order they were taken,
            // so continuing after the last one keeps a chunk's slots in long runs (one H2D copy
            // per run, copy_chunk_in) instead of refilling scattered low slots
            auto it = free_slots.lower_bound(next_slot);
            if (it == free_slots.end()) it = free_slots.begin();
            const int s = *it;
            free_slots.erase(it);
            next_slot = s + 1;
            ctx->fslot_h[t0 + i] = s;
            fc.wait_pair = std::max(fc.wait_pair, tag_pair[s]);
            fc.wait_fwd = std::max(fc.wait_fwd, tag_fwd[s]);
        }
        cur_f = (int)ctx->fwd.size();
        ctx->fwd.push_back(fc);
        ctx->ops_step.push_back(Op{Op::FWD, cur_f});
        for (int lt = t0; lt < t0 + nt; ++lt) {
            const int t = lt + hb;
            if (t >= L.t_begin) {   // pairs with tile B = t become ready (tile A < B is ready)
                if (t % m >= 1) pending.push_back(P{lt - 1, lt, t, 0});
                if (t / m >= 1) pending.push_back(P{lt - m, lt, t, 1});
            }
            if (refs[lt] == 0) release(lt, -1, cur_f);   // read by no pair (e.g. a 1x1 grid)
        }
        while ((int)pending.size() >= cp) emit_pairs(cp);
    }
    while (!pending.empty()) emit_pairs(std::min((int)pending.size(), cp));
    ctx->n_interior = (int64_t)ctx->pairs_h.size();
    ctx->c_boundary = (int)ctx->pch.size();
    return true;
}

// ------------------------------------------------------------ enqueue ----
static bool serial(const stitch_ctx* ctx) {
    return !ctx->concurrent || ctx->timing == 1 || ctx->timing == 2;
}

// Host-to-device copy of a forward chunk's tiles into their slots (runs of consecutive slots
// coalesced into one copy).  src: the caller's buffer, tile 0 = local tile 0.
static stitch_status copy_chunk_in(stitch_ctx* ctx, const FwdChunk& fc, const uint16_t* src,
                                   cudaStream_t s) {
    const size_t tile_px = (size_t)ctx->H * ctx->W;
    for (int i = 0; i < fc.nt;) {
        int j = i + 1;
        while (j < fc.nt && ctx->fslot_h[fc.t0 + j] == ctx->fslot_h[fc.t0 + i] + (j - i)) ++j;
        CK(cudaMemcpyAsync(ctx->raw + (size_t)ctx->fslot_h[fc.t0 + i] * tile_px,
                           src + (size_t)(fc.t0 + i) * tile_px, (size_t)(j - i) * tile_px * 2,
                           cudaMemcpyHostToDevice, s),
           "tile H2D");
        i = j;
    }
    return STITCH_OK;
}

static void launch_fwd(stitch_ctx* ctx, int t0, int nt, cudaStream_t s, int si) {
    const PlanOps* o = ctx->ops;
    if (ctx->prec) {   // fp64 path (f2): D1, D2 (resident tiles: slot = local tile)
        tl_wrap(ctx, s, si, 0, [&] { o->d1(ctx->raw, ctx->Gd, t0, nt, ctx->twMd, ctx->twWd, s); });
        mark(ctx, 0);
        tl_wrap(ctx, s, si, 1, [&] { o->d2(ctx->Gd, ctx->Ud, nullptr, t0, nt, ctx->twHd, true, s); });
        mark(ctx, 1);
        ctx->launches += 2;
        return;
    }
    tl_wrap(ctx, s, si, 0, [&] {
        o->k1(ctx->raw, ctx->G, t0, nt, ctx->fslot, ctx->twM, ctx->twW, ctx->grid_k1, s);
    });
    mark(ctx, 0);
    tl_wrap(ctx, s, si, 1, [&] {
        o->k2(ctx->G, nullptr, ctx->spec, t0, nt, ctx->fslot, ctx->twH, true, ctx->col_ahead, s);
    });
    mark(ctx, 1);
    ctx->launches += 2;
}

// The halo exchange (rank k: send the spectra of its last tile row to k+1, receive its halo
// row from k-1), one NCCL group on stream s.
static stitch_status exchange(stitch_ctx* ctx, cudaStream_t s) {
    const NcclApi& api = nccl();
    const size_t per = ctx->L.spec_tile_bytes;
    ncclResult_t r;
    if ((r = api.group_start()) != ncclSuccess) return nccl_fail(ctx, r, "ncclGroupStart");
    if (ctx->send_cnt > 0 &&
        (r = api.send(ctx->spec + (size_t)ctx->fslot_h[ctx->send_lt] * (per / 4),
                      (size_t)ctx->send_cnt * per, ncclUint8, ctx->L.rank + 1, ctx->comm, s)) !=
            ncclSuccess) {
        api.group_end();
        return nccl_fail(ctx, r, "ncclSend");
    }
    if (ctx->recv_cnt > 0 &&
        (r = api.recv(ctx->spec + (size_t)ctx->fslot_h[ctx->recv_lt] * (per / 4),
                      (size_t)ctx->recv_cnt * per, ncclUint8, ctx->L.rank - 1, ctx->comm, s)) !=
            ncclSuccess) {
        api.group_end();
        return nccl_fail(ctx, r, "ncclRecv");
    }
    if ((r = api.group_end()) != ncclSuccess) return nccl_fail(ctx, r, "ncclGroupEnd");
    return STITCH_OK;
}

// Enqueue a list of forward / exchange / pair ops (the whole step or a part of it) on the
// context's streams.  Concurrent: forward chunks on s_fwd (their H2D on s_h2d), pair chunks'
// K3 + K4 on s_pair and K5 on s_ccf, the exchange on s_comm, joined by events; serial (timing
// modes 1-2, or STITCH_FLAG_SERIAL): everything on the context stream in list order.
// src: host tiles (local tile 0 first) copied per forward chunk, or nullptr (resident).
// [pa, pb): the pairs these ops cover (keys/moments cleared first, K6 over them last).
static stitch_status enqueue_ops(stitch_ctx* ctx, const std::vector<Op>& ops, const uint16_t* src,
                                 bool wait_fwd, int64_t pa, int64_t pb) {
    const PlanOps* o = ctx->ops;
    cudaStream_t m = ctx->stream;
    const bool ser = serial(ctx);
    cudaStream_t sf = ser ? m : ctx->s_fwd, sp = ser ? m : ctx->s_pair, sk = ser ? m : ctx->s_ccf;
    cudaStream_t sh = ser ? m : ctx->s_h2d, sc = ser ? m : ctx->s_comm;
    const int64_t np = pb - pa;
    if (np > 0) {
        CK(cudaMemsetAsync(ctx->keys + pa, 0, (size_t)np * sizeof(unsigned long long), m), "memset");
        CK(cudaMemsetAsync(ctx->mom + pa * 20, 0, (size_t)np * 20 * sizeof(unsigned long long), m),
           "memset");
    }
    if (ctx->timing == 3) {
        ctx->tl.clear();
        ctx->tl_used = 0;
        CK(tl_event(ctx, &ctx->tl_origin), "event");
        CK(cudaEventRecord(ctx->tl_origin, m), "event");
    }
    if (!ser) {
        CK(cudaEventRecord(ctx->ev_fork, m), "fork");
        for (cudaStream_t st : {sf, sp, sk, sh, sc})
            if (st) CK(cudaStreamWaitEvent(st, ctx->ev_fork, 0), "fork wait");
    }
    if (src && ctx->L.exchange && ctx->recv_cnt > 0) {
        // the halo's spectra arrive by NCCL, its pixels (K5 reads tile A) from the host: copied
        // ahead of the first forward chunk's tiles on the same stream, so every pair chunk
        // (ordered after a forward chunk) finds them
        FwdChunk halo{ctx->recv_lt, ctx->recv_cnt};
        stitch_status st = copy_chunk_in(ctx, halo, src, sh);
        if (st != STITCH_OK) return st;
    }
    int waited = -1, last_fwd = -1;
    bool halo_waited = false, any_k4 = false;
    // K5 runs over groups of consecutive pair chunks holding >= K5_MIN_PAIRS pairs (a K5
    // launch of a few pairs cannot fill the GPU: the fp64 path's 8-pair chunks made it 5x
    // slower); every chunk of a group gets its ev_k5 once the group's K5 is enqueued.
    constexpr int K5_MIN_PAIRS = 128;
    int g_first = -1, g_last = -1;   // pending group: pair chunks [g_first, g_last]
    auto flush_k5 = [&]() -> stitch_status {
        if (g_first < 0) return STITCH_OK;
        const PairChunk &a = ctx->pch[g_first], &b = ctx->pch[g_last];
        const int64_t q0 = a.p0;
        const int nq = (int)(b.p0 + b.np - a.p0);
        if (!ser) CK(cudaStreamWaitEvent(sk, ctx->ev_k4[g_last], 0), "wait k4");
        tl_wrap(ctx, sk, 2, 4, [&] {
            o->k5(ctx->raw, ctx->pairs, ctx->keys, ctx->mom, (int)q0, nq, sk);
        });
        mark(ctx, 4);
        ctx->launches += 1;
        if (!ser)
            for (int c = g_first; c <= g_last; ++c)
                CK(cudaEventRecord(ctx->ev_k5[c], sk), "event");
        g_first = g_last = -1;
        return STITCH_OK;
    };
    for (const Op& op : ops) {
        if (op.kind == Op::FWD) {
            const FwdChunk& fc = ctx->fwd[op.idx];
            if (fc.wait_pair >= 0 && g_first >= 0 && fc.wait_pair >= g_first) {
                stitch_status st = flush_k5();   // the slots it waits for are freed by this K5
                if (st != STITCH_OK) return st;
            }
            if (!ser) {   // bounded mode: the slots this chunk takes must be free
                if (fc.wait_pair >= 0) {
                    CK(cudaStreamWaitEvent(sf, ctx->ev_k5[fc.wait_pair], 0), "wait slot");
                    if (src) CK(cudaStreamWaitEvent(sh, ctx->ev_k5[fc.wait_pair], 0), "wait slot");
                }
                if (fc.wait_fwd >= 0 && src)
                    CK(cudaStreamWaitEvent(sh, ctx->ev_fwd[fc.wait_fwd], 0), "wait slot");
            }
            if (src) {
                stitch_status st = copy_chunk_in(ctx, fc, src, sh);
                if (st != STITCH_OK) return st;
                if (!ser) {
                    CK(cudaEventRecord(ctx->ev_h2d[op.idx], sh), "event");
                    CK(cudaStreamWaitEvent(sf, ctx->ev_h2d[op.idx], 0), "wait H2D");
                }
            }
            launch_fwd(ctx, fc.t0, fc.nt, sf, 0);
            if (!ser) CK(cudaEventRecord(ctx->ev_fwd[op.idx], sf), "event");
            last_fwd = op.idx;
        } else if (op.kind == Op::EXCH) {
            if (!ser && last_fwd >= 0) CK(cudaStreamWaitEvent(sc, ctx->ev_fwd[last_fwd], 0), "wait");
            stitch_status st = exchange(ctx, sc);
            if (st != STITCH_OK) return st;
            if (!ser) CK(cudaEventRecord(ctx->ev_halo, sc), "event");
        } else {
            const PairChunk& pc = ctx->pch[op.idx];
            if (!ser) {
                if (wait_fwd && pc.need > waited) {
                    CK(cudaStreamWaitEvent(sp, ctx->ev_fwd[pc.need], 0), "wait forward");
                    waited = pc.need;
                }
                if (pc.boundary && ctx->L.exchange && !halo_waited) {
                    CK(cudaStreamWaitEvent(sp, ctx->ev_halo, 0), "wait halo");
                    halo_waited = true;
                }
            }
            if (ctx->timing && !any_k4 && ser) CK(cudaEventRecord(ctx->ev[1], m), "event");
            any_k4 = true;
            if (ctx->prec) {   // fp64 path (f2): D3, D4 (per-block argmax partials), D5 -> keys
                tl_wrap(ctx, sp, 1, 2, [&] {
                    o->d3(ctx->Ud, ctx->Qd, ctx->pairs, (int)pc.p0, pc.np, ctx->twHd, sp);
                });
                mark(ctx, 2);
                tl_wrap(ctx, sp, 1, 3, [&] {
                    o->d4(ctx->Qd, ctx->part_v, ctx->part_i, (int)pc.p0, pc.np, ctx->twMd,
                          ctx->twWd, sp);
                    const size_t pb0 = (size_t)pc.p0 * o->nblk64;
                    d5_argmax_keys<<<(unsigned)((pc.np + 7) / 8), 256, 0, sp>>>(
                        ctx->part_v + pb0, ctx->part_i + pb0, ctx->keys + pc.p0, o->nblk64, pc.np);
                });
                mark(ctx, 3);
                ctx->launches += 1;
            } else {
                tl_wrap(ctx, sp, 1, 2, [&] {
                    o->k3(ctx->spec, ctx->Q, ctx->pairs, (int)pc.p0, pc.np, ctx->twH, sp);
                });
                mark(ctx, 2);
                tl_wrap(ctx, sp, 1, 3, [&] {
                    o->k4(ctx->Q, ctx->keys, (int)pc.p0, pc.np, ctx->twM, ctx->twW, ctx->grid_k4,
                          sp);
                });
                mark(ctx, 3);
            }
            if (!ser) CK(cudaEventRecord(ctx->ev_k4[op.idx], sp), "event");
            ctx->launches += 2;
            if (g_first < 0 || g_last != op.idx - 1 ||
                ctx->pch[op.idx].p0 + pc.np - ctx->pch[g_first].p0 > 65535) {
                stitch_status st = flush_k5();
                if (st != STITCH_OK) return st;
                g_first = op.idx;
            }
            g_last = op.idx;
            if (pc.p0 + pc.np - ctx->pch[g_first].p0 >= K5_MIN_PAIRS) {
                stitch_status st = flush_k5();
                if (st != STITCH_OK) return st;
            }
        }
    }
    {
        stitch_status st = flush_k5();
        if (st != STITCH_OK) return st;
    }
    if (ctx->timing && ser) CK(cudaEventRecord(ctx->ev[2], m), "event");
    if (np > 0) {
        tl_wrap(ctx, sk, 2, 5, [&] {
            // the key's value is max |c| (fp64 path) or max |c| x 32767^2 (Q15 phasor NCPS)
            k6_finalize<<<(unsigned)((np + 127) / 128), 128, 0, sk>>>(
                ctx->keys + pa, ctx->mom + pa * 20, ctx->res + pa, ctx->H, ctx->W, (int)np,
                (double)ctx->W * ctx->H * (ctx->prec ? Q31_S * Q31_S : NCPS_Q15_SCALE * o->q_scale));
        });
        mark(ctx, 5);
        ctx->launches += 1;
    }
    CK(cudaGetLastError(), "launch");
    if (!ser) {
        int j = 0;
        for (cudaStream_t st : {sf, sp, sk, sh, sc}) {
            if (!st) continue;
            CK(cudaEventRecord(ctx->ev_join[j], st), "join");
            CK(cudaStreamWaitEvent(m, ctx->ev_join[j], 0), "join wait");
            ++j;
        }
    }
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

static stitch_status step_end(stitch_ctx* ctx) {
    if (ctx->timing) CK(cudaEventRecord(ctx->ev[3], ctx->stream), "event");
    return STITCH_OK;
}

extern "C++" {
// Enqueue `body` (which launches on ctx->stream) directly, or -- graph mode, no event
// timing, no NCCL -- as a CUDA graph captured once per key on the internal capture stream
// and replayed on the caller's stream.  Every launch parameter (pointers, tensor maps, the
// schedule) is fixed per context, so a replay is exactly the captured sequence; only the
// host source of the H2D copies may change between replays (`src`): the graph's memcpy nodes
// are then re-pointed in place (cudaGraphExecMemcpyNodeSetParams), so one executable graph
// serves any number of caller buffers.
template <class F>
static stitch_status run_graphed(stitch_ctx* ctx, uint64_t key, F body,
                                 const uint16_t* src = nullptr) {
    if (ctx->timing || !ctx->use_graph || ctx->comm) return body();
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
        stitch_ctx::GraphRec rec;
        rec.graph = g;
        rec.launches = ctx->launches - l0;
        rec.src = reinterpret_cast<const char*>(src);
        if (src) {   // remember the H2D nodes (the only memcpy nodes of a step)
            size_t nn = 0;
            CK(cudaGraphGetNodes(g, nullptr, &nn), "graph nodes");
            std::vector<cudaGraphNode_t> nodes(nn);
            CK(cudaGraphGetNodes(g, nodes.data(), &nn), "graph nodes");
            for (cudaGraphNode_t nd : nodes) {
                cudaGraphNodeType ty;
                CK(cudaGraphNodeGetType(nd, &ty), "node type");
                if (ty != cudaGraphNodeTypeMemcpy) continue;
                cudaMemcpy3DParms p;
                CK(cudaGraphMemcpyNodeGetParams(nd, &p), "memcpy params");
                rec.h2d.push_back(nd);
                rec.h2d_p.push_back(p);
            }
        }
        e = cudaGraphInstantiate(&rec.exec, g, 0);
        if (e != cudaSuccess) {
            cudaGraphDestroy(g);
            return cuda_fail(ctx, e, "graph instantiate");
        }
        it = ctx->graphs.emplace(key, rec).first;
        ctx->launches = l0;
    }
    stitch_ctx::GraphRec& rec = it->second;
    if (src && reinterpret_cast<const char*>(src) != rec.src) {
        const char* ns = reinterpret_cast<const char*>(src);
        for (size_t i = 0; i < rec.h2d.size(); ++i) {
            cudaMemcpy3DParms p = rec.h2d_p[i];
            p.srcPtr.ptr = const_cast<char*>(ns + (static_cast<const char*>(p.srcPtr.ptr) - rec.src));
            CK(cudaGraphExecMemcpyNodeSetParams(rec.exec, rec.h2d[i], &p), "re-point H2D node");
            rec.h2d_p[i] = p;
        }
        rec.src = ns;
    }
    CK(cudaGraphLaunch(rec.exec, ctx->stream), "graph launch");
    ctx->launches += rec.launches;
    return STITCH_OK;
}
}  // extern "C++"

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
    if (ctx->timing) {   // stage events a split step did not record read as 0
        for (int i = 0; i < 4; ++i) {
            if (cudaEventElapsedTime(&ctx->ms[i], ctx->ev[i < 3 ? i : 0], ctx->ev[i < 3 ? i + 1 : 3]) !=
                cudaSuccess) {
                ctx->ms[i] = 0.f;
                cudaGetLastError();
            }
        }
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

extern "C" {

const char* stitch_status_string(stitch_status s) {
    switch (s) {
        case STITCH_OK: return "ok";
        case STITCH_ERR_INVALID_ARG: return "invalid argument";
        case STITCH_ERR_UNSUPPORTED: return "unsupported tile size or mode";
        case STITCH_ERR_OUT_OF_MEMORY: return "out of device memory";
        case STITCH_ERR_CUDA: return "CUDA error";
        case STITCH_ERR_NCCL: return "NCCL error";
        case STITCH_ERR_STATE: return "invalid call order";
    }
    return "unknown status";
}

stitch_status stitch_nccl_unique_id(void* out128) {
    if (!out128) return STITCH_ERR_INVALID_ARG;
    const NcclApi& api = nccl();
    if (!api.ok) return STITCH_ERR_NCCL;
    ncclUniqueId id;
    if (api.get_unique_id(&id) != ncclSuccess) return STITCH_ERR_NCCL;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(out128, &id, sizeof(id));
    return STITCH_OK;
}

stitch_status stitch_workspace_size(const stitch_config* cfg, size_t* bytes) {
    const PlanOps* ops;
    if (!bytes) return STITCH_ERR_INVALID_ARG;
    stitch_status s = check_config(cfg, &ops);
    if (s != STITCH_OK) return s;
    Layout L;
    if ((s = make_layout(cfg, ops, &L)) != STITCH_OK) return s;
    if (L.pool) {   // the bounded mode's schedule must exist for this pool (host simulation)
        stitch_ctx tmp;
        tmp.L = L;
        tmp.n = cfg->grid_rows;
        tmp.m = cfg->grid_cols;
        std::string why;
        if (!build_pooled(&tmp, &why)) return STITCH_ERR_INVALID_ARG;
    }
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
    DevGuard guard(ctx->cfg.device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    if (ctx->comm) nccl().comm_destroy(ctx->comm);
    for (auto& e : ctx->ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->kev)
        if (e) cudaEventDestroy(e);
    for (auto& g : ctx->graphs) {
        if (g.second.exec) cudaGraphExecDestroy(g.second.exec);
        if (g.second.graph) cudaGraphDestroy(g.second.graph);
    }
    if (ctx->cap_stream) cudaStreamDestroy(ctx->cap_stream);
    for (auto* v : {&ctx->ev_fwd, &ctx->ev_k4, &ctx->ev_k5, &ctx->ev_h2d, &ctx->tl_pool})
        for (auto& e : *v)
            if (e) cudaEventDestroy(e);
    for (cudaEvent_t e : {ctx->ev_fork, ctx->ev_halo})
        if (e) cudaEventDestroy(e);
    for (auto& e : ctx->ev_join)
        if (e) cudaEventDestroy(e);
    for (cudaStream_t st : {ctx->s_fwd, ctx->s_pair, ctx->s_ccf, ctx->s_h2d, ctx->s_comm})
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
    ctx->prec = L.prec;
    // the static schedule (host only: an infeasible pool fails before any device work)
    if (L.pool) {
        std::string why;
        if (!build_pooled(ctx, &why)) {
            delete ctx;
            return STITCH_ERR_INVALID_ARG;
        }
    } else {
        build_resident(ctx);
    }
    ctx->res_h.resize((size_t)L.npairs);
    DevGuard guard(cfg->device);
    if (guard.err != cudaSuccess) {
        delete ctx;
        return STITCH_ERR_CUDA;
    }
    auto bail = [&](stitch_status st) {
        stitch_destroy(ctx);
        return st;
    };
    cudaError_t e;
    if ((e = ops->setup(&ctx->grid_k1, &ctx->grid_k4)) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    if (ctx->prec && (e = ops->d_setup()) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cfg->device);
    ctx->col_ahead = 2 * sms;   // K2's L2 prefetch one wave (2 CTAs per SM) ahead
    ctx->use_graph = !(cfg->flags & STITCH_FLAG_NO_GRAPH);
    ctx->concurrent = !(cfg->flags & STITCH_FLAG_SERIAL);

    if (ctx->concurrent) {
        for (cudaStream_t* st : {&ctx->s_fwd, &ctx->s_pair, &ctx->s_ccf, &ctx->s_h2d})
            if (cudaStreamCreateWithFlags(st, cudaStreamNonBlocking) != cudaSuccess)
                return bail(STITCH_ERR_CUDA);
        auto mk = [&](std::vector<cudaEvent_t>& v, size_t k) {
            v.assign(k, nullptr);
            for (auto& ev : v)
                if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) return false;
            return true;
        };
        if (!mk(ctx->ev_fwd, ctx->fwd.size()) || !mk(ctx->ev_h2d, ctx->fwd.size()) ||
            !mk(ctx->ev_k4, ctx->pch.size()) || !mk(ctx->ev_k5, ctx->pch.size()))
            return bail(STITCH_ERR_CUDA);
        for (cudaEvent_t* ev : {&ctx->ev_fork, &ctx->ev_halo})
            if (cudaEventCreateWithFlags(ev, cudaEventDisableTiming) != cudaSuccess)
                return bail(STITCH_ERR_CUDA);
        for (auto& ev : ctx->ev_join)
            if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess)
                return bail(STITCH_ERR_CUDA);
    }
    if (ctx->use_graph &&
        cudaStreamCreateWithFlags(&ctx->cap_stream, cudaStreamNonBlocking) != cudaSuccess)
        return bail(STITCH_ERR_CUDA);
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
    ctx->pairs = (PairIdx*)(b + L.off_pairs);
    ctx->keys = (unsigned long long*)(b + L.off_keys);
    ctx->mom = (unsigned long long*)(b + L.off_mom);
    ctx->res = (stitch_pair*)(b + L.off_res);
    ctx->twM = (float2*)(b + L.off_tw);
    ctx->twH = ctx->twM + tw_row(ops);
    ctx->twW = ctx->twH + tw_col(ops);
    ctx->fslot = (int32_t*)(b + L.off_fslot);
    if (ctx->prec) {
        ctx->Ud = (int2*)(b + L.off_spec);
        ctx->Gd = (double2*)(b + L.off_g);
        ctx->Qd = (double2*)(b + L.off_q);
        ctx->twMd = (double2*)(b + L.off_tw);
        ctx->twHd = ctx->twMd + tw_row(ops);
        ctx->twWd = ctx->twHd + tw_col(ops);
        const size_t np1 = (size_t)(L.npairs > 0 ? L.npairs : 1) * ops->nblk64;
        ctx->part_v = (double*)(b + L.off_part);
        ctx->part_i = (uint32_t*)(b + L.off_part + np1 * sizeof(double));
    }

    // Twiddles w_N^e = exp(-2 pi i e / N), computed in double, rounded once.
    //   stage-2 tables: tw2[b*(r1-1) + j-1] = w_N^{j b}, b < r0, 1 <= j < r1 (fft_engine.cuh)
    auto fill_tw = [&](auto* dst, auto make) {
        auto w = [&](long ex, long N) {
            const double a = -2.0 * M_PI * (double)(ex % N) / (double)N;
            return make(std::cos(a), std::sin(a));
        };
        auto fill2 = [&](auto* d, int r0, int r1) {
            const int N = r0 * r1;
            for (int bb = 0; bb < r0; ++bb)
                for (int j = 1; j < r1; ++j) d[(size_t)bb * (r1 - 1) + j - 1] = w((long)j * bb, N);
        };
        fill2(dst, ops->row_r0, ops->row_r1);
        fill2(dst + tw_row(ops), ops->col_r0, ops->col_r1);
        for (int k = 0; k < ops->W; ++k) dst[tw_row(ops) + tw_col(ops) + k] = w(k, ops->W);
    };
    std::vector<float2> tw(tw_count(ops));
    std::vector<double2> twd;
    if (ctx->prec) {
        twd.resize(tw_count(ops));
        fill_tw(twd.data(), [](double c, double sn) { return make_double2(c, sn); });
        e = cudaMemcpyAsync(ctx->twMd, twd.data(), twd.size() * sizeof(double2),
                            cudaMemcpyHostToDevice, ctx->stream);
    } else {
        fill_tw(tw.data(), [](double c, double sn) { return make_float2((float)c, (float)sn); });
        e = cudaMemcpyAsync(ctx->twM, tw.data(), tw.size() * sizeof(float2),
                            cudaMemcpyHostToDevice, ctx->stream);
    }
    if (e != cudaSuccess) return bail(STITCH_ERR_CUDA);
    if (!ctx->pairs_h.empty() &&
        cudaMemcpyAsync(ctx->pairs, ctx->pairs_h.data(), ctx->pairs_h.size() * sizeof(PairIdx),
                        cudaMemcpyHostToDevice, ctx->stream) != cudaSuccess)
        return bail(STITCH_ERR_CUDA);
    if (cudaMemcpyAsync(ctx->fslot, ctx->fslot_h.data(), ctx->fslot_h.size() * sizeof(int32_t),
                        cudaMemcpyHostToDevice, ctx->stream) != cudaSuccess)
        return bail(STITCH_ERR_CUDA);
    for (auto& ev : ctx->ev)
        if (cudaEventCreate(&ev) != cudaSuccess) return bail(STITCH_ERR_CUDA);
    if (cudaStreamSynchronize(ctx->stream) != cudaSuccess) return bail(STITCH_ERR_CUDA);

    // NCCL communicator (collective over the world: every rank calls stitch_init)
    if (L.exchange) {
        const NcclApi& api = nccl();
        if (!api.ok) return bail(STITCH_ERR_NCCL);
        ncclUniqueId id;
        std::memcpy(&id, cfg->nccl_id, sizeof(id));
        if (api.comm_init_rank(&ctx->comm, L.world, id, L.rank) != ncclSuccess) {
            ctx->comm = nullptr;
            return bail(STITCH_ERR_NCCL);
        }
        if (cudaStreamCreateWithFlags(&ctx->s_comm, cudaStreamNonBlocking) != cudaSuccess)
            return bail(STITCH_ERR_CUDA);
        const int64_t nt = (int64_t)ctx->n * ctx->m;
        if (L.rank + 1 < L.world) {   // rank+1's halo: the last m tiles of this band
            int nb, ne;
            band_of(nt, L.rank + 1, L.world, &nb, &ne);
            const int nh = nb - ctx->m > 0 ? nb - ctx->m : 0;
            ctx->send_lt = nh - L.h_begin;
            ctx->send_cnt = nb - nh;
        }
        ctx->recv_lt = 0;
        ctx->recv_cnt = L.t_begin - L.h_begin;
    }
    *out = ctx;
    return STITCH_OK;
}

static stitch_status load_common(stitch_ctx* ctx, const uint16_t* src, int first_tile,
                                 int64_t count, bool on_device) {
    if (ctx->L.pool)
        return fail(ctx, STITCH_ERR_STATE,
                    "bounded-mode context: tiles arrive with stitch_compute_translations_from_host_async");
    if (first_tile > ctx->L.h_begin || first_tile + count < ctx->L.t_end || first_tile < 0)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range does not cover [halo_begin, tile_end)");
    const size_t tile = (size_t)ctx->H * ctx->W;
    CK(cudaMemcpyAsync(ctx->raw, src + (size_t)(ctx->L.h_begin - first_tile) * tile,
                       (size_t)ctx->L.nlocal * tile * sizeof(uint16_t),
                       on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, ctx->stream),
       "load tiles");
    // host memory: return only once the copy is done, so the caller may reuse the buffer
    if (!on_device) CK(cudaStreamSynchronize(ctx->stream), "load synchronize");
    ctx->loaded = true;
    ctx->computed = false;
    return STITCH_OK;
}

stitch_status stitch_load_tiles(stitch_ctx* ctx, const uint16_t* tiles, int32_t first_tile,
                                int32_t count, int32_t on_device) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!tiles) return fail(ctx, STITCH_ERR_INVALID_ARG, "null tiles pointer");
    GUARD(ctx);
    return load_common(ctx, tiles, first_tile, count, on_device != 0);
}

stitch_status stitch_resident_range(stitch_ctx* ctx, int32_t* halo_begin, int32_t* tile_begin,
                                    int32_t* tile_end) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (halo_begin) *halo_begin = ctx->L.h_begin;
    if (tile_begin) *tile_begin = ctx->L.t_begin;
    if (tile_end) *tile_end = ctx->L.t_end;
    return STITCH_OK;
}

static stitch_status load_grid(stitch_ctx* ctx, const uint16_t* src, size_t n_bytes, bool dev) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!src) return fail(ctx, STITCH_ERR_INVALID_ARG, "null grid pointer");
    if (n_bytes != (size_t)ctx->n * ctx->m * ctx->H * ctx->W * sizeof(uint16_t))
        return fail(ctx, STITCH_ERR_INVALID_ARG, "n_bytes != n*m*H*W*2");
    GUARD(ctx);
    return load_common(ctx, src, 0, (int64_t)ctx->n * ctx->m, dev);
}

stitch_status stitch_load_grid(stitch_ctx* ctx, const uint16_t* host_grid, size_t n_bytes) {
    return load_grid(ctx, host_grid, n_bytes, false);
}

stitch_status stitch_load_grid_device(stitch_ctx* ctx, const uint16_t* dev_grid, size_t n_bytes) {
    return load_grid(ctx, dev_grid, n_bytes, true);
}

stitch_status stitch_forward_async(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    return stitch_forward_range_async(ctx, ctx->L.h_begin, ctx->L.nlocal);
}

stitch_status stitch_forward_range_async(stitch_ctx* ctx, int32_t first_tile, int32_t count) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (ctx->L.pool) return fail(ctx, STITCH_ERR_STATE, "split step: not in the bounded mode");
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "forward before load");
    if (count < 0 || first_tile < ctx->L.h_begin || first_tile + (int64_t)count > ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range not resident");
    GUARD(ctx);
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    const int lt0 = first_tile - ctx->L.h_begin, ct = ctx->L.chunk_tiles;
    const uint64_t key = (2ull << 60) | ((uint64_t)(uint32_t)first_tile << 30) | (uint32_t)count;
    st = run_graphed(ctx, key, [&]() -> stitch_status {
        for (int t0 = lt0; t0 < lt0 + count; t0 += ct) {
            const int nt = std::min(ct, lt0 + count - t0);
            launch_fwd(ctx, t0, nt, ctx->stream, 0);
        }
        CK(cudaGetLastError(), "forward launch");
        return STITCH_OK;
    });
    if (st == STITCH_OK && ctx->timing) CK(cudaEventRecord(ctx->ev[1], ctx->stream), "event");
    return st;
}

stitch_status stitch_pairs_part_async(stitch_ctx* ctx, int32_t part) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (part < 0 || part > 2) return fail(ctx, STITCH_ERR_INVALID_ARG, "part must be 0, 1 or 2");
    if (ctx->L.pool) return fail(ctx, STITCH_ERR_STATE, "split step: not in the bounded mode");
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "pairs before load");
    GUARD(ctx);
    const int c0 = part == 2 ? ctx->c_boundary : 0;
    const int c1 = part == 1 ? ctx->c_boundary : (int)ctx->pch.size();
    const int64_t pa = part == 2 ? ctx->n_interior : 0;
    const int64_t pb = part == 1 ? ctx->n_interior : ctx->L.npairs;
    std::vector<Op> ops;
    for (int c = c0; c < c1; ++c) ops.push_back(Op{Op::PAIR, c});
    stitch_status st = run_graphed(ctx, (3ull << 60) | (uint64_t)part,
                                   [&]() { return enqueue_ops(ctx, ops, nullptr, false, pa, pb); });
    if (st == STITCH_OK) ctx->computed = true;
    return st;
}

stitch_status stitch_pairs_async(stitch_ctx* ctx) { return stitch_pairs_part_async(ctx, 0); }

stitch_status stitch_compute_translations_async(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (ctx->L.pool)
        return fail(ctx, STITCH_ERR_STATE,
                    "bounded-mode context: use stitch_compute_translations_from_host_async");
    if (!ctx->loaded) return fail(ctx, STITCH_ERR_STATE, "compute before load");
    GUARD(ctx);
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    st = run_graphed(ctx, 1ull << 60, [&]() {
        return enqueue_ops(ctx, ctx->ops_step, nullptr, true, 0, ctx->L.npairs);
    });
    if (st == STITCH_OK) ctx->computed = true;
    return st == STITCH_OK ? step_end(ctx) : st;
}

stitch_status stitch_compute_translations_from_host_async(stitch_ctx* ctx, const uint16_t* tiles,
                                                         int32_t first_tile, int32_t count) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!tiles) return fail(ctx, STITCH_ERR_INVALID_ARG, "null tiles pointer");
    if (first_tile > ctx->L.h_begin || first_tile + (int64_t)count < ctx->L.t_end || first_tile < 0)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range does not cover [halo_begin, tile_end)");
    GUARD(ctx);
    const uint16_t* src = tiles + (size_t)(ctx->L.h_begin - first_tile) * ctx->H * ctx->W;
    cudaPointerAttributes pa;
    const bool pinned = cudaPointerGetAttributes(&pa, tiles) == cudaSuccess &&
                        pa.type == cudaMemoryTypeHost;
    cudaGetLastError();   // clear a pointer-query error on pageable memory
    stitch_status st = step_begin(ctx);
    if (st != STITCH_OK) return st;
    auto body = [&]() { return enqueue_ops(ctx, ctx->ops_step, src, true, 0, ctx->L.npairs); };
    // pinned: one captured graph whose H2D nodes are re-pointed at each new buffer; pageable
    // memory cannot be captured (its copies are staged by the driver): direct launches
    st = pinned ? run_graphed(ctx, 4ull << 60, body, src) : body();
    if (st != STITCH_OK) return st;
    if (!ctx->L.pool) ctx->loaded = true;   // resident: every tile is now on the device
    ctx->computed = true;
    return step_end(ctx);
}

stitch_status stitch_spectra_range(stitch_ctx* ctx, int32_t first_tile, int32_t count,
                                   void** dev_ptr, size_t* bytes) {
    if (!ctx || !dev_ptr || !bytes) return STITCH_ERR_INVALID_ARG;
    if (ctx->L.pool) return fail(ctx, STITCH_ERR_STATE, "bounded mode: spectra are not resident");
    if (count < 0 || first_tile < ctx->L.h_begin || first_tile + (int64_t)count > ctx->L.t_end)
        return fail(ctx, STITCH_ERR_INVALID_ARG, "tile range not resident");
    const size_t per = ctx->L.spec_tile_bytes;
    *dev_ptr = reinterpret_cast<char*>(ctx->prec ? (void*)ctx->Ud : (void*)ctx->spec) +
               (size_t)(first_tile - ctx->L.h_begin) * per;
    *bytes = (size_t)count * per;
    return STITCH_OK;
}

stitch_status stitch_get_translations(stitch_ctx* ctx, stitch_pair* west, stitch_pair* north) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!west || !north) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output array");
    if (!ctx->computed) return fail(ctx, STITCH_ERR_STATE, "no computed translations");
    GUARD(ctx);
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
    GUARD(ctx);
    // The resident store keeps Q15 unit phasors; recompute the complex spectrum of this tile
    // with the same K1 + K2 kernels (G slot 0, K2 writing the complex spectrum row-major into
    // the Q chunk buffer) and copy it out.
    const int lt = tile - ctx->L.h_begin;
    const PlanOps* o = ctx->ops;
    o->k1(ctx->raw, ctx->G, lt, 1, ctx->fslot, ctx->twM, ctx->twW, ctx->grid_k1, ctx->stream);
    o->k2(ctx->G, ctx->Q, ctx->spec, lt, 1, ctx->fslot, ctx->twH, false, 0, ctx->stream);
    CK(cudaGetLastError(), "spectrum launch");
    CK(cudaMemcpy2DAsync(host_out, ctx->ops->WC * sizeof(float2), ctx->Q,
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
    GUARD(ctx);
    // the resident store keeps unit phasors: recompute this tile's complex spectrum with the
    // same D1 + D2 kernels (Gd slot 0; D2 writing the complex spectrum row-major into Qd)
    const int lt = tile - ctx->L.h_begin;
    const PlanOps* o = ctx->ops;
    o->d1(ctx->raw, ctx->Gd, lt, 1, ctx->twMd, ctx->twWd, ctx->stream);
    o->d2(ctx->Gd, ctx->Ud, ctx->Qd, lt, 1, ctx->twHd, false, ctx->stream);
    CK(cudaGetLastError(), "spectrum launch");
    CK(cudaMemcpy2DAsync(host_out, ctx->ops->WC * sizeof(double2), ctx->Qd,
                         ctx->ops->WP * sizeof(double2), ctx->ops->WC * sizeof(double2), ctx->H,
                         cudaMemcpyDeviceToHost, ctx->stream),
       "copy spectrum");
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    return STITCH_OK;
}

stitch_status stitch_debug_surface(stitch_ctx* ctx, int32_t tile, int32_t kind, float* host_out) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    if (!host_out) return fail(ctx, STITCH_ERR_INVALID_ARG, "null output");
    if (ctx->prec || ctx->L.pool)
        return fail(ctx, STITCH_ERR_STATE, "surface hook: fp32 resident contexts only");
    if (!ctx->computed) return fail(ctx, STITCH_ERR_STATE, "surface before a compute");
    int64_t p = -1;
    for (int64_t i = 0; i < ctx->L.npairs; ++i)
        if (ctx->pair_tile[i] == tile && ctx->pair_kind[i] == kind) p = i;
    if (p < 0) return fail(ctx, STITCH_ERR_INVALID_ARG, "the context computes no such pair");
    GUARD(ctx);
    const PlanOps* o = ctx->ops;
    float* surf = reinterpret_cast<float*>(ctx->G);   // H*W floats fit one chunk slot of G
    const float scale = (float)(1.0 / ((double)ctx->W * ctx->H * NCPS_Q15_SCALE * ctx->ops->q_scale));
    o->k3(ctx->spec, ctx->Q, ctx->pairs, (int)p, 1, ctx->twH, ctx->stream);
    o->k4s(ctx->Q, surf, scale, ctx->twM, ctx->twW, ctx->grid_k4, ctx->stream);
    CK(cudaGetLastError(), "surface launch");
    CK(cudaMemcpyAsync(host_out, surf, (size_t)ctx->H * ctx->W * sizeof(float),
                       cudaMemcpyDeviceToHost, ctx->stream),
       "copy surface");
    CK(cudaStreamSynchronize(ctx->stream), "synchronize");
    return STITCH_OK;
}

stitch_status stitch_synchronize(stitch_ctx* ctx) {
    if (!ctx) return STITCH_ERR_INVALID_ARG;
    GUARD(ctx);
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
    if (forward_ffts) {
        int64_t f = 0;
        for (const FwdChunk& fc : ctx->fwd) f += fc.nt;
        *forward_ffts = f;
    }
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
    if (enabled == 3 && !ctx->concurrent)
        return fail(ctx, STITCH_ERR_STATE, "timeline needs the concurrent schedule");
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
