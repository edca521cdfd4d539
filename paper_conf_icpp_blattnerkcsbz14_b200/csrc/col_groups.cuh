// col_groups.cuh — persistent column kernels with two compute groups and a three-buffer TMA
// ring (K2g, K3g).
//
// The one-panel-per-CTA column kernels (K2t/K3t) spend ~30 % of their stall samples waiting
// for their panel at CTA start (ncu r01c, profiles/experiments): with two 7-warp CTAs per SM
// nothing prefetches the next panel, because the landing buffer doubles as the stage exchange
// and the radix-40 butterfly held in registers caps the register budget.  Here one CTA per SM
// runs two independent 7-warp groups (named barriers 1 and 2, never a CTA-wide barrier after
// the prologue) over three landing/exchange buffers.  The CTA's items k = 0, 1, 2, ... (panel
// items blockIdx.x + k*gridDim.x) alternate between the groups (k even: group 0, k odd:
// group 1); item k lives in buffer k % 3.  When a group finishes item k it issues the TMA for
// item k + 3 into the buffer it just freed and moves on to item k + 2, whose panel was
// requested when the OTHER group finished item k - 1.  After the first item the groups run
// about one TMA latency apart and neither waits for data again.
#pragma once
#include "pciam_kernels.cuh"

namespace stitch {

template <class PL>
struct ColGroups {
    static constexpr int GT = (PL::COL_T + 31) / 32 * 32;   // threads per group (whole warps)
    static constexpr int NT = 2 * GT;                       // threads per CTA
    static constexpr size_t BUF = (PL::COL_BUF + 127) / 128 * 128;
    static constexpr size_t OFF_TW = 3 * BUF;
    static constexpr size_t OFF_BAR = OFF_TW + (size_t)(PL::COL_TW2N > 0 ? PL::COL_TW2N : 2) * 8;
    static constexpr size_t SMEM = OFF_BAR + 3 * 8;
    // launched with NT <= 512 threads under __launch_bounds__(512, 1): <= 128 registers, so
    // 14 warps fit the 4 x 16K-register sub-partitions
    static constexpr bool OK = SMEM <= 227 * 1024 && PL::CI::STAGES == 2 && NT <= 512;
    using Grp = GroupOf<GT>;
};


// K2g: forward column FFT of a chunk of G (as K2t), phase-coded into the resident spectrum.
template <class PL>
__global__ void __launch_bounds__(512, 1)   // <= 128 registers (16K per sub-partition at 4 warps each)
    k2g_fwd_cols(const __grid_constant__ CUtensorMap tmG, uint32_t* __restrict__ spec, int tile0,
                 int ntiles, const float2* __restrict__ tw2) {
    using CG = ColGroups<PL>;
    using Grp = typename CG::Grp;
    extern __shared__ __align__(128) unsigned char gsmem[];
    constexpr int NP = PL::WP / PL::COL_P;
    float2* tws = reinterpret_cast<float2*>(gsmem + CG::OFF_TW);
    uint64_t* bar = reinterpret_cast<uint64_t*>(gsmem + CG::OFF_BAR);
    const int nitems = ntiles * NP;
    const int nk = ((int)blockIdx.x < nitems) ? (nitems - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
    auto issue = [&](int k) {                 // TMA of this CTA's item k into buffer k % 3
        const int item = blockIdx.x + k * gridDim.x;
        const int tl = item / NP, panel = item - tl * NP;
        uint64_t* b = &bar[k % 3];
        mbar_arrive_expect_tx(b, (uint32_t)PL::COL_LAND_C);
        tma_panel<PL>(gsmem + (size_t)(k % 3) * CG::BUF, &tmG, 2 * panel * PL::COL_P, tl * PL::H,
                      8, b);
    };
    if (threadIdx.x == 0) {
        prefetch_tensormap(&tmG);
        for (int i = 0; i < 3; ++i) mbar_init(&bar[i], 1);
        fence_mbar_init();
    }
    for (int i = threadIdx.x; i < PL::COL_TW2N; i += CG::NT) tws[i] = __ldg(tw2 + i);
    __syncthreads();                          // the only CTA-wide barrier
    if (threadIdx.x == 0)
        for (int k = 0; k < 3 && k < nk; ++k) issue(k);
    const int g = Grp::id();
    using Run = FftRun<typename PL::Col, -1, PL::COL_P, CG::GT, ColMap, true, float2, Grp>;
#pragma unroll 1
    for (int k = g; k < nk; k += 2) {
        unsigned char* buf = gsmem + (size_t)(k % 3) * CG::BUF;
        mbar_wait(&bar[k % 3], (k / 3) & 1);
        const int item = blockIdx.x + k * gridDim.x;
        const int tl = item / NP, c0 = (item - tl * NP) * PL::COL_P;
        LandSrc<PL> src{reinterpret_cast<const float2*>(buf)};
        typename PL::ColX xc{reinterpret_cast<float2*>(buf)};
        PhaseDst<PL> dst{spec + (size_t)(tile0 + tl) * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tws);
        Grp::sync();                          // every read of this buffer is done
        if (Grp::tid() == 0 && k + 3 < nk) {
            fence_proxy_async();
            issue(k + 3);
        }
    }
}

// K3g: NCPS from two phasor panels + inverse column FFT -> Q (as K3t).
template <class PL>
__global__ void __launch_bounds__(512, 1)   // <= 128 registers (16K per sub-partition at 4 warps each)
    k3g_pair_cols(const __grid_constant__ CUtensorMap tmS, float2* __restrict__ Q,
                  const PairIdx* __restrict__ pairs, int pair0, int npairs,
                  const float2* __restrict__ tw2) {
    using CG = ColGroups<PL>;
    using Grp = typename CG::Grp;
    extern __shared__ __align__(128) unsigned char gsmem[];
    constexpr int NP = PL::WP / PL::COL_P;
    float2* tws = reinterpret_cast<float2*>(gsmem + CG::OFF_TW);
    uint64_t* bar = reinterpret_cast<uint64_t*>(gsmem + CG::OFF_BAR);
    const int nitems = npairs * NP;
    const int nk = ((int)blockIdx.x < nitems) ? (nitems - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
    auto issue = [&](int k) {
        const int item = blockIdx.x + k * gridDim.x;
        const int pl = item / NP, panel = item - pl * NP;
        const PairIdx pr = pairs[pair0 + pl];
        unsigned char* buf = gsmem + (size_t)(k % 3) * CG::BUF;
        uint64_t* b = &bar[k % 3];
        mbar_arrive_expect_tx(b, (uint32_t)(2 * PL::H * PL::COL_P * 4));
        tma_panel<PL>(buf, &tmS, panel * PL::COL_P, pr.a * PL::H, 4, b);
        tma_panel<PL>(buf + PL::COL_PHASE_B, &tmS, panel * PL::COL_P, pr.b * PL::H, 4, b);
    };
    if (threadIdx.x == 0) {
        prefetch_tensormap(&tmS);
        for (int i = 0; i < 3; ++i) mbar_init(&bar[i], 1);
        fence_mbar_init();
    }
    for (int i = threadIdx.x; i < PL::COL_TW2N; i += CG::NT) tws[i] = __ldg(tw2 + i);
    __syncthreads();
    if (threadIdx.x == 0)
        for (int k = 0; k < 3 && k < nk; ++k) issue(k);
    const int g = Grp::id();
    using Run = FftRun<typename PL::Col, +1, PL::COL_P, CG::GT, ColMap, true, float2, Grp>;
#pragma unroll 1
    for (int k = g; k < nk; k += 2) {
        unsigned char* buf = gsmem + (size_t)(k % 3) * CG::BUF;
        mbar_wait(&bar[k % 3], (k / 3) & 1);
        const int item = blockIdx.x + k * gridDim.x;
        const int pl = item / NP, c0 = (item - pl * NP) * PL::COL_P;
        NcpsPhaseSrc<PL> src{reinterpret_cast<const uint32_t*>(buf),
                             reinterpret_cast<const uint32_t*>(buf + PL::COL_PHASE_B)};
        typename PL::ColX xc{reinterpret_cast<float2*>(buf)};
        PanelIO<PL> dst{Q + (size_t)pl * PL::H * PL::WP + c0};
        Run::template run<true>(src, xc, dst, tws);
        Grp::sync();
        if (Grp::tid() == 0 && k + 3 < nk) {
            fence_proxy_async();
            issue(k + 3);
        }
    }
}

}  // namespace stitch
