// fft_engine.cuh — batched in-CTA mixed-radix Stockham FFT for sm_100a.
//
// A CTA transforms L lines of length N.  Each stage of radix R (Stockham
// autosort, NS = product of the radices already applied) gives every thread
// whole radix-R butterflies held in registers:
//     inputs   n = b + j*(N/R),                 j < R
//     twiddle  v[j] *= w_N^{SIGN * j*k*(N/(NS*R))},  k = b mod NS
//     DFT_R    straight-line codelet (codelets.cuh)
//     outputs  n = (b/NS)*NS*R + k + j*NS
// The first stage reads from a caller "source" functor (global memory with
// the producer's arithmetic fused in: uint16->fp32, NCPS, C2R pre-twiddle)
// and the last stage writes to a "destination" functor (global memory or the
// fused argmax epilogue), so a two-stage transform makes exactly one shared-
// memory round trip.  No cuFFT, no tensor cores: the path is HBM/FP32-bound.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "codelets.cuh"

namespace stitch {

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
    return make_float2(fmaf(a.x, b.x, -a.y * b.y), fmaf(a.x, b.y, a.y * b.x));
}

// Shared-memory line storage, line-major with one float2 of padding per 16
// elements so stride-R Stockham writes spread over the 32 banks.
template <int STRIDE>
struct RowSmem {
    float2* s;
    static __host__ __device__ constexpr int phys(int n) { return n + (n >> 4); }
    __device__ __forceinline__ float2 load(int line, int n) const { return s[line * STRIDE + phys(n)]; }
    __device__ __forceinline__ void store(int line, int n, float2 v) const { s[line * STRIDE + phys(n)] = v; }
};

// Column-panel storage: element n of line (column) c at n*P + c, so 16
// consecutive threads touch 16 consecutive columns (one 128-byte wavefront).
template <int P>
struct ColSmem {
    float2* s;
    __device__ __forceinline__ float2 load(int line, int n) const { return s[n * P + line]; }
    __device__ __forceinline__ void store(int line, int n, float2 v) const { s[n * P + line] = v; }
};

// Butterfly id g -> (line, b).  Row map: consecutive threads walk one line.
struct RowMap {
    template <int NB, int L>
    static __device__ __forceinline__ void map(int g, int& line, int& b) {
        line = g / NB;
        b = g - line * NB;
    }
};
// Column map: consecutive threads walk across the lines (columns) of a panel.
struct ColMap {
    template <int NB, int L>
    static __device__ __forceinline__ void map(int g, int& line, int& b) {
        b = g / L;
        line = g - b * L;
    }
};

template <int N, int R, int NS, int SIGN>
__device__ __forceinline__ void butterfly(float2 (&v)[R], int b, const float2* __restrict__ tw) {
    if constexpr (NS > 1) {
        const int k = b % NS;
        constexpr int TS = N / (NS * R);
#pragma unroll
        for (int j = 1; j < R; ++j) {
            float2 w = __ldg(&tw[j * k * TS]);
            if constexpr (SIGN > 0) w.y = -w.y;
            v[j] = cmul(v[j], w);
        }
    }
    Dft<R, SIGN>::run(v);
}

// One Stockham stage.  INPLACE: src and dst alias the same shared memory, so
// every thread loads all of its butterflies before a barrier, then stores.
template <int N, int R, int NS, int SIGN, int L, int T, class Map, bool INPLACE, class Src,
          class Dst>
__device__ __forceinline__ void fft_stage(const Src& src, Dst& dst, const float2* __restrict__ tw) {
    static_assert(N % R == 0, "radix must divide N");
    constexpr int NB = N / R;
    constexpr int TOTAL = L * NB;
    constexpr int ITER = (TOTAL + T - 1) / T;
    if constexpr (INPLACE) {
        float2 v[ITER][R];
#pragma unroll
        for (int it = 0; it < ITER; ++it) {
            const int g = threadIdx.x + it * T;
            if (TOTAL % T == 0 || g < TOTAL) {
                int line, b;
                Map::template map<NB, L>(g, line, b);
#pragma unroll
                for (int j = 0; j < R; ++j) v[it][j] = src.load(line, b + j * NB);
            }
        }
        __syncthreads();
#pragma unroll
        for (int it = 0; it < ITER; ++it) {
            const int g = threadIdx.x + it * T;
            if (TOTAL % T == 0 || g < TOTAL) {
                int line, b;
                Map::template map<NB, L>(g, line, b);
                butterfly<N, R, NS, SIGN>(v[it], b, tw);
                const int base = (b / NS) * (NS * R) + (b % NS);
#pragma unroll
                for (int j = 0; j < R; ++j) dst.store(line, base + j * NS, v[it][j]);
            }
        }
    } else {
#pragma unroll
        for (int it = 0; it < ITER; ++it) {
            const int g = threadIdx.x + it * T;
            if (TOTAL % T == 0 || g < TOTAL) {
                int line, b;
                Map::template map<NB, L>(g, line, b);
                float2 v[R];
#pragma unroll
                for (int j = 0; j < R; ++j) v[j] = src.load(line, b + j * NB);
                butterfly<N, R, NS, SIGN>(v, b, tw);
                const int base = (b / NS) * (NS * R) + (b % NS);
#pragma unroll
                for (int j = 0; j < R; ++j) dst.store(line, base + j * NS, v[j]);
            }
        }
    }
}

// A length-N transform as a list of radices (applied left to right).
template <int N_, int... Rs>
struct Radix {
    static constexpr int N = N_;
    static constexpr int count = sizeof...(Rs);
};

template <class RX, int SIGN, int L, int T, class Map, bool LAST_INPLACE>
struct FftRun;

template <int N, int R0, int SIGN, int L, int T, class Map, bool LAST_INPLACE>
struct FftRun<Radix<N, R0>, SIGN, L, T, Map, LAST_INPLACE> {
    template <class Src, class Sm, class Dst>
    static __device__ __forceinline__ void run(const Src& src, Sm& sm, Dst& dst, const float2* tw) {
        static_assert(N == R0, "single-stage plan");
        fft_stage<N, R0, 1, SIGN, L, T, Map, false>(src, dst, tw);
    }
};

template <int N, int R0, int R1, int SIGN, int L, int T, class Map, bool LAST_INPLACE>
struct FftRun<Radix<N, R0, R1>, SIGN, L, T, Map, LAST_INPLACE> {
    template <class Src, class Sm, class Dst>
    static __device__ __forceinline__ void run(const Src& src, Sm& sm, Dst& dst, const float2* tw) {
        static_assert(N == R0 * R1, "radices must multiply to N");
        fft_stage<N, R0, 1, SIGN, L, T, Map, false>(src, sm, tw);
        __syncthreads();
        fft_stage<N, R1, R0, SIGN, L, T, Map, LAST_INPLACE>(sm, dst, tw);
    }
};

template <int N, int R0, int R1, int R2, int SIGN, int L, int T, class Map, bool LAST_INPLACE>
struct FftRun<Radix<N, R0, R1, R2>, SIGN, L, T, Map, LAST_INPLACE> {
    template <class Src, class Sm, class Dst>
    static __device__ __forceinline__ void run(const Src& src, Sm& sm, Dst& dst, const float2* tw) {
        static_assert(N == R0 * R1 * R2, "radices must multiply to N");
        fft_stage<N, R0, 1, SIGN, L, T, Map, false>(src, sm, tw);
        __syncthreads();
        fft_stage<N, R1, R0, SIGN, L, T, Map, true>(sm, sm, tw);
        __syncthreads();
        fft_stage<N, R2, R0 * R1, SIGN, L, T, Map, LAST_INPLACE>(sm, dst, tw);
    }
};

}  // namespace stitch
