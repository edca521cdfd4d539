// fft_engine.cuh — batched in-CTA mixed-radix Stockham FFT for sm_100a.
//
// A CTA transforms L lines of length N = R0 * R1 (one or two radix stages).
// Stockham autosort, two stages:
//   stage 1 (radix R0, butterfly b < R1):  in  n = b + j*R1          (j < R0)
//                                           out (u = j, v = b)        n = b*R0 + j
//   stage 2 (radix R1, butterfly b < R0):  in  (u = b, v = j)        n = b + j*R0 (j < R1)
//                                           twiddle w_N^{SIGN j b}
//                                           out n = b + j*R0
// so the exchange buffer is an R1 x R0 matrix written at (u=j, v=b) and read at
// (u=b, v=j): one shared-memory round trip per transform.  Each thread owns whole
// radix-R butterflies in registers (straight-line codelets, codelets.cuh).
// The first stage reads from a caller "source" functor (global memory with the
// producer's arithmetic fused in: uint16->fp32, NCPS, C2R pre-twiddle) and the
// second writes to a "destination" functor (global memory, shared memory, or the
// argmax epilogue).  Every address inside a butterfly is base + constant offset.
// No cuFFT, no tensor cores: the path is HBM- / FP32-issue-bound.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "codelets.cuh"   // includes f32x2.cuh

namespace stitch {

// fp32 complex products on the packed f32x2 instructions (two instructions each, f32x2.cuh)
__device__ __forceinline__ float2 cmul(float2 a, float2 b) { return cmul2(a, b); }
__device__ __forceinline__ float2 cmulc(float2 a, float2 b) { return cmulc2(a, b); }  // a * conj(b)
// fp64 twins (the f2 path instantiates the engine with C = double2)
__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
    return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
__device__ __forceinline__ double2 cmulc(double2 a, double2 b) {
    return make_double2(fma(a.x, b.x, a.y * b.y), fma(a.y, b.x, -a.x * b.y));
}

// Modular inverse of a mod m and gcd, at compile time (prime-factor index maps).
__host__ __device__ constexpr int modinv(int a, int m) {
    int r = 1;
    for (int x = 1; x < m; ++x)
        if ((a * x) % m == 1) r = x;
    return r;
}
__host__ __device__ constexpr int gcd_c(int a, int b) { return b == 0 ? a : gcd_c(b, a % b); }

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

// Exchange buffer for row lines: line-major, each line an R1 x (R0+PAD) matrix.
template <int R0, int R1, int PAD, class C = float2>
struct RowXchg {
    C* s;
    static constexpr int LSTRIDE = R1 * (R0 + PAD);
    __device__ __forceinline__ C& at(int line, int u, int v) const {
        return s[line * LSTRIDE + v * (R0 + PAD) + u];
    }
    // element n of the transform in natural order: the slot stage 2 read it from
    // (u = n mod R0, v = n / R0), so stage 2 may write its outputs back in place
    __device__ __forceinline__ C& nat(int line, int n) const {
        if constexpr (PAD == 0)
            return s[line * LSTRIDE + n];       // v * R0 + u == n
        else
            return at(line, n % R0, n / R0);
    }
    __device__ __forceinline__ void store(int line, int n, C v) const { nat(line, n) = v; }
};
// Exchange buffer for a panel of P columns: element (u, v) of column c at
// (v*(R0+PAD) + u)*P + c, so a warp's 8-byte accesses span all 32 banks.
template <int R0, int R1, int PAD, int P, class C = float2>
struct ColXchg {
    C* s;
    __device__ __forceinline__ C& at(int line, int u, int v) const {
        return s[(v * (R0 + PAD) + u) * P + line];
    }
};

// Stage-2 twiddle table layout: tw2[b*(R1-1) + (j-1)] = w_N^{-j b}, b < R0, 1 <= j < R1.
template <int R0, int R1>
struct Tw2 {
    static constexpr int SIZE = R0 * (R1 - 1);
};

struct NoMid {
    __device__ __forceinline__ void operator()() const {}
};

// A destination may take a whole butterfly's outputs at once (element b + j*STRIDE gets
// v[j]) by defining store_batch<R, STRIDE>(line, b, v); otherwise they are stored one by one.
template <class D, class = void>
struct HasBatch {
    static constexpr bool value = false;
};
template <class D>
struct HasBatch<D, decltype((void)&D::BATCH)> {
    static constexpr bool value = true;
};
template <int R, int STRIDE, class Dst, class C>
__device__ __forceinline__ void store_butterfly(Dst& dst, int line, int b, C (&v)[R]) {
    if constexpr (HasBatch<Dst>::value) {
        dst.template store_batch<R, STRIDE>(line, b, v);
    } else {
#pragma unroll
        for (int j = 0; j < R; ++j) dst.store(line, b + j * STRIDE, v[j]);
    }
}

template <int N_, int... Rs>
struct Radix {
    static constexpr int N = N_;
    static constexpr int count = sizeof...(Rs);
};

// The threads that run one transform batch: the whole CTA (default), or one of several
// independent thread groups of a CTA (GroupOf<GT>: group g = threadIdx.x / GT synchronises on
// named barrier 1 + g, so groups never wait for each other).
struct CtaGrp {
    static __device__ __forceinline__ int tid() { return threadIdx.x; }
    static __device__ __forceinline__ void sync() { __syncthreads(); }
};
template <int GT>
struct GroupOf {
    static_assert(GT % 32 == 0, "thread groups are whole warps");
    static __device__ __forceinline__ int tid() { return threadIdx.x % GT; }
    static __device__ __forceinline__ int id() { return threadIdx.x / GT; }
    static __device__ __forceinline__ void sync() {
        asm volatile("bar.sync %0, %1;" ::"r"(1 + id()), "n"(GT) : "memory");
    }
};

// C: the complex element type (float2, or double2 for the fp64 path f2); Grp: the thread group
template <class RX, int SIGN, int L, int T, class Map, bool TW_SMEM = false, class C = float2,
          class Grp = CtaGrp>
struct FftRun;

// One stage: N = R0, no twiddles, source -> destination.
template <int N, int R0, int SIGN, int L, int T, class Map, bool TW_SMEM, class C, class Grp>
struct FftRun<Radix<N, R0>, SIGN, L, T, Map, TW_SMEM, C, Grp> {
    static_assert(N == R0, "single-stage plan");
    static constexpr int R1 = 1;
    template <bool IN_PLACE = false, class Src, class Xc, class Dst, class Mid = NoMid,
              class AfterLoads = NoMid>
    static __device__ __forceinline__ void run(const Src& src, const Xc&, Dst& dst,
                                               const C* __restrict__, const Mid& mid = Mid(),
                                               const AfterLoads& after_loads = AfterLoads()) {
        // one butterfly per line (the source is consumed inside the loop; `mid` runs after it)
        constexpr int TOTAL = L;
        constexpr int ITER = (TOTAL + T - 1) / T;
#pragma unroll
        for (int it = 0; it < ITER; ++it) {
            const int g = Grp::tid() + it * T;
            if (TOTAL % T == 0 || g < TOTAL) {
                const int line = g;
                C v[R0];
#pragma unroll
                for (int j = 0; j < R0; ++j) v[j] = src.load(line, j);
                Dft<R0, SIGN>::run(v);
                store_butterfly<R0, 1>(dst, line, 0, v);
            }
        }
        Grp::sync();
        after_loads();
        mid();
    }
};

// Two stages: N = R0 * R1, one exchange through shared memory.
template <int N, int R0_, int R1_, int SIGN, int L, int T, class Map, bool TW_SMEM, class C,
          class Grp>
struct FftRun<Radix<N, R0_, R1_>, SIGN, L, T, Map, TW_SMEM, C, Grp> {
    static constexpr int R0 = R0_, R1 = R1_;
    static_assert(N == R0 * R1, "radices must multiply to N");
    // Stage 1: radix R0 over R1 butterflies per line, source -> exchange.  IN_PLACE: the
    // source is the exchange buffer itself (a landing buffer reused as the exchange), so
    // every thread loads all of its butterflies before a barrier, then computes and stores.
    template <bool IN_PLACE, class Src, class Xc, class AfterLoads = NoMid>
    static __device__ __forceinline__ void stage1(const Src& src, const Xc& xc,
                                                  const AfterLoads& after_loads = AfterLoads()) {
        constexpr int TOTAL = L * R1;
        constexpr int ITER = (TOTAL + T - 1) / T;
        if constexpr (IN_PLACE) {
            C v[ITER][R0];
#pragma unroll
            for (int it = 0; it < ITER; ++it) {
                const int g = Grp::tid() + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    int line, b;
                    Map::template map<R1, L>(g, line, b);
#pragma unroll
                    for (int j = 0; j < R0; ++j) v[it][j] = src.load(line, b + j * R1);
                }
            }
            Grp::sync();
            after_loads();   // the source buffer is free from here on
#pragma unroll
            for (int it = 0; it < ITER; ++it) {
                const int g = Grp::tid() + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    int line, b;
                    Map::template map<R1, L>(g, line, b);
                    Dft<R0, SIGN>::run(v[it]);
#pragma unroll
                    for (int j = 0; j < R0; ++j) xc.at(line, j, b) = v[it][j];
                }
            }
        } else {
#pragma unroll
            for (int it = 0; it < ITER; ++it) {
                const int g = Grp::tid() + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    int line, b;
                    Map::template map<R1, L>(g, line, b);
                    C v[R0];
#pragma unroll
                    for (int j = 0; j < R0; ++j) v[j] = src.load(line, b + j * R1);
                    Dft<R0, SIGN>::run(v);
#pragma unroll
                    for (int j = 0; j < R0; ++j) xc.at(line, j, b) = v[j];
                }
            }
        }
    }

    // `mid` runs (in every thread) after the barrier that ends stage 1, i.e. once the
    // source has been fully consumed: persistent kernels prefetch their next input there.
    template <bool IN_PLACE = false, class Src, class Xc, class Dst, class Mid = NoMid,
              class AfterLoads = NoMid>
    static __device__ __forceinline__ void run(const Src& src, const Xc& xc, Dst& dst,
                                               const C* __restrict__ tw2,
                                               const Mid& mid = Mid(),
                                               const AfterLoads& after_loads = AfterLoads()) {
        stage1<IN_PLACE>(src, xc, after_loads);
        Grp::sync();
        mid();
        {   // stage 2: radix R1 over R0 butterflies per line, exchange -> destination
            constexpr int TOTAL = L * R0;
            constexpr int ITER = (TOTAL + T - 1) / T;
            // not unrolled: one copy of the (large) butterfly + epilogue keeps the kernel
            // inside the instruction cache
#pragma unroll 1
            for (int it = 0; it < ITER; ++it) {
                const int g = Grp::tid() + it * T;
                if (TOTAL % T == 0 || g < TOTAL) {
                    int line, b;
                    Map::template map<R0, L>(g, line, b);
                    C v[R1];
#pragma unroll
                    for (int j = 0; j < R1; ++j) v[j] = xc.at(line, b, j);
                    const C* tw = tw2 + b * (R1 - 1);
#pragma unroll
                    for (int j = 1; j < R1; ++j) {
                        const C w = TW_SMEM ? tw[j - 1] : __ldg(tw + (j - 1));
                        v[j] = SIGN < 0 ? cmul(v[j], w) : cmulc(v[j], w);
                    }
                    Dft<R1, SIGN>::run(v);
                    store_butterfly<R1, R0>(dst, line, b, v);
                }
            }
        }
    }
};

}  // namespace stitch
