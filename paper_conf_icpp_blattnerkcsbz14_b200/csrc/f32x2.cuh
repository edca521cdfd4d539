// f32x2.cuh -- complex fp32 arithmetic on Blackwell's packed fp32 instructions (sm_100a).
//
// A float2 (re, im) is one 64-bit register pair; add / sub / mul / fma.rn.f32x2 (PTX ISA 8.6+,
// SASS FADD2 / FMUL2 / FFMA2) do both components in one instruction.  Measured on B200
// (tools/microbench/ffma2_rate.cu): a packed instruction issues at half the rate of a scalar
// one and retires the same 128 fp32 lane-operations per clock per SM -- so the FP work of the
// FFT butterflies takes HALF the issue slots, which is what bounds the issue-bound row
// kernels.  ptxas folds the operand views below into the packed instruction's source
// selectors (no extra instructions): K(c) broadcasts a real constant or register half
// (immediate / R.F32), I(v) = i v = (-v.im, v.re) and MI(v) = -i v (swapped halves with one
// negated: R.F32x2.LO_HI.NP), NEG(v) = -v.  Every operation is correctly rounded per
// component, as the scalar FFMA / FADD / FMUL it replaces.
#pragma once
#include <cuda_runtime.h>

namespace stitch {

__device__ __forceinline__ unsigned long long f2_bits(float2 a) {
    return *reinterpret_cast<unsigned long long*>(&a);
}
__device__ __forceinline__ float2 f2_val(unsigned long long r) {
    return *reinterpret_cast<float2*>(&r);
}
__device__ __forceinline__ float2 f2add(float2 a, float2 b) {
    unsigned long long d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)));
    return f2_val(d);
}
__device__ __forceinline__ float2 f2sub(float2 a, float2 b) {
    unsigned long long d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)));
    return f2_val(d);
}
__device__ __forceinline__ float2 f2mul(float2 a, float2 b) {   // component-wise
    unsigned long long d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)));
    return f2_val(d);
}
__device__ __forceinline__ float2 f2fma(float2 a, float2 b, float2 c) {   // a * b + c
    unsigned long long d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)), "l"(f2_bits(c)));
    return f2_val(d);
}
__device__ __forceinline__ float2 K(float c) { return make_float2(c, c); }
__device__ __forceinline__ float2 I(float2 v) { return make_float2(-v.y, v.x); }
__device__ __forceinline__ float2 MI(float2 v) { return make_float2(v.y, -v.x); }
__device__ __forceinline__ float2 NEG(float2 v) { return make_float2(-v.x, -v.y); }
// complex products: a w = a w.re + (i a) w.im;  a conj(w) = a w.re - (i a) w.im
__device__ __forceinline__ float2 cmul2(float2 a, float2 w) { return f2fma(I(a), K(w.y), f2mul(a, K(w.x))); }
__device__ __forceinline__ float2 cmulc2(float2 a, float2 w) { return f2fma(MI(a), K(w.y), f2mul(a, K(w.x))); }

}  // namespace stitch
