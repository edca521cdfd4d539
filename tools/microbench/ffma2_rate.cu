// Throughput of Blackwell's packed fp32 (FFMA2 / FADD2) against scalar FFMA / FADD on sm_100a:
// independent chains per thread, enough warps to saturate; prints warp-instructions and fp32
// lane-operations per cycle per SM for each form.  nvcc -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long pk(float2 a) { return *reinterpret_cast<unsigned long long*>(&a); }
__device__ __forceinline__ float2 up(unsigned long long r) { return *reinterpret_cast<float2*>(&r); }
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
    unsigned long long d;
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(pk(a)), "l"(pk(b)), "l"(pk(c)));
    return up(d);
}
__device__ __forceinline__ float2 fadd2(float2 a, float2 b) {
    unsigned long long d;
    asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(pk(a)), "l"(pk(b)));
    return up(d);
}
constexpr int CH = 8, IT = 4096;

template <int MODE>
__global__ void bench(float2* out, float s) {
    float2 x[CH], y = make_float2(s, 1.f - s), z = make_float2(0.5f * s, s * s);
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c * 0.5f);
    for (int i = 0; i < IT; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c) {
            if constexpr (MODE == 0) {          // FFMA, 3 registers (two per complex)
                x[c].x = fmaf(x[c].x, y.x, z.x);
                x[c].y = fmaf(x[c].y, y.y, z.y);
            } else if constexpr (MODE == 1) {   // FFMA, immediate multiplier
                x[c].x = fmaf(x[c].x, 0.99991f, z.x);
                x[c].y = fmaf(x[c].y, 0.99993f, z.y);
            } else if constexpr (MODE == 2) {   // FFMA2, 3 registers
                x[c] = ffma2(x[c], y, z);
            } else if constexpr (MODE == 3) {   // FFMA2, broadcast scalar constant
                x[c] = ffma2(x[c], make_float2(0.99991f, 0.99991f), z);
            } else if constexpr (MODE == 4) {   // FADD2
                x[c] = fadd2(x[c], z);
            } else if constexpr (MODE == 5) {   // FADD x2
                x[c].x = x[c].x + z.x;
                x[c].y = x[c].y + z.y;
            } else if constexpr (MODE == 6) {   // one FFMA2 (chain c) + one scalar FFMA (chain c+CH/2)
                if (c < CH / 2) x[c] = ffma2(x[c], y, z);
                else x[c].x = fmaf(x[c].x, y.x, z.x);
            } else {                            // two FFMA2 + one scalar FFMA per 3 chains
                if (c % 3 != 2) x[c] = ffma2(x[c], y, z);
                else x[c].x = fmaf(x[c].x, y.x, z.x);
            }
        }
    }
    float2 acc = make_float2(0.f, 0.f);
#pragma unroll
    for (int c = 0; c < CH; ++c) acc = make_float2(acc.x + x[c].x, acc.y + x[c].y);
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int MODE>
void run(const char* name, float2* out, int sms, int clk_khz) {
    const int blocks = sms * 4, threads = 512;
    bench<MODE><<<blocks, threads>>>(out, 0.5f);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    bench<MODE><<<blocks, threads>>>(out, 0.5f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const bool packed = MODE == 2 || MODE == 3 || MODE == 4;
    // lane operations and warp instructions per chain-iteration (per thread)
    double ops = CH * 2.0, inst = packed ? CH : 2.0 * CH;
    if (MODE == 6) { ops = CH / 2 * 2.0 + CH / 2 * 1.0; inst = CH; }
    if (MODE == 7) { int p2 = 0, p1 = 0; for (int c = 0; c < CH; ++c) (c % 3 != 2 ? p2 : p1)++;
                     ops = p2 * 2.0 + p1; inst = p2 + p1; }
    const double lane_ops = (double)blocks * threads * IT * ops;
    const double warp_inst = (double)blocks * threads / 32 * IT * inst;
    const double cyc = ms * 1e-3 * clk_khz * 1e3;
    printf("%-24s %8.3f ms  %6.2f warp-inst/clk/SM  %7.1f fp32 lane-ops/clk/SM\n", name, ms,
           warp_inst / cyc / sms, lane_ops / cyc / sms);
}

int main() {
    int sms, clk;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float2* out;
    cudaMalloc(&out, sizeof(float2) * sms * 4 * 512);
    printf("SMs %d, clock %d MHz (max; the rates assume it)\n", sms, clk / 1000);
    run<0>("FFMA 3-reg", out, sms, clk);
    run<1>("FFMA imm", out, sms, clk);
    run<2>("FFMA2 3-reg", out, sms, clk);
    run<3>("FFMA2 bcast const", out, sms, clk);
    run<4>("FADD2", out, sms, clk);
    run<5>("FADD", out, sms, clk);
    run<6>("FFMA2 + FFMA (1:1)", out, sms, clk);
    run<7>("FFMA2 + FFMA (2:1)", out, sms, clk);
    return 0;
}
