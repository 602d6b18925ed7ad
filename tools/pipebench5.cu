// pipebench5.cu — FFMA2 issue rate of the "input PAIR x broadcast WEIGHT"
// forms (tuning tool for conv_tb.cuh): the pair (x_j, x_j+1) in a vector
// register pair times one weight broadcast from a uniform register (pw_ur) or
// from a vector register (pw_r), and with one input pair shared by several
// accumulators (the stencil's reuse, pw_ur_sh).  Reference: the round-1
// form "broadcast input x uniform weight pair" (bc_ur).  8 chains per
// thread, 16 warps per SM.  Rates are warp instructions.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int ITERS = 8192, CH = 8;
struct Wt { float w[CH]; float2 wp[CH]; };
typedef unsigned long long u64;
__device__ __forceinline__ u64 pk(float2 f) { return *reinterpret_cast<u64*>(&f); }
__device__ __forceinline__ void f2_pw(u64& a, u64 x, float w) {
    asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%2, %2};\n\tfma.rn.f32x2 %0, %1, t, %0;\n\t}" : "+l"(a) : "l"(x), "f"(w));
}
__device__ __forceinline__ void f2_bc(u64& a, float x, u64 w) {
    asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%1, %1};\n\tfma.rn.f32x2 %0, t, %2, %0;\n\t}" : "+l"(a) : "f"(x), "l"(w));
}
__global__ void k_bc_ur(float* out, float s, const __grid_constant__ Wt wt) {
    u64 a[CH]; float x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = pk(make_float2(threadIdx.x + c, c)); x[c] = s * c + threadIdx.x; }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) f2_bc(a[c], x[c], pk(wt.wp[c]));
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_pw_ur(float* out, float s, const __grid_constant__ Wt wt) {
    u64 a[CH], x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = pk(make_float2(threadIdx.x + c, c)); x[c] = pk(make_float2(s * c + threadIdx.x, s - c)); }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) f2_pw(a[c], x[c], wt.w[c]);
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_pw_r(float* out, float s) {
    u64 a[CH], x[CH]; float w[CH];
    for (int c = 0; c < CH; ++c) {
        a[c] = pk(make_float2(threadIdx.x + c, c)); x[c] = pk(make_float2(s * c + threadIdx.x, s - c));
        w[c] = s + c * 0.001f + threadIdx.x * 1e-6f;
    }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) f2_pw(a[c], x[c], w[c]);
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
// the stencil's pattern: 2 input pairs, each feeding 4 accumulators with 4 weights
__global__ void k_pw_ur_sh(float* out, float s, const __grid_constant__ Wt wt) {
    u64 a[CH], x0 = pk(make_float2(s + threadIdx.x, s)), x1 = pk(make_float2(s - threadIdx.x, s + 1));
    for (int c = 0; c < CH; ++c) a[c] = pk(make_float2(threadIdx.x + c, c));
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int c = 0; c < CH; ++c) f2_pw(a[c], c < CH / 2 ? x0 : x1, wt.w[c % (CH / 2)]);
        x0 += 0x100000001ull; x1 += 0x100000001ull;
    }
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out; cudaMalloc(&out, sms * 512 * 4 * 4);
    Wt wt;
    for (int i = 0; i < CH; ++i) { wt.w[i] = 0.999f + i * 1e-4f; wt.wp[i] = make_float2(0.999f + i * 1e-4f, 0.998f - i * 1e-4f); }
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char* nm, auto launch) {
        launch(); cudaDeviceSynchronize(); cudaEventRecord(e0);
        for (int r = 0; r < 10; ++r) launch();
        cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
        double wi = 10.0 * sms * 16 * (double)ITERS * CH;
        printf("%-12s %.3f warp-instr/clk/SM at %d MHz nominal (%.2f ms) %s\n", nm, wi / (ms * 1e-3 * clk * 1e3) / sms, clk / 1000, ms, cudaGetErrorString(cudaGetLastError()));
    };
    run("bc_ur", [&] { k_bc_ur<<<sms, 512>>>(out, 1.0001f, wt); });
    run("pw_ur", [&] { k_pw_ur<<<sms, 512>>>(out, 1.0001f, wt); });
    run("pw_r", [&] { k_pw_r<<<sms, 512>>>(out, 1.0001f); });
    run("pw_ur_sh", [&] { k_pw_ur_sh<<<sms, 512>>>(out, 1.0001f, wt); });
    return 0;
}
