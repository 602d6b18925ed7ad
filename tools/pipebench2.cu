// pipebench2.cu — FFMA issue rate by operand form (tuning tool): R,R,R vs
// R,imm,R vs R,UR,R, 8 independent chains per thread, 16 warps per SM.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int ITERS = 8192, CH = 8;
struct Wt { float w[8]; };
__global__ void k_rrr(float* out, float s) {
    float a[CH], x[CH], w[CH];
    for (int c = 0; c < CH; ++c) { a[c] = threadIdx.x + c; x[c] = s * c + threadIdx.x; w[c] = s + c * 0.001f; }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(a[c]) : "f"(x[c]), "f"(w[c]));
    float t = 0; for (int c = 0; c < CH; ++c) t += a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_imm(float* out, float s) {
    float a[CH], x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = threadIdx.x + c; x[c] = s * c + threadIdx.x; }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) asm volatile("fma.rn.f32 %0, %1, 0f3F7FF972, %0;" : "+f"(a[c]) : "f"(x[c]));
    float t = 0; for (int c = 0; c < CH; ++c) t += a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_ur(float* out, float s, const __grid_constant__ Wt wt) {
    float a[CH], x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = threadIdx.x + c; x[c] = s * c + threadIdx.x; }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(a[c]) : "f"(x[c]), "f"(wt.w[c]));
    float t = 0; for (int c = 0; c < CH; ++c) t += a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
// FFMA2 (fma.rn.f32x2, sm_100a): two fp32 FMAs per lane per instruction.
// rr: all operands register pairs; bc: the weight a broadcast scalar (UR).
__global__ void k_f2rr(float* out, float s) {
    unsigned long long a[CH], x[CH], w[CH];
    for (int c = 0; c < CH; ++c) {
        float2 fa = make_float2(threadIdx.x + c, c), fx = make_float2(s * c + threadIdx.x, s), fw = make_float2(s + c * 0.001f, s);
        a[c] = *reinterpret_cast<unsigned long long*>(&fa); x[c] = *reinterpret_cast<unsigned long long*>(&fx);
        w[c] = *reinterpret_cast<unsigned long long*>(&fw);
    }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(a[c]) : "l"(x[c]), "l"(w[c]));
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_f2bc(float* out, float s, const __grid_constant__ Wt wt) {
    unsigned long long a[CH], x[CH];
    for (int c = 0; c < CH; ++c) {
        float2 fa = make_float2(threadIdx.x + c, c), fx = make_float2(s * c + threadIdx.x, s);
        a[c] = *reinterpret_cast<unsigned long long*>(&fa); x[c] = *reinterpret_cast<unsigned long long*>(&fx);
    }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) {
            float2 wv = make_float2(wt.w[c], wt.w[c]);
            unsigned long long W = *reinterpret_cast<unsigned long long*>(&wv);
            asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(a[c]) : "l"(x[c]), "l"(W));
        }
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
int main() {
    int sms, clk; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0); cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out; cudaMalloc(&out, sms * 512 * 4 * 4);
    Wt wt; for (int i = 0; i < 8; ++i) wt.w[i] = 0.999f + i * 1e-4f;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char* nm, auto launch) {
        launch(); cudaDeviceSynchronize(); cudaEventRecord(e0);
        for (int r = 0; r < 10; ++r) launch();
        cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
        double wi = 10.0 * sms * 16 * (double)ITERS * CH;
        printf("%-6s %.3f warp-FFMA/clk/SM at %d MHz nominal (%.2f ms) %s\n", nm, wi / (ms * 1e-3 * clk * 1e3) / sms, clk / 1000, ms, cudaGetErrorString(cudaGetLastError()));
    };
    run("rrr", [&] { k_rrr<<<sms, 512>>>(out, 1.0001f); });
    run("imm", [&] { k_imm<<<sms, 512>>>(out, 1.0001f); });
    run("f2rr", [&] { k_f2rr<<<sms, 512>>>(out, 1.0001f); });   // x2: each instruction is 2 FMAs per lane
    run("f2bc", [&] { k_f2bc<<<sms, 512>>>(out, 1.0001f, wt); });
    run("ur", [&] { k_ur<<<sms, 512>>>(out, 1.0001f, wt); });
    return 0;
}
