// pipebench3.cu — FFMA2 issue rate for the stencil operand forms (tuning tool):
// broadcast scalar input x weight pair from a uniform register (bcur, the
// conv3d form) vs from a vector register pair (bcr, what ptxas emits once the
// weight pairs outgrow the 63 uniform registers); scalar FFMA forms for scale.
// 8 independent chains per thread, 16 warps per SM.  Rates are instructions.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int ITERS = 8192, CH = 8;
struct Wt { float2 w[CH]; };
__device__ __forceinline__ unsigned long long u64(float2 f) { return *reinterpret_cast<unsigned long long*>(&f); }
__global__ void k_bcur(float* out, float s, const __grid_constant__ Wt wt) {
    unsigned long long a[CH]; float x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = u64(make_float2(threadIdx.x + c, c)); x[c] = s * c + threadIdx.x; }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c)
            asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%1, %1};\n\tfma.rn.f32x2 %0, t, %2, %0;\n\t}" : "+l"(a[c]) : "f"(x[c]), "l"(u64(wt.w[c])));
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_bcr(float* out, float s) {
    unsigned long long a[CH], w[CH]; float x[CH];
    for (int c = 0; c < CH; ++c) {
        a[c] = u64(make_float2(threadIdx.x + c, c)); x[c] = s * c + threadIdx.x;
        w[c] = u64(make_float2(s + c * 0.001f + threadIdx.x * 1e-6f, s - c * 0.001f));
    }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c)
            asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%1, %1};\n\tfma.rn.f32x2 %0, t, %2, %0;\n\t}" : "+l"(a[c]) : "f"(x[c]), "l"(w[c]));
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
// shared input across chains (the stencil's reuse: one value, several accumulators)
__global__ void k_bcur_shared(float* out, float s, const __grid_constant__ Wt wt) {
    unsigned long long a[CH]; float x = s + threadIdx.x;
    for (int c = 0; c < CH; ++c) a[c] = u64(make_float2(threadIdx.x + c, c));
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int c = 0; c < CH; ++c)
            asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%1, %1};\n\tfma.rn.f32x2 %0, t, %2, %0;\n\t}" : "+l"(a[c]) : "f"(x), "l"(u64(wt.w[c])));
        x += 1.0f;
    }
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
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
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out; cudaMalloc(&out, sms * 512 * 4 * 4);
    Wt wt; for (int i = 0; i < CH; ++i) wt.w[i] = make_float2(0.999f + i * 1e-4f, 0.998f - i * 1e-4f);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char* nm, auto launch) {
        launch(); cudaDeviceSynchronize(); cudaEventRecord(e0);
        for (int r = 0; r < 10; ++r) launch();
        cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
        double wi = 10.0 * sms * 16 * (double)ITERS * CH;
        printf("%-12s %.3f warp-instr/clk/SM at %d MHz nominal (%.2f ms) %s\n", nm, wi / (ms * 1e-3 * clk * 1e3) / sms, clk / 1000, ms, cudaGetErrorString(cudaGetLastError()));
    };
    run("rrr", [&] { k_rrr<<<sms, 512>>>(out, 1.0001f); });
    run("f2_bc_ur", [&] { k_bcur<<<sms, 512>>>(out, 1.0001f, wt); });
    run("f2_bc_r", [&] { k_bcr<<<sms, 512>>>(out, 1.0001f); });
    run("f2_bc_ur_sh", [&] { k_bcur_shared<<<sms, 512>>>(out, 1.0001f, wt); });
    return 0;
}
