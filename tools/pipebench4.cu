// pipebench4.cu — FFMA2 issue rate of the "input pair x broadcast weight" form
// (conv r >= 3, MAPSM_CONV_PAIR_MODE 2): acc(pair) += in(pair) * w(scalar),
// the weight from a uniform register (kernel parameter) or a vector register;
// 8 independent chains per thread, 16 warps per SM (and 8 warps, 2 per SMSP).
#include <cstdio>
#include <cuda_runtime.h>
constexpr int ITERS = 8192, CH = 8;
struct Ws { float w[CH]; };
__device__ __forceinline__ unsigned long long u64(float2 f) { return *reinterpret_cast<unsigned long long*>(&f); }
__device__ __forceinline__ void fp(unsigned long long& a, unsigned long long x, float w) {
    asm volatile("{\n\t.reg .b64 t;\n\tmov.b64 t, {%2, %2};\n\tfma.rn.f32x2 %0, %1, t, %0;\n\t}" : "+l"(a) : "l"(x), "f"(w));
}
__global__ void k_pair_ur(float* out, float s, const __grid_constant__ Ws wt) {
    unsigned long long a[CH], x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = u64(make_float2(threadIdx.x + c, c)); x[c] = u64(make_float2(s * c, s + threadIdx.x)); }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) fp(a[c], x[c], wt.w[c]);
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
__global__ void k_pair_r(float* out, float s) {
    unsigned long long a[CH], x[CH]; float w[CH];
    for (int c = 0; c < CH; ++c) {
        a[c] = u64(make_float2(threadIdx.x + c, c)); x[c] = u64(make_float2(s * c, s + threadIdx.x));
        w[c] = s + c * 0.001f + threadIdx.x * 1e-6f;
    }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int c = 0; c < CH; ++c) fp(a[c], x[c], w[c]);
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
// shared weight across chains (one tap, several output pairs) and shared input pair
__global__ void k_pair_r_shared_w(float* out, float s) {
    unsigned long long a[CH], x[CH]; float w = s + threadIdx.x * 1e-6f;
    for (int c = 0; c < CH; ++c) { a[c] = u64(make_float2(threadIdx.x + c, c)); x[c] = u64(make_float2(s * c, s + threadIdx.x)); }
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int c = 0; c < CH; ++c) fp(a[c], x[c], w);
        w += 1e-7f;
    }
    float t = 0; for (int c = 0; c < CH; ++c) { float2 f = *reinterpret_cast<float2*>(&a[c]); t += f.x + f.y; }
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out; cudaMalloc(&out, sms * 512 * 4 * 4);
    Ws wt; for (int i = 0; i < CH; ++i) wt.w[i] = 0.999f + i * 1e-4f;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char* nm, int thr, auto launch) {
        launch(); cudaDeviceSynchronize(); cudaEventRecord(e0);
        for (int r = 0; r < 10; ++r) launch();
        cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
        double wi = 10.0 * sms * (thr / 32) * (double)ITERS * CH;
        printf("%-16s %4d thr  %.3f warp-instr/clk/SM at %d MHz nominal (%.2f ms) %s\n", nm, thr,
               wi / (ms * 1e-3 * clk * 1e3) / sms, clk / 1000, ms, cudaGetErrorString(cudaGetLastError()));
    };
    for (int thr : {512, 256}) {
        run("pair_x_ur", thr, [&] { k_pair_ur<<<sms, thr>>>(out, 1.0001f, wt); });
        run("pair_x_r", thr, [&] { k_pair_r<<<sms, thr>>>(out, 1.0001f); });
        run("pair_x_r_sharedw", thr, [&] { k_pair_r_shared_w<<<sms, thr>>>(out, 1.0001f); });
    }
    return 0;
}
