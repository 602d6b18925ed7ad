// atomsbench.cu — shared-memory atomic issue cap of the histogram kernel's
// access pattern: [bin][lane] table (lane l -> bank l, one wavefront per
// warp-instruction), pseudo-random bins; vs a non-atomic LDS+STS
// read-modify-write of a per-warp private table.  Rates per SM.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int N = 4096;
__global__ void __launch_bounds__(256) k_atoms(unsigned* out, unsigned seed) {
    __shared__ unsigned sh[256][32];
    for (int i = threadIdx.x; i < 256 * 32; i += 256) (&sh[0][0])[i] = 0;
    __syncthreads();
    const unsigned lane = threadIdx.x & 31;
    unsigned x = seed ^ (threadIdx.x * 2654435761u) ^ (blockIdx.x * 40503u);
#pragma unroll 16
    for (int i = 0; i < N; ++i) {
        x = x * 1664525u + 1013904223u;
        atomicAdd(&sh[x >> 24][lane], 1u);
    }
    __syncthreads();
    out[blockIdx.x * 256 + threadIdx.x] = sh[threadIdx.x][lane];
}
__global__ void __launch_bounds__(256) k_rmw(unsigned* out, unsigned seed) {
    extern __shared__ unsigned short shd[];  // [8 warps][256 bins][32 lanes]: private counters
    unsigned short (*sh)[256][32] = reinterpret_cast<unsigned short (*)[256][32]>(shd);
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 8 * 256 * 32; i += 256) shd[i] = 0;
    __syncthreads();
    const unsigned lane = threadIdx.x & 31;
    unsigned x = seed ^ (threadIdx.x * 2654435761u) ^ (blockIdx.x * 40503u);
#pragma unroll 16
    for (int i = 0; i < N; ++i) {
        x = x * 1664525u + 1013904223u;
        unsigned short* p = &sh[warp][x >> 24][lane];
        *p = *p + 1;
    }
    __syncthreads();
    out[blockIdx.x * 256 + threadIdx.x] = sh[warp][threadIdx.x][lane];
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    unsigned* out; cudaMalloc(&out, sms * 16 * 256 * 4);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char* nm, int ctas_per_sm, auto launch) {
        launch(sms * ctas_per_sm); cudaDeviceSynchronize(); cudaEventRecord(e0);
        for (int r = 0; r < 5; ++r) launch(sms * ctas_per_sm);
        cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
        double wi = 5.0 * ctas_per_sm * 8 * (double)N;  // warp-ops per SM
        printf("%-8s %d CTA/SM: %.3f warp-ops/clk/SM = %.2f clk per warp-op (%.3f ms) %s\n", nm, ctas_per_sm,
               wi / (ms * 1e-3 * clk * 1e3), (ms * 1e-3 * clk * 1e3) / wi, ms, cudaGetErrorString(cudaGetLastError()));
    };
    for (int c : {2, 4, 6})
        run("atoms", c, [&](int g) { k_atoms<<<g, 256>>>(out, 7u); });
    cudaFuncSetAttribute(k_rmw, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072);
    for (int c : {1})
        run("lds+sts", c, [&](int g) { k_rmw<<<g, 256, 131072>>>(out, 7u); });
    return 0;
}
