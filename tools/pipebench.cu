// pipebench.cu — issue-rate microbenchmarks of the instruction forms the
// stencil kernels are built from (tuning tool, not part of the library).
// Each thread runs 8 independent dependency chains of one instruction form;
// the grid fills every SM with 16 warps.  Prints warp-instructions per clock
// per SM (4.0 = one per SMSP per clock).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pipebench pipebench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;
constexpr int CH = 8;

struct Wt { float w[8]; };

#define BODY(STMT)                                                  \
    _Pragma("unroll 1") for (int it = 0; it < ITERS; ++it) {        \
        _Pragma("unroll") for (int c = 0; c < CH; ++c) { STMT; }    \
    }

__global__ void k_ffma_rrr(float* out, float b, float cc) {
    float a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x + c;
    float bb = b * threadIdx.x, ccc = cc + threadIdx.x;
    BODY(asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[c]) : "f"(bb), "f"(ccc)));
    float s = 0; for (int c = 0; c < CH; ++c) s += a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// weight from the kernel parameter bank (as conv_tma_kernel does)
__global__ void k_ffma_rcr(float* out, const __grid_constant__ Wt wt) {
    float a[CH], x[CH];
    for (int c = 0; c < CH; ++c) { a[c] = threadIdx.x + c; x[c] = threadIdx.x * 0.5f + c; }
    BODY(a[c] = __fmaf_rn(wt.w[c], x[c], a[c]); x[c] = __fmaf_rn(wt.w[(c + 1) & 7], a[c], x[c]));
    float s = 0; for (int c = 0; c < CH; ++c) s += a[c] + x[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_ffma_imm(float* out) {
    float a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x + c;
    BODY(asm volatile("fma.rn.f32 %0, %0, 0f3F800001, 0f3F000000;" : "+f"(a[c])));
    float s = 0; for (int c = 0; c < CH; ++c) s += a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_lop3(uint32_t* out, uint32_t b, uint32_t cc) {
    uint32_t a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 7 + c;
    uint32_t bb = b ^ threadIdx.x, ccc = cc + threadIdx.x;
    BODY(asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[c]) : "r"(bb), "r"(ccc)));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_shf(uint32_t* out, uint32_t b) {
    uint32_t a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 7 + c;
    uint32_t bb = b ^ threadIdx.x;
    BODY(asm volatile("shf.l.wrap.b32 %0, %1, %0, 1;" : "+r"(a[c]) : "r"(bb)));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_imad(uint32_t* out, uint32_t b, uint32_t cc) {
    uint32_t a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 7 + c;
    uint32_t bb = b ^ threadIdx.x, ccc = cc + threadIdx.x;
    BODY(asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(bb), "r"(ccc)));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_imadhi(uint32_t* out, uint32_t b) {
    uint32_t a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 7 + c;
    uint32_t bb = b ^ threadIdx.x;
    BODY(asm volatile("mad.hi.u32 %0, %0, %1, %0;" : "+r"(a[c]) : "r"(bb)));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// mix: 1 LOP3 + 1 IMAD per step (both pipes)
__global__ void k_mix(uint32_t* out, uint32_t b, uint32_t cc) {
    uint32_t a[CH], d[CH];
    for (int c = 0; c < CH; ++c) { a[c] = threadIdx.x * 7 + c; d[c] = threadIdx.x * 3 + c; }
    uint32_t bb = b ^ threadIdx.x, ccc = cc + threadIdx.x;
    BODY(asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[c]) : "r"(bb), "r"(ccc));
         asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(d[c]) : "r"(bb), "r"(ccc)));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c] ^ d[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_shfl(uint32_t* out) {
    uint32_t a[CH];
    for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 7 + c;
    BODY(a[c] = __shfl_down_sync(0xffffffffu, a[c], 1));
    uint32_t s = 0; for (int c = 0; c < CH; ++c) s ^= a[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
    int sms, clk;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    void* out;
    cudaMalloc(&out, (size_t)sms * 4 * 512 * 4);
    Wt wt;
    for (int i = 0; i < 8; ++i) wt.w[i] = 0.999f + i * 1e-4f;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int threads = 512, blocks = sms;  // 16 warps per SM
    auto run = [&](const char* name, int per_step, auto launch) {
        launch();
        cudaDeviceSynchronize();
        cudaEventRecord(e0);
        for (int r = 0; r < 5; ++r) launch();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        const double warp_instr = 5.0 * blocks * (threads / 32) * (double)ITERS * CH * per_step;
        const double clocks = ms * 1e-3 * clk * 1e3;  // at the nominal max clock
        printf("%-12s %.3f warp-instr/clk/SM (%.2f ms, err=%s)\n", name, warp_instr / clocks / sms, ms,
               cudaGetErrorString(cudaGetLastError()));
    };
    run("ffma_rrr", 1, [&] { k_ffma_rrr<<<blocks, threads>>>((float*)out, 1.0001f, 0.5f); });
    run("ffma_rcr", 2, [&] { k_ffma_rcr<<<blocks, threads>>>((float*)out, wt); });
    run("ffma_imm", 1, [&] { k_ffma_imm<<<blocks, threads>>>((float*)out); });
    run("lop3", 1, [&] { k_lop3<<<blocks, threads>>>((uint32_t*)out, 3u, 5u); });
    run("shf", 1, [&] { k_shf<<<blocks, threads>>>((uint32_t*)out, 3u); });
    run("imad", 1, [&] { k_imad<<<blocks, threads>>>((uint32_t*)out, 3u, 5u); });
    run("imad_hi", 1, [&] { k_imadhi<<<blocks, threads>>>((uint32_t*)out, 3u); });
    run("lop3+imad", 2, [&] { k_mix<<<blocks, threads>>>((uint32_t*)out, 3u, 5u); });
    run("shfl", 1, [&] { k_shfl<<<blocks, threads>>>((uint32_t*)out); });
    return 0;
}
