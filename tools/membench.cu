// membench.cu — HBM access-pattern microbenchmarks for the Life kernel design
// (tuning tool, not part of the library).  All variants copy a 65536 x 8192 B
// (512 MiB) "slab" to a second buffer, i.e. exactly the traffic of one Life
// generation at 65536^2, with different access structures:
//   0 flat     : grid-stride uint4 copy (the shape of torch's copy)
//   1 strips   : each warp streams a 512 B-wide strip down a chunk of rows (LDG/STG)
//   2 strips+P : same with P rows of loads in flight per lane
//   3 tma      : producer/consumer cp.async.bulk ring, NC warps x 512 B strip, NS stages
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o membench membench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

constexpr int64_t ROWS = 65536, PITCH = 8192, PW = PITCH / 4;

__global__ void flat_copy(const uint4* __restrict__ a, uint4* __restrict__ b, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = __ldg(a + i);
}

template <int P>
__global__ void strip_copy(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, int64_t nchunks) {
    const int lane = threadIdx.x & 31;
    const int64_t wg = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
    const int64_t strips = PW / 128;
    const int64_t strip = wg % strips, chunk = wg / strips;
    if (chunk >= nchunks) return;
    const int64_t ys = chunk * ROWS / nchunks, ye = (chunk + 1) * ROWS / nchunks;
    const uint32_t* ip = in + ys * PW + strip * 128 + lane * 4;
    uint32_t* op = out + ys * PW + strip * 128 + lane * 4;
    uint4 ring[P];
#pragma unroll
    for (int k = 0; k < P; ++k) ring[k] = __ldg(reinterpret_cast<const uint4*>(ip + (ys + k < ye ? k : 0) * PW));
    int64_t y = ys;
    for (; y + 2 * P <= ye; y += P) {
#pragma unroll
        for (int k = 0; k < P; ++k) {
            uint4 v = ring[k];
            ring[k] = __ldg(reinterpret_cast<const uint4*>(ip + (y - ys + k + P) * PW));
            *reinterpret_cast<uint4*>(op + (y - ys + k) * PW) = v;
        }
    }
    for (; y < ye; ++y) *reinterpret_cast<uint4*>(op + (y - ys) * PW) = __ldg(reinterpret_cast<const uint4*>(ip + (y - ys) * PW));
}

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int NC, int NS>
__global__ void __launch_bounds__((NC + 1) * 32) tma_copy(const uint32_t* __restrict__ in, uint32_t* __restrict__ out,
                                                         int64_t nchunks) {
    extern __shared__ __align__(128) uint8_t smem[];
    constexpr int SB = NC * 512;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * SB);
    uint64_t* empty = full + NS;
    const int64_t strips = PITCH / SB;
    const int64_t strip = blockIdx.x % strips, chunk = blockIdx.x / strips;
    const int64_t ys = chunk * ROWS / nchunks, ye = (chunk + 1) * ROWS / nchunks;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(&empty[s])), "r"(NC));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int n = (int)(ye - ys);
    if (warp == NC) {
        if (lane == 0) {
            for (int i = 0; i < n; ++i) {
                const int s = i % NS;
                if (i >= NS) {
                    uint32_t ok = 0;
                    do {
                        asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                                     : "=r"(ok) : "r"(sa(&empty[s])), "r"((uint32_t)(((i / NS) + 1) & 1)) : "memory");
                    } while (!ok);
                }
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&full[s])), "r"(SB) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                                 sa(smem + s * SB)), "l"(in + (ys + i) * PW + strip * (SB / 4)), "r"(SB), "r"(sa(&full[s]))
                             : "memory");
            }
        }
        return;
    }
    uint32_t* op = out + ys * PW + strip * (SB / 4) + (warp * 32 + lane) * 4;
    for (int i = 0; i < n; ++i) {
        const int s = i % NS;
        uint32_t ok = 0;
        do {
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(sa(&full[s])), "r"((uint32_t)((i / NS) & 1)) : "memory");
        } while (!ok);
        uint4 v = *reinterpret_cast<const uint4*>(smem + s * SB + (warp * 32 + lane) * 16);
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(&empty[s])) : "memory");
        *reinterpret_cast<uint4*>(op + (int64_t)i * PW) = v;
    }
}

template <class F>
float timeit(F f, int reps = 20) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f();
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    for (int i = 0; i < reps; ++i) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / reps;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t bytes = ROWS * PITCH;
    uint32_t *a, *b;
    CK(cudaMalloc(&a, bytes));
    CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(a, 1, bytes));
    auto report = [&](const char* name, float ms) {
        printf("%-28s %8.3f us  %7.1f GB/s (read+write)\n", name, ms * 1e3, 2.0 * bytes / (ms * 1e-3) / 1e9);
    };
    for (int bpsm : {2, 4, 8}) {
        char nm[64];
        snprintf(nm, 64, "flat grid=%dxSM", bpsm);
        report(nm, timeit([&] { flat_copy<<<sms * bpsm, 256>>>((const uint4*)a, (uint4*)b, bytes / 16); }));
    }
    for (int wps : {16, 32, 48, 64}) {
        int64_t warps = (int64_t)sms * wps;
        int64_t nch = warps / (PW / 128);
        char nm[64];
        snprintf(nm, 64, "strip P=1 warps/SM=%d", wps);
        report(nm, timeit([&] { strip_copy<1><<<(unsigned)((nch * 16 + 7) / 8), 256>>>(a, b, nch); }));
        snprintf(nm, 64, "strip P=4 warps/SM=%d", wps);
        report(nm, timeit([&] { strip_copy<4><<<(unsigned)((nch * 16 + 7) / 8), 256>>>(a, b, nch); }));
        snprintf(nm, 64, "strip P=8 warps/SM=%d", wps);
        report(nm, timeit([&] { strip_copy<8><<<(unsigned)((nch * 16 + 7) / 8), 256>>>(a, b, nch); }));
    }
    {
        const int smem = 12 * 4096 + 2 * 12 * 8;
        CK(cudaFuncSetAttribute(tma_copy<8, 12>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        for (int cps : {1, 2, 3, 4}) {
            int64_t nch = (int64_t)sms * cps / 2;
            char nm[64];
            snprintf(nm, 64, "tma NC=8 NS=12 cta/SM=%d", cps);
            report(nm, timeit([&] { tma_copy<8, 12><<<(unsigned)(nch * 2), 9 * 32, smem>>>(a, b, nch); }));
        }
        const int smem2 = 24 * 4096 + 2 * 24 * 8;
        CK(cudaFuncSetAttribute(tma_copy<8, 24>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        for (int cps : {1, 2}) {
            int64_t nch = (int64_t)sms * cps / 2;
            char nm[64];
            snprintf(nm, 64, "tma NC=8 NS=24 cta/SM=%d", cps);
            report(nm, timeit([&] { tma_copy<8, 24><<<(unsigned)(nch * 2), 9 * 32, smem2>>>(a, b, nch); }));
        }
        const int smem3 = 12 * 8192 + 2 * 12 * 8;
        CK(cudaFuncSetAttribute(tma_copy<16, 12>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem3));
        for (int cps : {1, 2}) {
            int64_t nch = (int64_t)sms * cps;
            char nm[64];
            snprintf(nm, 64, "tma NC=16 NS=12 cta/SM=%d", cps);
            report(nm, timeit([&] { tma_copy<16, 12><<<(unsigned)(nch), 17 * 32, smem3>>>(a, b, nch); }));
        }
    }
    CK(cudaDeviceSynchronize());
    return 0;
}
