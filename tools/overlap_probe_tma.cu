// overlap_probe_tma.cu — as overlap_probe.cu, but the bandwidth grid moves its
// rows with TMA bulk copies through an mbarrier ring (the structure of the
// Life interior kernel): global -> shared (cp.async.bulk + mbarrier), then
// shared -> global (cp.async.bulk store), 146 CTAs.  Side ops on another
// stream: sys / gpu fences, NCCL self send/recv.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/opt tools/overlap_probe_tma.cu -lnccl
#include <cuda_runtime.h>
#include <nccl.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>

#ifndef PROBE_NS
#define PROBE_NS 16
#endif
constexpr int NS = PROBE_NS, ROW = 8192;  // stages x bytes

__device__ __forceinline__ void mbar_init(uint64_t* b, int n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(n));
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, unsigned tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned ph) {
    asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W; }"
                 ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(ph) : "memory");
}

__global__ void tma_copy(const char* a, char* b, size_t nrows) {
    extern __shared__ __align__(128) char sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + NS * ROW);
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) mbar_init(&full[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    size_t r0 = blockIdx.x * nrows / gridDim.x, r1 = (blockIdx.x + 1) * nrows / gridDim.x;
    unsigned ph[NS] = {};
    size_t issued = r0;
    for (; issued < r1 && issued < r0 + NS; ++issued) {
        int s = (issued - r0) % NS;
        mbar_expect(&full[s], ROW);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"((unsigned)__cvta_generic_to_shared(sm + s * ROW)), "l"(a + issued * ROW), "r"(ROW),
                       "r"((unsigned)__cvta_generic_to_shared(&full[s])) : "memory");
    }
    for (size_t r = r0; r < r1; ++r) {
        int s = (r - r0) % NS;
        mbar_wait(&full[s], ph[s]);
        ph[s] ^= 1;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                     ::"l"(b + r * ROW), "r"((unsigned)__cvta_generic_to_shared(sm + s * ROW)), "r"(ROW) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        if (issued < r1) {
            asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(NS - 1) : "memory");
            int s2 = (issued - r0) % NS;
            mbar_expect(&full[s2], ROW);
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"((unsigned)__cvta_generic_to_shared(sm + s2 * ROW)), "l"(a + issued * ROW), "r"(ROW),
                           "r"((unsigned)__cvta_generic_to_shared(&full[s2])) : "memory");
            ++issued;
        }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// TMA loads into the ring; 16 consumer warps copy each stage to global memory
// with 16-byte st.global (the Life interior's store path), 544 threads.
__global__ void tma_ld_st(const char* a, char* b, size_t nrows) {
    extern __shared__ __align__(128) char sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + NS * ROW);
    uint64_t* empty = full + NS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 16); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    size_t r0 = blockIdx.x * nrows / gridDim.x, r1 = (blockIdx.x + 1) * nrows / gridDim.x;
    if (warp == 16) {
        if (lane == 0)
            for (size_t r = r0; r < r1; ++r) {
                int s = (r - r0) % NS; unsigned ph = ((r - r0) / NS) & 1;
                if (r - r0 >= NS) mbar_wait(&empty[s], ph ^ 1);
                mbar_expect(&full[s], ROW);
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"((unsigned)__cvta_generic_to_shared(sm + s * ROW)), "l"(a + r * ROW), "r"(ROW),
                               "r"((unsigned)__cvta_generic_to_shared(&full[s])) : "memory");
            }
        return;
    }
    for (size_t r = r0; r < r1; ++r) {
        int s = (r - r0) % NS; unsigned ph = ((r - r0) / NS) & 1;
        mbar_wait(&full[s], ph);
        const uint4 v = reinterpret_cast<const uint4*>(sm + s * ROW)[warp * 32 + lane];
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((unsigned)__cvta_generic_to_shared(&empty[s])) : "memory");
        reinterpret_cast<uint4*>(b + r * ROW)[warp * 32 + lane] = v;
    }
}

__global__ void side(int mode, long long ns, unsigned int* flag) {
    long long t0 = clock64();
    const long long cyc = ns * 19 / 10;
    unsigned v = 0;
    while (clock64() - t0 < cyc) {
        if (mode == 1) __threadfence_system();
        if (mode == 2) __threadfence();
        if (mode == 3) asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    }
    if (v == 7777777) flag[1] = 1;
}

int main(int argc, char** argv) {
    const size_t bytes = (argc > 1 ? (size_t)atoll(argv[1]) : 64ull) << 20;
    char *a, *b, *s0, *s1;
    unsigned* flag;
    cudaMalloc(&a, bytes); cudaMalloc(&b, bytes); cudaMalloc(&s0, 1 << 20); cudaMalloc(&s1, 1 << 20);
    cudaMalloc(&flag, 64); cudaMemset(flag, 0, 64); cudaMemset(a, 1, bytes);
    const int smem = NS * ROW + NS * 8;
    cudaFuncSetAttribute(tma_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(tma_ld_st, cudaFuncAttributeMaxDynamicSharedMemorySize, smem + NS * 8);
    cudaStream_t m, s;
    cudaStreamCreateWithFlags(&m, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    ncclComm_t comm;
    if (argc > 2) {  // as the library: a one-rank communicator from a unique id (bootstrap + proxy thread)
        ncclUniqueId id;
        ncclGetUniqueId(&id);
        ncclCommInitRank(&comm, 1, id, 0);
    } else {
        int dev0 = 0;
        ncclCommInitAll(&comm, 1, &dev0);
    }
    cudaEvent_t e0, e1, go;
    cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventCreateWithFlags(&go, cudaEventDisableTiming);
    const char* names[] = {"none", "spin+threadfence_system", "spin+threadfence(gpu)", "spin+ld.acquire.sys",
                           "NCCL self send/recv 2x8KB", "spin only", "2-CTA ring kernel, then NCCL",
                           "2-CTA ring kernel only"};
    printf("%s grid, working set 2 x %zu MiB\n", getenv("PROBE_LDST") ? "TMA-load / st.global" : "TMA", bytes >> 20);
    for (int mode = 0; mode <= 7; ++mode) {
        float tot = 0;
        const int reps = 40;
        for (int r = 0; r < reps + 5; ++r) {
            cudaEventRecord(go, m);
            cudaStreamWaitEvent(s, go, 0);
            cudaEventRecord(e0, m);
            if (getenv("PROBE_LDST"))
                tma_ld_st<<<146, 544, smem + NS * 8, m>>>(a, b, bytes / ROW);
            else
                tma_copy<<<146, 32, smem, m>>>(a, b, bytes / ROW);
            if (mode >= 1 && mode <= 3) side<<<1, 128, 0, s>>>(mode, 10000, flag);
            if (mode == 5) side<<<1, 128, 0, s>>>(0, 10000, flag);
            if (mode == 7) tma_ld_st<<<2, 544, smem + NS * 8, s>>>(a, s1, 2);
            if (mode == 4 || mode == 6) {
                if (mode == 6) tma_ld_st<<<2, 544, smem + NS * 8, s>>>(a, s1, 2);  // a 2-row "boundary" launch first
                ncclGroupStart();
                ncclSend(s0, 8192, ncclUint8, 0, comm, s); ncclSend(s0 + 8192, 8192, ncclUint8, 0, comm, s);
                ncclRecv(s1, 8192, ncclUint8, 0, comm, s); ncclRecv(s1 + 8192, 8192, ncclUint8, 0, comm, s);
                ncclGroupEnd();
            }
            cudaEventRecord(e1, m);
            cudaStreamSynchronize(m); cudaStreamSynchronize(s);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 5) tot += ms;
        }
        printf("%-28s TMA grid %.2f us\n", names[mode], tot / reps * 1e3);
    }
    printf("status %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
