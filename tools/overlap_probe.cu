// overlap_probe.cu — does a small kernel beside a bandwidth-bound grid slow
// the grid down, and which of its operations does it?  (the
// Life interior runs 25 us alone but 31-36 us beside a 10 us NCCL kernel.)
// A copy grid on 146 SMs streams a 2 x 64 MiB working set (the per-GPU slab
// of Life 65536^2 at N = 8, L2-assisted) while one CTA on another stream
// runs for ~10 us doing: nothing / sys-scope fences / gpu-scope fences /
// sys-scope acquire polling / small stores + sys fence; and copy-engine
// memcpys.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/op tools/overlap_probe.cu
#include <cuda_runtime.h>
#include <nccl.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>

__global__ void copy_grid(const uint4* __restrict__ a, uint4* __restrict__ b, size_t n) {
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    for (; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

__global__ void side(int mode, long long ns, unsigned int* flag, uint4* scratch) {
    long long t0 = clock64();
    const long long cyc = ns * 19 / 10;  // ~1.9 GHz
    unsigned int v = 0;
    int it = 0;
    while (clock64() - t0 < cyc) {
        switch (mode) {
            case 1: break;
            case 2: __threadfence_system(); break;
            case 3: __threadfence(); break;
            case 4: asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory"); break;
            case 5:
                scratch[(threadIdx.x + it * blockDim.x) & 1023] = make_uint4(it, v, 0, 0);
                __threadfence_system();
                break;
            case 6: asm volatile("fence.proxy.async.global;" ::: "memory"); break;
            case 7: asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(flag) : "memory"); break;
        }
        ++it;
    }
    if (v == 12345678) flag[1] = it;
}

int main(int argc, char** argv) {
    const size_t bytes = (argc > 1 ? (size_t)atoll(argv[1]) : 64ull) << 20;  // MiB per buffer
    uint4 *a, *b, *scratch;
    unsigned int* flag;
    char *s0, *s1;
    cudaMalloc(&a, bytes);
    cudaMalloc(&b, bytes);
    cudaMalloc(&scratch, 1 << 20);
    cudaMalloc(&flag, 64);
    cudaMalloc(&s0, 1 << 20);
    cudaMalloc(&s1, 1 << 20);
    cudaMemset(a, 1, bytes);
    cudaMemset(flag, 0, 64);
    cudaStream_t m, s;
    cudaStreamCreateWithFlags(&m, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t e0, e1, go;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventCreateWithFlags(&go, cudaEventDisableTiming);
    const size_t n = bytes / 16;
    const char* names[] = {"none", "spin", "spin+threadfence_system", "spin+threadfence(gpu)",
                           "spin+ld.acquire.sys", "spin+st+threadfence_system", "spin+fence.proxy.async",
                           "spin+red.release.sys", "4 x cudaMemcpyAsync 8KB D2D",
                           "NCCL self send/recv 2 x 8KB (one group)", "2 x copy kernel 8KB (1 CTA)"};
    ncclComm_t comm;
    int dev0 = 0;
    ncclCommInitAll(&comm, 1, &dev0);
    printf("working set 2 x %zu MiB%s\n", bytes >> 20, getenv("PROBE_PINGPONG") ? " (ping-pong)" : "");
    for (int mode = 0; mode <= 10; ++mode) {
        float tot = 0;
        const int reps = 40;
        for (int r = 0; r < reps + 5; ++r) {
            cudaEventRecord(go, m);
            cudaStreamWaitEvent(s, go, 0);
            cudaEventRecord(e0, m);
            if (getenv("PROBE_PINGPONG") && (r & 1))
                copy_grid<<<146, 1024, 0, m>>>(b, a, n);  // ping-pong: read what the last launch wrote
            else
                copy_grid<<<146, 1024, 0, m>>>(a, b, n);
            if (mode >= 1 && mode <= 7) side<<<1, 128, 0, s>>>(mode, 10000, flag, scratch);
            if (mode == 9) {
                ncclGroupStart();
                ncclSend(s0, 8192, ncclUint8, 0, comm, s);
                ncclSend(s0 + 8192, 8192, ncclUint8, 0, comm, s);
                ncclRecv(s1, 8192, ncclUint8, 0, comm, s);
                ncclRecv(s1 + 8192, 8192, ncclUint8, 0, comm, s);
                ncclGroupEnd();
            }
            if (mode == 10)
                for (int k = 0; k < 2; ++k)
                    copy_grid<<<1, 512, 0, s>>>(reinterpret_cast<const uint4*>(s0 + k * 8192),
                                                reinterpret_cast<uint4*>(s1 + k * 8192), 512);
            if (mode == 8)
                for (int k = 0; k < 4; ++k) cudaMemcpyAsync(s1 + k * 8192, s0 + k * 8192, 8192, cudaMemcpyDeviceToDevice, s);
            cudaEventRecord(e1, m);
            cudaStreamSynchronize(m);
            cudaStreamSynchronize(s);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 5) tot += ms;
        }
        printf("%-32s copy grid %.2f us\n", names[mode], tot / reps * 1e3);
    }
    cudaError_t e = cudaGetLastError();
    printf("status %s\n", cudaGetErrorString(e));
    return 0;
}
