// runtime.h — internals shared by the host runtime's translation units
// (api.cpp: grids, iteration, exchange, chained tasks; unmodified.cpp:
// unmodified routines).  Not part of the C ABI.
#pragma once
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdint>
#include <vector>

#include "mapsm.h"
#include "nccl.h"

namespace mapsm {
mapsm_status compute_plan(int64_t h, int g, int r, mapsm_boundary b, int rank, mapsm_slab_plan* out);
// The ordered halo-exchange messages of one pass (plan.cpp; <= 4); returns the count.
int exchange_messages(const mapsm_slab_plan& p, int64_t h, int64_t depth, int64_t halo, int64_t pitch,
                      mapsm_msg* out);

// Records a thread-local error message (mapsm_last_error) and returns s.
mapsm_status fail(mapsm_status s, const char* fmt, ...);

// Restores the caller's current device on scope exit (torch relies on it).
struct DeviceGuard {
    int prev = -1;
    DeviceGuard() { cudaGetDevice(&prev); }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

// NCCL, loaded on first use with dlopen("libnccl.so.2"): inside a torch
// process this resolves to the NCCL torch already loaded (one per process).
struct NcclApi {
    void* h = nullptr;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclCommAbort) commAbort = nullptr;
    decltype(&ncclCommGetAsyncError) commGetAsyncError = nullptr;
    decltype(&ncclSend) send = nullptr;
    decltype(&ncclRecv) recv = nullptr;
    decltype(&ncclGroupStart) groupStart = nullptr;
    decltype(&ncclGroupEnd) groupEnd = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclGetErrorString) errStr = nullptr;
};
extern NcclApi g_nccl;
mapsm_status nccl_load();
}  // namespace mapsm

struct mapsm_ctx_s;
// Releases the unmodified-routine state of a context (unmodified.cpp).
void blas_release(mapsm_ctx_s* c);

#define CK(expr)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (expr);                                                              \
        if (e_ != cudaSuccess)                                                                \
            return ::mapsm::fail(e_ == cudaErrorMemoryAllocation ? MAPSM_ENOMEM : MAPSM_ECUDA, \
                                 "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

#define TRY(expr)                          \
    do {                                   \
        mapsm_status s_ = (expr);          \
        if (s_ != MAPSM_OK) return s_;     \
    } while (0)

#define NK(expr)                                                                              \
    do {                                                                                      \
        ncclResult_t r_ = (expr);                                                             \
        if (r_ != ncclSuccess)                                                                \
            return ::mapsm::fail(MAPSM_ENCCL, "%s failed: %s", #expr, ::mapsm::g_nccl.errStr(r_)); \
    } while (0)

// One context per process (rank) or one per single-process multi-slab run.
struct mapsm_ctx_s {
    bool local = false;            // single-process multi-slab mode
    int rank = 0, world = 1;       // process rank / count (multi-process mode)
    int g = 1;                     // total slabs
    int first_slab = 0;            // global index of local slab 0
    std::vector<int> devices;      // device per local slab
    cudaStream_t user_stream = nullptr;
    ncclComm_t comm = nullptr;
    int live_grids = 0;
    void* blas = nullptr;          // unmodified-routine state (unmodified.cpp), created on first use
    // FIFO order of the host<->device transfers of the ctx's own-stream grids
    // (api.cpp xfer_begin / xfer_end): the transfer issued first completes
    // first, instead of all in-flight uploads sharing the copy engine.
    cudaEvent_t ev_h2d = nullptr, ev_d2h = nullptr;
};
