// api.cpp — host runtime of libmapsm behind the C ABI of include/mapsm.h.
//
// Paper components (§4, Fig 1a) and what replaces them here:
//   Scheduler + Alg 1  -> mapsm_iterate: per iteration, per slab,
//       boundary-row kernel -> event -> halo exchange on a side stream, while
//       the interior kernel runs on the compute stream; the compute stream
//       waits for the exchange before the next iteration ("segment ready"
//       events, Alg 1 lines 16/20).  Iterations are captured in CUDA graphs.
//   Invoker threads        -> one process per GPU (NCCL mode) or one
//       host thread issuing to per-slab streams (local mode).
//   Memory Analyzer + Allocator     -> mapsm_window_set (plan.cpp + cudaMalloc
//       of both buffers with 2r halo rows each, once).
//   Location Monitor + Alg 2        -> the static halo plan (plan.cpp) on the
//       iterated path; the general monitor (locmon.cpp) for chained tasks
//       (mapsm_task_histogram) whose partition differs from the grid's.
//   P2P copies      -> ncclSend/ncclRecv over NVLink (NCCL
//       mode) or cudaMemcpyAsync peer copies (local mode).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <algorithm>
#include <array>
#include <mutex>
#include <string>
#include <vector>

#include "mapsm.h"
#include "kernels.h"
#include "locmon.h"
#include "runtime.h"

using namespace mapsm;

// ----------------------------------------------------------------- errors

static thread_local std::string g_last_error;

mapsm_status mapsm::fail(mapsm_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return s;
}

// ------------------------------------------------------------------- NCCL

NcclApi mapsm::g_nccl;

mapsm_status mapsm::nccl_load() {
    if (g_nccl.h) return MAPSM_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return fail(MAPSM_ENCCL, "dlopen(libnccl.so.2) failed: %s", dlerror());
#define SYM(field, name)                                                              \
    g_nccl.field = reinterpret_cast<decltype(g_nccl.field)>(dlsym(h, name));          \
    if (!g_nccl.field) return fail(MAPSM_ENCCL, "NCCL symbol %s missing", name);
    SYM(getUniqueId, "ncclGetUniqueId");
    SYM(commInitRank, "ncclCommInitRank");
    SYM(commDestroy, "ncclCommDestroy");
    SYM(commAbort, "ncclCommAbort");
    SYM(commGetAsyncError, "ncclCommGetAsyncError");
    SYM(send, "ncclSend");
    SYM(recv, "ncclRecv");
    SYM(groupStart, "ncclGroupStart");
    SYM(groupEnd, "ncclGroupEnd");
    SYM(allReduce, "ncclAllReduce");
    SYM(allGather, "ncclAllGather");
    SYM(errStr, "ncclGetErrorString");
#undef SYM
    g_nccl.h = h;
    return MAPSM_OK;
}

// ---------------------------------------------------------------- objects

struct TimingPair {
    cudaEvent_t a, b;
};

struct Slab {
    int rank = 0;      // global slab index
    int device = 0;
    int num_sms = 148;
    mapsm_slab_plan plan{};
    char* base[2] = {nullptr, nullptr};  // allocation base (row -r)
    cudaStream_t main = nullptr, side = nullptr;
    bool own_main = false;
    cudaEvent_t ev_b = nullptr, ev_h = nullptr;
    cudaEvent_t ev_i = nullptr;  // interior launch done (concurrent-boundary schedule)
    cudaGraphExec_t graph[2] = {nullptr, nullptr};
    int64_t graph_iters = 0;
    cudaGraphExec_t graph_tb[2] = {nullptr, nullptr};  // deep-halo passes (K generations each)
    int64_t graph_tb_passes = 0;
    unsigned long long* hist = nullptr;  // 256 partial counts (histogram op)
    unsigned long long* hist_acc = nullptr;  // 256 counts + CTA ticket, zero between single-launch histograms
    unsigned int* gbar = nullptr;        // grid-barrier word of the persistent Life kernel
    uint32_t* rxbuf = nullptr;           // SMEM-resident Life: halo exchange slots
    unsigned int* rflags = nullptr;      // ... and per-CTA pass counters
    int64_t rxbytes = 0;
    // fused peer-memory exchange (MAPSM_OPT_EXCHANGE = P2P): my mailbox and
    // the neighbours' buffers / mailboxes (same process, or CUDA IPC)
    void* mailbox = nullptr;
    char* up_base[2] = {nullptr, nullptr};
    char* down_base[2] = {nullptr, nullptr};
    char* up_mail = nullptr;
    char* down_mail = nullptr;
    int64_t up_rows = 0;                 // owned rows of the up neighbour (its bottom halo follows them)
    std::vector<void*> ipc_opened;       // peer mappings to close at destroy
    void* staging = nullptr;   // device staging for host bind/gather (Life)
    int64_t staging_bytes = 0;
    std::vector<TimingPair> t_bulk, t_bnd;
    size_t t_bulk_used = 0, t_bnd_used = 0;
    LaunchRec rec_bulk, rec_bnd;   // last launches (mapsm_launch_query)
};

enum GridState { ST_CREATED = 0, ST_WINDOW = 1, ST_OP = 2, ST_BOUND = 3 };

struct mapsm_grid_s {
    mapsm_ctx ctx = nullptr;
    int64_t w = 0, h = 0;
    int64_t d = 0;                  // planes of a Window(3D) grid (0 = 2-D grid)
    int64_t rpitch = 0;             // device row pitch (== pitch for 2-D; pitch = h * rpitch for 3-D)
    mapsm_dtype dtype = MAPSM_U8;
    int r = 0;
    mapsm_boundary boundary = MAPSM_WRAP;
    mapsm_op op = MAPSM_OP_LIFE;
    float wt[9 * 9 * 9] = {0};      // conv weights: (2r+1)^2 up to r = 8, (2r+1)^3 up to r = 4
    int state = ST_CREATED;
    int64_t pitch = 0;
    int64_t elem = 1;               // host bytes per cell
    std::vector<Slab> slabs;
    int cur = 0;                    // buffer holding the current generation
    int64_t gen = 0, launches = 0, exchanges = 0, device_bytes = 0;
    bool opt_graphs = true, opt_no_exchange = false, opt_timing = false, opt_persistent = true;
    int opt_persistent_mode = 1;  // 1: SMEM-resident kernel when the slab fits, 2: grid-barrier kernel only
    bool opt_own_stream = false;  // the grid's slabs use private streams instead of the ctx stream
    bool opt_p2p = false;       // fused compute + peer-memory halo exchange
    bool opt_ce = false;
    bool opt_host_packed = false;  // Life: host rows are bit-packed (the device row format)        // ... with the rows moved by copy-engine peer copies (MAPSM_EXCHANGE_CE)
    int opt_exchange_sms = -1;  // SMs the interior launch leaves to the exchange in flight (-1: auto)
    bool conc_open = false;     // concurrent-boundary schedule: the side stream is forked from main
    int tb_k = 1;               // generations per pass (MAPSM_OPT_DEEP_HALO); 1 = per-generation path
    int64_t halo = 0;           // halo rows allocated above/below each slab (r, or K*r with deep halos)
    bool deep_valid = false;    // the current buffer's halos are valid to depth `halo` (else only r)
    bool p2p_linked = false;    // peer pointers resolved
    int64_t opt_graph_iters = 16;
    bool used_graphs = false;
    // Segment Location Monitor of this datum (Alg 2) and the buffers of the
    // last re-partitioned chained task (location kTaskLoc + j).
    mapsm::LocationMonitor lm{2};
    bool lm_dirty = true;       // the datum changed since the monitor last saw it
    struct TaskBuf {
        int device = 0;
        int64_t y0 = 0, rows = 0;
        char* ptr = nullptr;    // rows x pitch
        unsigned long long* hist = nullptr;
    };
    int wslot = -1;             // conv r = 2..4: __constant__ weight slot (conv_upload_weights)
    bool wslot_current = false; // the slot holds the current weights on every slab device
    int task_slabs = 0;         // target partition the task buffers belong to
    std::vector<TaskBuf> tbufs;  // one per target slab this process owns
    bool packed() const { return dtype == MAPSM_U8 && r == 1; }
    // partition units: rows of a 2-D grid, planes of a 3-D grid (each unit is `pitch` bytes)
    int64_t units() const { return d ? d : h; }
    int64_t rows_per_unit() const { return d ? h : 1; }   // Life: bit-packed rows
};

static const size_t kMailboxBytes = 64;  // >= sizeof(tma::Mailbox)

// __constant__ weight slots of the r = 2..4 conv kernels, shared by all grids
// of the process (kConvWeightSlots at a time).
static std::mutex g_wslot_mu;
static uint64_t g_wslot_used = 0;
static int wslot_acquire() {
    std::lock_guard<std::mutex> lk(g_wslot_mu);
    for (int i = 0; i < kConvWeightSlots; ++i)
        if (!(g_wslot_used >> i & 1)) {
            g_wslot_used |= 1ull << i;
            return i;
        }
    return -1;
}
static void wslot_release(int i) {
    if (i < 0) return;
    std::lock_guard<std::mutex> lk(g_wslot_mu);
    g_wslot_used &= ~(1ull << i);
}

static char* row_ptr(const mapsm_grid_s* g, const Slab& s, int b, int64_t y) {
    return s.base[b] + (y + g->halo) * g->pitch;
}

// The partition of slab k of a grid.  A one-rank NCCL context (world == 1
// with a communicator, mapsm.h) closes the WRAP row ring through NCCL: its
// halos are exchanged with itself (up == down == 0, send-up / send-down /
// recv-bottom / recv-top to rank 0, matched in issue order as between two
// ranks) instead of the local read-side row map.
static mapsm_status slab_plan(const mapsm_grid_s* g, int64_t halo, mapsm_boundary b, int k, mapsm_slab_plan* p) {
    const mapsm_ctx c = g->ctx;
    mapsm_status st = compute_plan(g->units(), c->g, (int)halo, b, k, p);
    if (st != MAPSM_OK) return st;
    if (!c->local && c->world == 1 && c->comm && b == MAPSM_WRAP && halo > 0) {
        p->up = p->down = 0;
        p->top_kind = p->bottom_kind = MAPSM_HALO_EXCHANGE;
        p->top_src_row = g->units() - halo;
        p->bottom_src_row = 0;
        p->n_send = p->n_recv = 2;
    }
    return MAPSM_OK;
}

static bool has_exchange(const Slab& s) {
    return s.plan.top_kind == MAPSM_HALO_EXCHANGE || s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
}

static int rowmap_of(int kind) {
    switch (kind) {
        case MAPSM_HALO_WRAP_LOCAL: return ROWMAP_WRAP;
        case MAPSM_HALO_CLAMP: return ROWMAP_CLAMP;
        default: return ROWMAP_HALO;  // exchanged rows or zeroed rows
    }
}

// ------------------------------------------------------------- context API

extern "C" mapsm_status mapsm_nccl_unique_id(void* out128) {
    if (!out128) return fail(MAPSM_EINVAL, "out128 is NULL");
    TRY(nccl_load());
    ncclUniqueId id;
    NK(g_nccl.getUniqueId(&id));
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    memcpy(out128, &id, sizeof id);
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_ctx_create(int rank, int world, int device, const void* nccl_unique_id,
                                         void* cuda_stream, mapsm_ctx* out) {
    if (!out) return fail(MAPSM_EINVAL, "out is NULL");
    *out = nullptr;
    if (world < 1 || rank < 0 || rank >= world) return fail(MAPSM_EINVAL, "bad rank %d / world %d", rank, world);
    if (world > 1 && !nccl_unique_id) return fail(MAPSM_EINVAL, "nccl_unique_id must be given when world > 1");
    int ndev = 0;
    CK(cudaGetDeviceCount(&ndev));
    if (device < 0 || device >= ndev) return fail(MAPSM_EINVAL, "device %d out of range (%d devices)", device, ndev);
    DeviceGuard dg;
    CK(cudaSetDevice(device));
    auto* c = new mapsm_ctx_s();
    c->local = false;
    c->rank = rank;
    c->world = world;
    c->g = world;
    c->first_slab = rank;
    c->devices = {device};
    c->user_stream = static_cast<cudaStream_t>(cuda_stream);
    if (nccl_unique_id) {  // world == 1 with an id: the one-rank NCCL ring (mapsm.h)
        mapsm_status s = nccl_load();
        if (s != MAPSM_OK) {
            delete c;
            return s;
        }
        ncclUniqueId id;
        memcpy(&id, nccl_unique_id, sizeof id);
        ncclResult_t r = g_nccl.commInitRank(&c->comm, world, id, rank);
        if (r != ncclSuccess) {
            delete c;
            return fail(MAPSM_ENCCL, "ncclCommInitRank failed: %s", g_nccl.errStr(r));
        }
    }
    *out = c;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_ctx_create_local(int nslabs, const int* devices, mapsm_ctx* out) {
    if (!out || !devices || nslabs < 1) return fail(MAPSM_EINVAL, "bad arguments");
    *out = nullptr;
    int ndev = 0;
    CK(cudaGetDeviceCount(&ndev));
    for (int i = 0; i < nslabs; ++i)
        if (devices[i] < 0 || devices[i] >= ndev) return fail(MAPSM_EINVAL, "device %d out of range", devices[i]);
    DeviceGuard dg;
    // Peer access between distinct devices (host-initiated P2P copies).
    for (int i = 0; i < nslabs; ++i)
        for (int j = 0; j < nslabs; ++j) {
            if (devices[i] == devices[j]) continue;
            int can = 0;
            CK(cudaDeviceCanAccessPeer(&can, devices[i], devices[j]));
            if (can) {
                CK(cudaSetDevice(devices[i]));
                cudaError_t e = cudaDeviceEnablePeerAccess(devices[j], 0);
                if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
                    return fail(MAPSM_ECUDA, "cudaDeviceEnablePeerAccess: %s", cudaGetErrorString(e));
                cudaGetLastError();
            }
        }
    auto* c = new mapsm_ctx_s();
    c->local = true;
    c->g = nslabs;
    c->devices.assign(devices, devices + nslabs);
    *out = c;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_ctx_destroy(mapsm_ctx c) {
    if (!c) return fail(MAPSM_EINVAL, "ctx is NULL");
    if (c->live_grids > 0) return fail(MAPSM_ESTATE, "ctx still has %d grids", c->live_grids);
    if (c->comm) g_nccl.commDestroy(c->comm);
    blas_release(c);
    if (c->ev_h2d) cudaEventDestroy(c->ev_h2d);
    if (c->ev_d2h) cudaEventDestroy(c->ev_d2h);
    delete c;
    return MAPSM_OK;
}

// ---------------------------------------------------------------- grid API

extern "C" mapsm_status mapsm_grid_create(mapsm_ctx ctx, int64_t w, int64_t h, mapsm_dtype dtype,
                                          mapsm_grid* out) {
    if (!ctx || !out) return fail(MAPSM_EINVAL, "NULL argument");
    *out = nullptr;
    if (w < 1 || h < 1) return fail(MAPSM_EINVAL, "grid must be at least 1x1 (w=%lld h=%lld)", (long long)w, (long long)h);
    if (dtype != MAPSM_U8 && dtype != MAPSM_F32) return fail(MAPSM_EUNSUPPORTED, "dtype %d", (int)dtype);
    auto* g = new mapsm_grid_s();
    g->ctx = ctx;
    g->w = w;
    g->h = h;
    g->dtype = dtype;
    g->elem = dtype == MAPSM_U8 ? 1 : 4;
    g->op = dtype == MAPSM_U8 ? MAPSM_OP_LIFE : MAPSM_OP_CONV;
    ctx->live_grids++;
    *out = g;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_grid_create_3d(mapsm_ctx ctx, int64_t w, int64_t h, int64_t d, mapsm_dtype dtype,
                                             mapsm_grid* out) {
    if (!ctx || !out) return fail(MAPSM_EINVAL, "NULL argument");
    *out = nullptr;
    if (w < 1 || h < 1 || d < 1) return fail(MAPSM_EINVAL, "volume must be at least 1x1x1");
    if (dtype != MAPSM_F32) return fail(MAPSM_EUNSUPPORTED, "Window(3D) grids are F32 (convolution)");
    TRY(mapsm_grid_create(ctx, w, h, dtype, out));
    (*out)->d = d;
    return MAPSM_OK;
}

static void free_slab(Slab& s) {
    cudaSetDevice(s.device);
    for (int b = 0; b < 2; ++b)
        if (s.base[b]) cudaFree(s.base[b]);
    if (s.staging) cudaFree(s.staging);
    if (s.hist) cudaFree(s.hist);
    if (s.hist_acc) cudaFree(s.hist_acc);
    if (s.gbar) cudaFree(s.gbar);
    if (s.rxbuf) cudaFree(s.rxbuf);
    if (s.rflags) cudaFree(s.rflags);
    if (s.mailbox) cudaFree(s.mailbox);
    for (void* q : s.ipc_opened) cudaIpcCloseMemHandle(q);
    for (int b = 0; b < 2; ++b) {
        if (s.graph[b]) cudaGraphExecDestroy(s.graph[b]);
        if (s.graph_tb[b]) cudaGraphExecDestroy(s.graph_tb[b]);
    }
    for (auto& t : s.t_bulk) { cudaEventDestroy(t.a); cudaEventDestroy(t.b); }
    for (auto& t : s.t_bnd) { cudaEventDestroy(t.a); cudaEventDestroy(t.b); }
    if (s.ev_b) cudaEventDestroy(s.ev_b);
    if (s.ev_h) cudaEventDestroy(s.ev_h);
    if (s.ev_i) cudaEventDestroy(s.ev_i);
    if (s.side) cudaStreamDestroy(s.side);
    if (s.own_main && s.main) cudaStreamDestroy(s.main);
    s = Slab();
}

// Halo rows per side: r, or K*r with deep halos (K generations per pass,
// MAPSM_OPT_DEEP_HALO; Life and the fp32 convolution).
static int64_t halo_rows(const mapsm_grid_s* g, int radius) {
    const bool life = g->dtype == MAPSM_U8 && radius == 1;
    const bool conv = g->dtype == MAPSM_F32 && radius >= 1;
    return (int64_t)radius * ((life || conv) && g->tb_k > 1 ? g->tb_k : 1);
}

static void drop_graphs(mapsm_grid_s* g) {
    for (auto& s : g->slabs)
        for (int b = 0; b < 2; ++b) {
            if (s.graph[b]) { cudaGraphExecDestroy(s.graph[b]); s.graph[b] = nullptr; }
            if (s.graph_tb[b]) { cudaGraphExecDestroy(s.graph_tb[b]); s.graph_tb[b] = nullptr; }
        }
}

// Partition (plan.cpp) and allocate both buffers of every local slab with
// g->halo rows above and below (the Memory Analyzer's bounding box).
static mapsm_status alloc_slabs(mapsm_grid_s* g, int radius, mapsm_boundary boundary) {
    mapsm_ctx c = g->ctx;
    const int64_t halo = halo_rows(g, radius);
    // validate the partition for every slab before allocating anything
    for (int k = 0; k < c->g; ++k) {
        mapsm_slab_plan p;
        if (slab_plan(g, halo, boundary, k, &p) != MAPSM_OK)
            return fail(MAPSM_EINVAL, "cannot split %lld rows over %d slabs with %lld halo rows (need >= that many rows each)",
                        (long long)g->units(), c->g, (long long)halo);
    }
    DeviceGuard dg;
    for (auto& s : g->slabs) free_slab(s);
    g->slabs.clear();
    g->device_bytes = 0;
    g->r = radius;
    g->wslot_current = false;  // (the boundary selects the kernel's translation unit; new slab devices)
    g->halo = halo;
    g->boundary = boundary;
    const int64_t row_bytes = g->packed() ? (g->w + 31) / 32 * 4 : g->w * g->elem;
    const int64_t align = row_bytes >= 128 ? 128 : 16;
    g->rpitch = (row_bytes + align - 1) / align * align;
    g->pitch = g->rpitch * g->rows_per_unit();  // a unit = one row (2-D) or one plane of h rows (3-D)
    const int nloc = c->local ? c->g : 1;
    g->slabs.resize(nloc);
    for (int i = 0; i < nloc; ++i) {
        Slab& s = g->slabs[i];
        s.rank = c->local ? i : c->first_slab;
        s.device = c->devices[c->local ? i : 0];
        // the plan's kinds / neighbours / rows do not depend on the halo
        // depth; alloc_rows does (rows + 2 * halo)
        slab_plan(g, halo, boundary, s.rank, &s.plan);
        CK(cudaSetDevice(s.device));
        CK(cudaDeviceGetAttribute(&s.num_sms, cudaDevAttrMultiProcessorCount, s.device));
        const size_t bytes = (size_t)s.plan.alloc_rows * (size_t)g->pitch;
        const int nbuf = radius == 0 ? 1 : 2;  // a reductive (non-iterated) task needs no double buffer
        CK(cudaMalloc(&s.mailbox, kMailboxBytes));
        CK(cudaMemset(s.mailbox, 0, kMailboxBytes));
        CK(cudaMalloc(&s.hist, 256 * sizeof(unsigned long long)));  // histogram / chained-task partials
        CK(cudaMalloc(&s.hist_acc, 257 * sizeof(unsigned long long)));
        CK(cudaMemset(s.hist_acc, 0, 257 * sizeof(unsigned long long)));
        g->device_bytes += 513 * sizeof(unsigned long long);
        for (int b = 0; b < nbuf; ++b) {
            cudaError_t e = cudaMalloc(&s.base[b], bytes);
            if (e != cudaSuccess) {
                cudaGetLastError();
                for (auto& t : g->slabs) free_slab(t);
                g->slabs.clear();
                g->state = ST_CREATED;
                return fail(MAPSM_ENOMEM, "cudaMalloc(%zu) on device %d: %s", bytes, s.device, cudaGetErrorString(e));
            }
            CK(cudaMemset(s.base[b], 0, bytes));  // ZERO halos are written once, here
            g->device_bytes += (int64_t)bytes;
        }
        if (!c->local && c->user_stream && !g->opt_own_stream) {
            s.main = c->user_stream;
            s.own_main = false;
        } else {
            CK(cudaStreamCreateWithFlags(&s.main, cudaStreamNonBlocking));
            s.own_main = true;
        }
        CK(cudaStreamCreateWithFlags(&s.side, cudaStreamNonBlocking));
        CK(cudaEventCreateWithFlags(&s.ev_b, cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&s.ev_h, cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&s.ev_i, cudaEventDisableTiming));
    }
    // slabs sharing a device split its SMs (their kernels run concurrently)
    for (auto& s : g->slabs) {
        int same = 0;
        for (auto& t : g->slabs) same += t.device == s.device;
        if (same > 1) s.num_sms = s.num_sms / same > 0 ? s.num_sms / same : 1;
    }
    // the memsets above ran on each device's legacy stream, which the
    // non-blocking slab streams do not wait for: finish them on every device
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaDeviceSynchronize());
    }
    g->p2p_linked = false;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_window_set(mapsm_grid g, int radius, mapsm_boundary boundary) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    if (g->state >= ST_BOUND) return fail(MAPSM_ESTATE, "window_set after bind (allocation depends on r)");
    if (boundary != MAPSM_WRAP && boundary != MAPSM_CLAMP && boundary != MAPSM_ZERO && boundary != MAPSM_NO_CHECKS)
        return fail(MAPSM_EINVAL, "boundary %d", (int)boundary);
    if ((radius == 0) != (boundary == MAPSM_NO_CHECKS))
        return fail(MAPSM_EUNSUPPORTED, "NO_CHECKS goes with radius 0 (histogram input), got r=%d b=%d", radius,
                    (int)boundary);
    if (g->dtype == MAPSM_U8) {
        if (radius != 1 && radius != 0)
            return fail(MAPSM_EUNSUPPORTED, "u8 grids: radius 1 (Life) or 0 (histogram), got %d", radius);
    } else if (g->d) {
        if (radius < 1 || radius > 4)
            return fail(MAPSM_EUNSUPPORTED, "Window(3D) conv radius must be 1..4, got %d", radius);
    } else {
        if (radius < 1 || radius > 8) return fail(MAPSM_EUNSUPPORTED, "conv radius must be 1..8, got %d", radius);
    }
    TRY(alloc_slabs(g, radius, boundary));
    g->state = ST_WINDOW;
    if (g->dtype == MAPSM_U8) {  // one operator per u8 radius: op_set is optional
        g->op = radius == 1 ? MAPSM_OP_LIFE : MAPSM_OP_HISTOGRAM;
        g->state = ST_OP;
    }
    return MAPSM_OK;
}

// The r = 2..4 conv kernels read their weights from a __constant__ slot of
// each device (conv_impl.cuh): acquire one and upload (at bind, and at op_set
// on a bound grid).  The grid's streams are drained first, so no kernel of
// this grid reads the slot while it is rewritten.
static mapsm_status upload_conv_weights(mapsm_grid_s* g) {
    if (g->op != MAPSM_OP_CONV || g->d || !conv_uses_weight_slot(g->r)) return MAPSM_OK;
    if (g->wslot >= 0 && g->wslot_current) return MAPSM_OK;
    if (g->wslot < 0) g->wslot = wslot_acquire();
    if (g->wslot < 0)
        return fail(MAPSM_ENOMEM, "more than %d live r = 2..4 convolution grids (weight slots)", kConvWeightSlots);
    const int cm = g->boundary == MAPSM_WRAP ? COL_WRAP : g->boundary == MAPSM_CLAMP ? COL_CLAMP : COL_ZERO;
    DeviceGuard dg;
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaStreamSynchronize(s.main));
        CK(conv_upload_weights(g->r, cm, g->wslot, g->wt));
    }
    g->wslot_current = true;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_op_set(mapsm_grid g, mapsm_op op, const float* weights) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    if (g->state < ST_WINDOW) return fail(MAPSM_ESTATE, "op_set before window_set");
    if (op == MAPSM_OP_LIFE) {
        if (g->dtype != MAPSM_U8 || g->r != 1) return fail(MAPSM_EUNSUPPORTED, "Life needs dtype U8 and radius 1");
        if (weights) return fail(MAPSM_EINVAL, "Life takes no weights");
    } else if (op == MAPSM_OP_HISTOGRAM) {
        if (g->dtype != MAPSM_U8 || g->r != 0)
            return fail(MAPSM_EUNSUPPORTED, "histogram needs dtype U8 and radius 0 (NO_CHECKS)");
        if (weights) return fail(MAPSM_EINVAL, "histogram takes no weights");
    } else if (op == MAPSM_OP_CONV) {
        if (g->dtype != MAPSM_F32) return fail(MAPSM_EUNSUPPORTED, "conv needs dtype F32");
        if (!weights) return fail(MAPSM_EINVAL, "conv needs (2r+1)^2 weights");
        const int k = 2 * g->r + 1;
        const size_t nw = (size_t)k * k * (g->d ? k : 1);
        if (nw > sizeof(g->wt) / sizeof(g->wt[0])) return fail(MAPSM_EUNSUPPORTED, "too many weights (%zu)", nw);
        memcpy(g->wt, weights, sizeof(float) * nw);
    } else {
        return fail(MAPSM_EUNSUPPORTED, "op %d", (int)op);
    }
    g->op = op;
    g->wslot_current = false;
    drop_graphs(g);
    if (g->state < ST_OP) g->state = ST_OP;
    if (g->state >= ST_BOUND) TRY(upload_conv_weights(g));
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_grid_slab(mapsm_grid g, int i, int64_t* y0, int64_t* rows) {
    if (!g || !y0 || !rows) return fail(MAPSM_EINVAL, "NULL argument");
    if (g->state < ST_WINDOW) return fail(MAPSM_ESTATE, "grid_slab before window_set");
    if (i < 0 || i >= (int)g->slabs.size()) return fail(MAPSM_EINVAL, "local slab %d out of range", i);
    *y0 = g->slabs[i].plan.y0;
    *rows = g->slabs[i].plan.rows;
    return MAPSM_OK;
}

// ------------------------------------------------------------ halo exchange

// Both exchange modes iterate the ordered message list of plan.cpp
// (exchange_messages, exported as mapsm_exchange_plan): NCCL issues it
// verbatim; local mode resolves every receive to the sending slab's matching
// send (the j-th receive from peer P takes P's j-th send to me — NCCL's
// pair-wise in-order matching) and performs it as a peer copy.
static int slab_messages(const mapsm_grid_s* g, const Slab& s, int64_t depth, mapsm_msg* out) {
    return exchange_messages(s.plan, g->units(), depth, g->halo, g->pitch, out);
}

// Local mode: slab i pulls its halos of buffer b from its neighbours with
// device/peer copies on its side stream, after the neighbours' ev_b.
static mapsm_status exchange_local(mapsm_grid_s* g, int b, bool wait_events, int64_t depth) {
    const int G = (int)g->slabs.size();
    std::vector<std::array<mapsm_msg, 4>> msgs(G);
    std::vector<int> nm(G);
    for (int k = 0; k < G; ++k) nm[k] = slab_messages(g, g->slabs[k], depth, msgs[k].data());
    for (int k = 0; k < G; ++k) {
        Slab& s = g->slabs[k];
        CK(cudaSetDevice(s.device));
        int nth_from[2] = {0, 0};  // receives so far from each of (at most) two peers
        int peers[2] = {-1, -1};
        for (int i = 0; i < nm[k]; ++i) {
            const mapsm_msg& m = msgs[k][i];
            if (m.kind != MAPSM_MSG_RECV) continue;
            int slot = (peers[0] == m.peer || peers[0] < 0) ? 0 : 1;
            peers[slot] = m.peer;
            const int j = nth_from[slot]++;
            // the j-th send of slab m.peer addressed to slab k
            const mapsm_msg* src = nullptr;
            int seen = 0;
            for (int q = 0; q < nm[m.peer] && !src; ++q) {
                const mapsm_msg& t = msgs[m.peer][q];
                if (t.kind == MAPSM_MSG_SEND && t.peer == k && seen++ == j) src = &t;
            }
            if (!src || src->bytes != m.bytes)
                return fail(MAPSM_ESTATE, "exchange plan: slab %d receive %d has no matching send", k, i);
            Slab& u = g->slabs[m.peer];
            if (wait_events) CK(cudaStreamWaitEvent(s.side, u.ev_b, 0));
            CK(cudaMemcpyAsync(s.base[b] + m.offset, u.base[b] + src->offset, (size_t)m.bytes, cudaMemcpyDefault,
                               s.side));
            g->exchanges++;
        }
        CK(cudaEventRecord(s.ev_h, s.side));
    }
    return MAPSM_OK;
}

// NCCL mode: one group per pass, issued on the side stream in the list's
// order (send-up, send-down, recv-bottom, recv-top; see plan.cpp).
static mapsm_status exchange_nccl(mapsm_grid_s* g, int b, int64_t depth) {
    Slab& s = g->slabs[0];
    mapsm_msg msgs[4];
    const int n = slab_messages(g, s, depth, msgs);
    NK(g_nccl.groupStart());
    for (int i = 0; i < n; ++i) {
        const mapsm_msg& m = msgs[i];
        if (m.kind == MAPSM_MSG_SEND)
            NK(g_nccl.send(s.base[b] + m.offset, (size_t)m.bytes, ncclUint8, m.peer, g->ctx->comm, s.side));
        else
            NK(g_nccl.recv(s.base[b] + m.offset, (size_t)m.bytes, ncclUint8, m.peer, g->ctx->comm, s.side));
    }
    NK(g_nccl.groupEnd());
    g->exchanges += s.plan.n_recv;
    return MAPSM_OK;
}

// ------------------------------------------------------------- compute step

// Deep halos with K = 2 on a 2-D r = 1..2 conv grid run the fused
// two-generation kernel (conv_tb.cuh): one HBM pass per two generations.
static bool conv_tb2_ok(const mapsm_grid_s* g) {
    return g->op == MAPSM_OP_CONV && !g->d && g->tb_k == 2 && conv_tb2_supported(g->r, g->w, g->pitch);
}

static mapsm_status launch_step(mapsm_grid_s* g, Slab& s, int b_in, const RowBands& bands, bool bulk,
                                const FusedLink* link = nullptr, int K = 1, cudaStream_t on = nullptr,
                                int sms = 0) {
    cudaStream_t st = on ? on : s.main;
    StencilGeom geom;
    geom.in = row_ptr(g, s, b_in, 0);
    geom.out = row_ptr(g, s, b_in ^ 1, 0);
    geom.pitch = g->pitch;
    geom.rows = s.plan.rows;
    geom.w = g->w;
    geom.top_map = rowmap_of(s.plan.top_kind);
    geom.bot_map = rowmap_of(s.plan.bottom_kind);
    geom.col_mode = g->boundary == MAPSM_WRAP ? COL_WRAP : g->boundary == MAPSM_CLAMP ? COL_CLAMP : COL_ZERO;
    geom.plane_rows = g->d ? g->h : 0;
    geom.rpitch = g->rpitch;
    geom.rec = bulk ? &s.rec_bulk : &s.rec_bnd;
    geom.wslot = g->wslot;
    geom.pdl = sms == 0;  // (the concurrent schedules pass their SM split)
    TimingPair* tp = nullptr;
    if (g->opt_timing && &s == &g->slabs[0]) {
        auto& vec = bulk ? s.t_bulk : s.t_bnd;
        size_t& used = bulk ? s.t_bulk_used : s.t_bnd_used;
        if (used == vec.size()) {
            TimingPair t;
            CK(cudaEventCreate(&t.a));
            CK(cudaEventCreate(&t.b));
            vec.push_back(t);
        }
        tp = &vec[used++];
        CK(cudaEventRecord(tp->a, st));
    }
    cudaError_t e;
    int nsm = sms > 0 ? sms : s.num_sms;

    if (g->op == MAPSM_OP_CONV && K == 2 && conv_tb2_ok(g))
        e = launch_conv_tb2(geom, bands, g->r, s.plan.top_kind == MAPSM_HALO_ZERO, s.plan.bottom_kind == MAPSM_HALO_ZERO,
                            nsm, st);
    else if (g->op == MAPSM_OP_LIFE && K > 1)
        e = launch_life_tb(geom, bands, K, s.plan.top_kind == MAPSM_HALO_ZERO, s.plan.bottom_kind == MAPSM_HALO_ZERO,
                           nsm, st);
    else if (g->op == MAPSM_OP_LIFE)
        e = launch_life_step(geom, bands, nsm, st, link);
    else if (g->d)
        e = launch_conv3d(geom, bands, g->r, g->wt, nsm, st);
    else
        e = launch_conv_step(geom, bands, g->r, g->wt, nsm, st, link);
    if (e != cudaSuccess) return fail(MAPSM_ECUDA, "stencil launch: %s", cudaGetErrorString(e));
    if (tp) CK(cudaEventRecord(tp->b, st));
    g->launches++;
    return MAPSM_OK;
}

// Output-row bands: rows sent to neighbours (boundary) and the rest (interior).
static void split_bands(const Slab& s, int64_t r, RowBands& bnd, RowBands& inner) {
    const int64_t rows = s.plan.rows;
    const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
    bnd.nbands = inner.nbands = 0;
    if (rows <= 2 * r) {  // tiny slab: everything is boundary
        bnd.begin[0] = 0; bnd.end[0] = rows; bnd.nbands = 1;
        return;
    }
    if (top) { bnd.begin[bnd.nbands] = 0; bnd.end[bnd.nbands] = r; bnd.nbands++; }
    if (bot) { bnd.begin[bnd.nbands] = rows - r; bnd.end[bnd.nbands] = rows; bnd.nbands++; }
    inner.begin[0] = top ? r : 0;
    inner.end[0] = bot ? rows - r : rows;
    inner.nbands = 1;
}

// One iteration for all local slabs, reading buffer b_in.
// One pass for all local slabs, reading buffer b_in: one generation (K == 1,
// halos of depth r), or K generations of the deep-halo kernel (halos of
// depth K*r, exchanged once per pass).
static mapsm_status pass_conv_deep(mapsm_grid_s* g, int b_in, int K);

// Concurrent-boundary schedule (NCCL mode, MAPSM_OPT_EXCHANGE_SMS = k > 0):
// generation t's boundary rows B(t) and its NCCL exchange X(t) run on the
// side stream on k SMs while the interior I(t) runs on the main stream on the
// other SMs.  B(t) reads I(t-1)'s rows and the halos X(t-1) delivered (side
// stream order); I(t) reads B(t-1)'s rows (not the halos).  So the chain
// I(t-1) -> I(t) -> ... is never held up by an exchange as long as B + X
// fit under I: per generation
//     side: wait I(t-1); B(t); record ev_b; X(t)
//     main: wait B(t-1);  I(t); record ev_i
// (issued main-wait first, so each wait sees the previous generation's
// record).  The side stream is forked from main on first use and joined back
// at the end of mapsm_iterate / of a captured graph (join_side).
static mapsm_status fork_side(mapsm_grid_s* g) {
    if (g->conc_open) return MAPSM_OK;
    Slab& s = g->slabs[0];
    CK(cudaEventRecord(s.ev_i, s.main));
    CK(cudaEventRecord(s.ev_b, s.main));
    CK(cudaStreamWaitEvent(s.side, s.ev_i, 0));
    g->conc_open = true;
    return MAPSM_OK;
}

static mapsm_status join_side(mapsm_grid_s* g) {
    if (!g->conc_open) return MAPSM_OK;
    Slab& s = g->slabs[0];
    DeviceGuard dg;
    CK(cudaSetDevice(s.device));
    CK(cudaEventRecord(s.ev_h, s.side));
    CK(cudaStreamWaitEvent(s.main, s.ev_h, 0));
    g->conc_open = false;
    return MAPSM_OK;
}

// MAPSM_OPT_EXCHANGE_SMS, resolved: -1 (default) = measured choice for the
// 2-D TMA kernels (Life 2, conv r <= 4: 4), 0 elsewhere.
static int exchange_sms(const mapsm_grid_s* g) {
    if (g->opt_exchange_sms >= 0) return g->opt_exchange_sms;
    if (g->d) return 0;
    if (g->op == MAPSM_OP_LIFE) return 2;
    if (g->op == MAPSM_OP_CONV && g->r <= 4) return 4;
    return 0;
}

static bool concurrent_boundary(const mapsm_grid_s* g) {
    return exchange_sms(g) > 0 && !g->ctx->local && !g->opt_timing && !g->opt_p2p &&
           g->slabs.size() == 1 && has_exchange(g->slabs[0]) && g->slabs[0].num_sms > exchange_sms(g);
}

static mapsm_status iterate_concurrent(mapsm_grid_s* g, int b_in, int K, int64_t depth) {
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    TRY(fork_side(g));
    RowBands bnd, inner;
    split_bands(s, depth, bnd, inner);
    CK(cudaStreamWaitEvent(s.main, s.ev_b, 0));  // I(t) after B(t-1)
    CK(cudaStreamWaitEvent(s.side, s.ev_i, 0));  // B(t) after I(t-1)
    const int k = exchange_sms(g);
    TRY(launch_step(g, s, b_in, bnd, false, nullptr, K, s.side, k));
    CK(cudaEventRecord(s.ev_b, s.side));
    if (!g->opt_no_exchange) TRY(exchange_nccl(g, b_in ^ 1, depth));
    if (inner.nbands > 0 && inner.end[0] > inner.begin[0])
        TRY(launch_step(g, s, b_in, inner, true, nullptr, K, s.main, s.num_sms - k));
    CK(cudaEventRecord(s.ev_i, s.main));
    return MAPSM_OK;
}

// xdepth > 0: exchange that many rows (the last generation of a conv deep-halo pass)
static mapsm_status iterate_once(mapsm_grid_s* g, int b_in, int K = 1, int64_t xdepth = 0) {
    if (K > 1 && g->op == MAPSM_OP_CONV && !conv_tb2_ok(g)) return pass_conv_deep(g, b_in, K);
    mapsm_ctx c = g->ctx;
    const int64_t depth = xdepth > 0 ? xdepth : (int64_t)g->r * K;
    if (xdepth == 0 && concurrent_boundary(g)) return iterate_concurrent(g, b_in, K, depth);
    TRY(join_side(g));  // (a trapezoid pass after concurrent generations)
    const bool exch = !g->opt_no_exchange;
    bool any_exchange = false;
    for (auto& s : g->slabs) any_exchange |= has_exchange(s);
    if (!any_exchange) {
        for (auto& s : g->slabs) {
            CK(cudaSetDevice(s.device));
            RowBands all;
            all.nbands = 1;
            all.begin[0] = 0;
            all.end[0] = s.plan.rows;
            TRY(launch_step(g, s, b_in, all, true, nullptr, K));
        }
        return MAPSM_OK;
    }
    std::vector<RowBands> inner(g->slabs.size());
    // 1. boundary rows first (they are what the neighbours wait for)
    for (size_t i = 0; i < g->slabs.size(); ++i) {
        Slab& s = g->slabs[i];
        CK(cudaSetDevice(s.device));
        RowBands bnd;
        split_bands(s, depth, bnd, inner[i]);
        TRY(launch_step(g, s, b_in, bnd, false, nullptr, K));
        CK(cudaEventRecord(s.ev_b, s.main));
    }
    // 2. halo exchange of the freshly computed rows on the side streams
    if (exch) {
        if (c->local) {
            TRY(exchange_local(g, b_in ^ 1, true, depth));
        } else {
            Slab& s = g->slabs[0];
            CK(cudaStreamWaitEvent(s.side, s.ev_b, 0));
            TRY(exchange_nccl(g, b_in ^ 1, depth));
            CK(cudaEventRecord(s.ev_h, s.side));
        }
    }
    // 3. interior rows overlap the exchange; then join before the next step
    for (size_t i = 0; i < g->slabs.size(); ++i) {
        Slab& s = g->slabs[i];
        CK(cudaSetDevice(s.device));
        if (inner[i].nbands > 0 && inner[i].end[0] > inner[i].begin[0])
            TRY(launch_step(g, s, b_in, inner[i], true, nullptr, K));
        if (exch) CK(cudaStreamWaitEvent(s.main, s.ev_h, 0));
    }
    return MAPSM_OK;
}

// Deep halos for the fp32 convolution (reading t1): a
// pass of K generations reads halos of depth K*r (exchanged once per pass)
// and computes a trapezoid: generation j (1..K) writes rows
// [-(K-j)*r, rows + (K-j)*r) on the exchanged sides (halo rows included, as
// the neighbour computes them: same cells, same fmaf chain, so the values are
// identical) and [0, rows) on the others.  Generation K is split into the
// boundary rows (the K*r rows the neighbours need), the exchange on the side
// stream and the interior, as the per-generation path does.  Every cell is
// computed by the same kernel as in K single generations: bit-identical.
static mapsm_status pass_conv_deep(mapsm_grid_s* g, int b_in, int K) {
    const int64_t r = g->r;
    TRY(join_side(g));
    int b = b_in;
    for (int j = 1; j < K; ++j) {
        for (auto& s : g->slabs) {
            CK(cudaSetDevice(s.device));
            const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
            RowBands tr;
            tr.nbands = 1;
            tr.begin[0] = top ? -(int64_t)(K - j) * r : 0;
            tr.end[0] = s.plan.rows + (bot ? (int64_t)(K - j) * r : 0);
            TRY(launch_step(g, s, b, tr, true));
        }
        b ^= 1;
    }
    return iterate_once(g, b, 1, (int64_t)K * r);  // generation K: boundary rows, K*r-row exchange, interior
}

// ------------------------------------------------ fused peer-memory exchange

// Can this grid run the fused exchange?  (TMA kernels, every slab > 2r rows.)
static bool p2p_eligible(const mapsm_grid_s* g) {
    if (g->op != MAPSM_OP_LIFE && g->op != MAPSM_OP_CONV) return false;
    if (g->op == MAPSM_OP_CONV && g->r > 4) return false;  // r = 5..8 run the shared-memory tile kernel
    if (g->op == MAPSM_OP_LIFE && (g->w % 128 != 0 || g->pitch % 16 != 0)) return false;
    if (g->op == MAPSM_OP_CONV && (g->w % 4 != 0 || g->pitch % 16 != 0)) return false;
    if (g->d) return false;  // Window(3D): copy exchange only
    return g->h / g->ctx->g > 2 * (int64_t)g->r;
}

static bool fused_now(const mapsm_grid_s* g) {
    if (!g->opt_p2p || g->opt_no_exchange) return false;
    for (auto& s : g->slabs)
        if (has_exchange(s)) return true;
    return false;
}

// Resolve the neighbours' buffers and mailboxes: plain pointers between slabs
// of one process; CUDA IPC handles (all-gathered with NCCL) across processes.
static mapsm_status p2p_link(mapsm_grid_s* g) {
    if (g->p2p_linked) return MAPSM_OK;
    mapsm_ctx c = g->ctx;
    if (c->local || c->world == 1) {  // (world == 1: the one-rank NCCL ring links to itself)
        for (auto& s : g->slabs) {
            if (s.plan.top_kind == MAPSM_HALO_EXCHANGE) {
                Slab& u = g->slabs[s.plan.up];
                s.up_base[0] = u.base[0];
                s.up_base[1] = u.base[1];
                s.up_mail = static_cast<char*>(u.mailbox);
                s.up_rows = u.plan.rows;
            }
            if (s.plan.bottom_kind == MAPSM_HALO_EXCHANGE) {
                Slab& d = g->slabs[s.plan.down];
                s.down_base[0] = d.base[0];
                s.down_base[1] = d.base[1];
                s.down_mail = static_cast<char*>(d.mailbox);
            }
        }
        g->p2p_linked = true;
        return MAPSM_OK;
    }
    // Across processes: every step that can fail locally is followed by the
    // same collectives on every rank (the handle all-gather, then an
    // all-reduce of the outcome), so a failure on one rank (no IPC, no peer
    // access) surfaces as the same error on all of them — never as a rank
    // waiting in a collective the failed one skipped — and the caller can
    // fall back to the NCCL exchange (bench.py does).
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    const int W = c->world;
    const size_t hb = 3 * sizeof(cudaIpcMemHandle_t);
    std::vector<char> mine(hb, 0), all(hb * W);
    cudaError_t le = cudaSuccess;  // first local failure
    void* mem[3] = {s.base[0], s.base[1], s.mailbox};
    for (int k = 0; k < 3 && le == cudaSuccess; ++k)
        le = cudaIpcGetMemHandle(reinterpret_cast<cudaIpcMemHandle_t*>(mine.data()) + k, mem[k]);
    if (le != cudaSuccess) cudaGetLastError();
    int* dev = nullptr;
    CK(cudaMalloc(&dev, hb * (W + 1) + 2 * sizeof(int)));
    char* hbuf = reinterpret_cast<char*>(dev) + 2 * sizeof(int);
    CK(cudaMemcpyAsync(hbuf, mine.data(), hb, cudaMemcpyHostToDevice, s.main));
    ncclResult_t nr = g_nccl.allGather(hbuf, hbuf + hb, hb, ncclUint8, c->comm, s.main);
    cudaError_t ce = cudaMemcpyAsync(all.data(), hbuf + hb, hb * W, cudaMemcpyDeviceToHost, s.main);
    cudaError_t se = cudaStreamSynchronize(s.main);
    if (nr != ncclSuccess || ce != cudaSuccess || se != cudaSuccess) {
        cudaFree(dev);
        if (nr != ncclSuccess) return fail(MAPSM_ENCCL, "IPC handle all-gather: %s", g_nccl.errStr(nr));
        return fail(MAPSM_ECUDA, "IPC handle all-gather copy failed");
    }
    auto open = [&](int rank, int k, void** out) -> cudaError_t {
        cudaIpcMemHandle_t h;
        memcpy(&h, all.data() + (size_t)rank * hb + k * sizeof(h), sizeof(h));
        cudaError_t e = cudaIpcOpenMemHandle(out, h, cudaIpcMemLazyEnablePeerAccess);
        if (e == cudaSuccess) s.ipc_opened.push_back(*out);
        else cudaGetLastError();
        return e;
    };
    void* pu[3] = {nullptr, nullptr, nullptr};
    void* pd[3] = {nullptr, nullptr, nullptr};
    const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
    const bool same = bot && top && s.plan.down == s.plan.up;  // g == 2 under WRAP: one peer, mapped once
    for (int k = 0; k < 3 && le == cudaSuccess && top; ++k) le = open(s.plan.up, k, &pu[k]);
    for (int k = 0; k < 3 && le == cudaSuccess && bot && !same; ++k) le = open(s.plan.down, k, &pd[k]);
    // every rank learns whether every rank linked
    int ok_h = le == cudaSuccess ? 1 : 0, all_ok = 0;
    CK(cudaMemcpyAsync(dev, &ok_h, sizeof(int), cudaMemcpyHostToDevice, s.main));
    nr = g_nccl.allReduce(dev, dev + 1, 1, ncclInt32, ncclMin, c->comm, s.main);
    ce = cudaMemcpyAsync(&all_ok, dev + 1, sizeof(int), cudaMemcpyDeviceToHost, s.main);
    se = cudaStreamSynchronize(s.main);
    cudaFree(dev);
    if (nr != ncclSuccess) return fail(MAPSM_ENCCL, "P2P link agreement: %s", g_nccl.errStr(nr));
    if (ce != cudaSuccess || se != cudaSuccess) return fail(MAPSM_ECUDA, "P2P link agreement copy failed");
    if (!all_ok) {
        for (void* q : s.ipc_opened) cudaIpcCloseMemHandle(q);
        s.ipc_opened.clear();
        if (le != cudaSuccess)
            return fail(MAPSM_EUNSUPPORTED, "P2P exchange: CUDA IPC linking failed here: %s", cudaGetErrorString(le));
        return fail(MAPSM_EUNSUPPORTED, "P2P exchange: CUDA IPC linking failed on another rank");
    }
    if (top) {
        s.up_base[0] = static_cast<char*>(pu[0]);
        s.up_base[1] = static_cast<char*>(pu[1]);
        s.up_mail = static_cast<char*>(pu[2]);
        mapsm_slab_plan up;
        compute_plan(g->units(), c->g, g->r, g->boundary, s.plan.up, &up);
        s.up_rows = up.rows;
    }
    if (bot) {
        void** q = same ? pu : pd;
        s.down_base[0] = static_cast<char*>(q[0]);
        s.down_base[1] = static_cast<char*>(q[1]);
        s.down_mail = static_cast<char*>(q[2]);
    }
    g->p2p_linked = true;
    return MAPSM_OK;
}

// The peer-memory link of slab s for a launch writing buffer bo: the
// neighbours' halo rows of bo and their mailboxes.
static FusedLink fused_link(const mapsm_grid_s* g, const Slab& s, int bo) {
    const int r = g->r;
    const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
    FusedLink L;
    L.mailbox = s.mailbox;
    L.dst_up = top ? s.up_base[bo] + (s.up_rows + g->halo) * g->pitch : nullptr;  // up's row up_rows (bottom halo)
    L.dst_down = bot ? s.down_base[bo] + (g->halo - r) * g->pitch : nullptr;      // down's row -r (top halo)
    L.sig_up = top ? reinterpret_cast<unsigned int*>(s.up_mail + 16) : nullptr;      // recv_bot
    L.sig_down = bot ? reinterpret_cast<unsigned int*>(s.down_mail + 12) : nullptr;  // recv_top
    L.wait_top = top;
    L.wait_bot = bot;
    return L;
}

// One fused iteration: per slab ONE launch with bands [top boundary rows,
// bottom boundary rows, interior]; the boundary CTAs deliver their rows into
// the neighbours' halos of the output buffer and signal their mailboxes.
static mapsm_status iterate_fused(mapsm_grid_s* g, int b_in) {
    const int r = g->r;
    const int bo = b_in ^ 1;
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
        const int64_t rows = s.plan.rows;
        RowBands bands;
        bands.nbands = 0;
        if (top) { bands.begin[bands.nbands] = 0; bands.end[bands.nbands] = r; bands.nbands++; }
        if (bot) { bands.begin[bands.nbands] = rows - r; bands.end[bands.nbands] = rows; bands.nbands++; }
        bands.begin[bands.nbands] = top ? r : 0;
        bands.end[bands.nbands] = bot ? rows - r : rows;
        bands.nbands++;
        const FusedLink L = fused_link(g, s, bo);
        TRY(launch_step(g, s, b_in, bands, true, &L));
        g->exchanges += s.plan.n_recv;
    }
    return MAPSM_OK;
}

// The concurrent-boundary schedule with the exchange fused into the boundary
// launch (MAPSM_OPT_EXCHANGE = P2P with MAPSM_OPT_EXCHANGE_SMS = k > 0): B(t)
// on the side stream on k SMs computes the boundary rows, stores them into
// the neighbours' halos (NVLink peer stores / same-process stores) and
// signals their mailboxes — its producers wait for the neighbours' B(t-1)
// deliveries before loading halo rows — while I(t) runs on the other SMs.
// No NCCL kernel on the chain: per generation it is B alone beside I.
static bool concurrent_p2p(const mapsm_grid_s* g) {
    return g->opt_exchange_sms > 0 && fused_now(g) && !g->ctx->local && !g->opt_timing && g->slabs.size() == 1 &&
           g->slabs[0].num_sms > g->opt_exchange_sms;
}

static mapsm_status iterate_concurrent_p2p(mapsm_grid_s* g, int b_in) {
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    TRY(fork_side(g));
    RowBands bnd, inner;
    split_bands(s, g->r, bnd, inner);
    const FusedLink L = fused_link(g, s, b_in ^ 1);
    CK(cudaStreamWaitEvent(s.main, s.ev_b, 0));  // I(t) after B(t-1)
    CK(cudaStreamWaitEvent(s.side, s.ev_i, 0));  // B(t) after I(t-1)
    const int k = g->opt_exchange_sms;
    TRY(launch_step(g, s, b_in, bnd, false, &L, 1, s.side, k));
    CK(cudaEventRecord(s.ev_b, s.side));
    g->exchanges += s.plan.n_recv;
    if (inner.nbands > 0 && inner.end[0] > inner.begin[0])
        TRY(launch_step(g, s, b_in, inner, true, nullptr, 1, s.main, s.num_sms - k));
    CK(cudaEventRecord(s.ev_i, s.main));
    return MAPSM_OK;
}

// Host-initiated peer copies (MAPSM_EXCHANGE_CE; the paper's P2P copies,
// P:L51 §2.1 "large host-initiated P2P copies"), in the concurrent-boundary
// schedule: B(t) on the side stream on k SMs — its producers wait until the
// neighbours' generation counts (in my mailbox) reach mine, i.e. their
// B(t-1) rows have landed in my halos — then the copy engines move my r
// first / last rows into the neighbours' halos (cudaMemcpyAsync over NVLink
// through the CUDA-IPC mappings) followed by my generation count into their
// mailboxes, while I(t) runs on the other SMs.  No NCCL kernel and no SM
// time for the transfer.  Ordering: a generation count is the number of
// completed B launches.  A neighbour's copy at t (into my halos of buffer
// (t+1) % 2, which my B(t-1) read) follows its B(t), whose producers waited
// for its count of me to reach t — written only after my B(t-1) finished;
// so a sender is at most one generation ahead and never overwrites halos
// still being read.
static mapsm_status iterate_concurrent_ce(mapsm_grid_s* g, int b_in) {
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    TRY(fork_side(g));
    const int r = g->r;
    const int bo = b_in ^ 1;
    RowBands bnd, inner;
    split_bands(s, r, bnd, inner);
    FusedLink L = fused_link(g, s, bo);
    L.dst_up = L.dst_down = nullptr;  // no peer stores in the kernel
    L.sig_up = L.sig_down = nullptr;
    L.ce = 1;
    const int k = exchange_sms(g) > 0 ? exchange_sms(g) : 2;
    CK(cudaStreamWaitEvent(s.main, s.ev_b, 0));  // I(t) after B(t-1)
    CK(cudaStreamWaitEvent(s.side, s.ev_i, 0));  // B(t) after I(t-1)
    TRY(launch_step(g, s, b_in, bnd, false, &L, 1, s.side, k));
    CK(cudaEventRecord(s.ev_b, s.side));
    const bool top = s.plan.top_kind == MAPSM_HALO_EXCHANGE, bot = s.plan.bottom_kind == MAPSM_HALO_EXCHANGE;
    const size_t rb = (size_t)r * (size_t)g->pitch;
    if (top)
        CK(cudaMemcpyAsync(s.up_base[bo] + (s.up_rows + g->halo) * g->pitch, row_ptr(g, s, bo, 0), rb,
                           cudaMemcpyDefault, s.side));
    if (bot)
        CK(cudaMemcpyAsync(s.down_base[bo] + (g->halo - r) * g->pitch, row_ptr(g, s, bo, s.plan.rows - r), rb,
                           cudaMemcpyDefault, s.side));
    if (top) CK(cudaMemcpyAsync(s.up_mail + 16, s.mailbox, 4, cudaMemcpyDefault, s.side));   // -> up's recv_bot
    if (bot) CK(cudaMemcpyAsync(s.down_mail + 12, s.mailbox, 4, cudaMemcpyDefault, s.side)); // -> down's recv_top
    g->exchanges += s.plan.n_recv;
    if (inner.nbands > 0 && inner.end[0] > inner.begin[0])
        TRY(launch_step(g, s, b_in, inner, true, nullptr, 1, s.main, s.num_sms - k));
    CK(cudaEventRecord(s.ev_i, s.main));
    return MAPSM_OK;
}

static mapsm_status step_all(mapsm_grid_s* g, int b_in) {
    if (fused_now(g) && g->opt_ce) return iterate_concurrent_ce(g, b_in);
    if (fused_now(g)) return concurrent_p2p(g) ? iterate_concurrent_p2p(g, b_in) : iterate_fused(g, b_in);
    return iterate_once(g, b_in);
}

// Deep-halo passes apply: Life with TMA-kernel rows (w % 128 == 0), every slab
// at least K rows (mirror rows at CLAMP edges); the fp32 convolution (2-D and
// Window(3D)) with every slab at least K*r units; copy/NCCL exchange.
static bool tb_active(const mapsm_grid_s* g) {
    if (g->tb_k <= 1 || g->opt_p2p) return false;
    if (g->op == MAPSM_OP_CONV) {
        for (auto& s : g->slabs)
            if (s.plan.rows < g->halo) return false;
        return true;
    }
    if (g->op != MAPSM_OP_LIFE) return false;
    if (g->w % 128 != 0 || g->pitch % 16 != 0) return false;
    for (auto& s : g->slabs)
        if (s.plan.rows < g->tb_k) return false;
    return true;
}

// Re-fill the current buffer's halos to depth g->halo (after per-generation
// steps, which only exchange r rows), ordered after the work already enqueued.
static mapsm_status refresh_deep_halos(mapsm_grid_s* g) {
    bool any = false;
    for (auto& s : g->slabs) any |= has_exchange(s);
    if (!any || g->opt_no_exchange) return MAPSM_OK;
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaEventRecord(s.ev_b, s.main));
    }
    if (g->ctx->local) {
        TRY(exchange_local(g, g->cur, true, g->halo));
    } else {
        Slab& s = g->slabs[0];
        CK(cudaStreamWaitEvent(s.side, s.ev_b, 0));
        TRY(exchange_nccl(g, g->cur, g->halo));
        CK(cudaEventRecord(s.ev_h, s.side));
    }
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaStreamWaitEvent(s.main, s.ev_h, 0));
    }
    return MAPSM_OK;
}

// Buffer flips of one deep-halo pass: the Life kernel does K generations in
// one launch (in -> out); the conv pass runs K single generations.
static int pass_flips(const mapsm_grid_s* g, int K) {
    return g->op == MAPSM_OP_CONV && !conv_tb2_ok(g) ? (K & 1) : 1;
}

static mapsm_status capture_graph(mapsm_grid_s* g, Slab& s, int start_cur, int64_t iters, int K = 1) {
    CK(cudaSetDevice(s.device));
    TRY(join_side(g));
    const int64_t l0 = g->launches, x0 = g->exchanges;
    CK(cudaStreamBeginCapture(s.main, cudaStreamCaptureModeThreadLocal));
    mapsm_status st = MAPSM_OK;
    int cur = start_cur;
    for (int64_t k = 0; k < iters && st == MAPSM_OK; ++k) {
        st = K > 1 ? iterate_once(g, cur, K) : step_all(g, cur);
        cur ^= K > 1 ? pass_flips(g, K) : 1;
    }
    if (st == MAPSM_OK) st = join_side(g);
    g->conc_open = false;
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(s.main, &graph);
    g->launches = l0;
    g->exchanges = x0;
    if (st != MAPSM_OK) {
        if (graph) cudaGraphDestroy(graph);
        return st;
    }
    if (e != cudaSuccess) return fail(MAPSM_ECUDA, "graph capture: %s", cudaGetErrorString(e));
    e = cudaGraphInstantiate(K > 1 ? &s.graph_tb[start_cur] : &s.graph[start_cur], graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) return fail(MAPSM_ECUDA, "graph instantiate: %s", cudaGetErrorString(e));
    if (K > 1)
        s.graph_tb_passes = iters;
    else
        s.graph_iters = iters;
    return MAPSM_OK;
}

static mapsm_status iterate_impl(mapsm_grid_s* g, int64_t n);

extern "C" mapsm_status mapsm_iterate(mapsm_grid g, int64_t n) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    mapsm_status st = iterate_impl(g, n);
    mapsm_status sj = join_side(g);
    return st != MAPSM_OK ? st : sj;
}

static mapsm_status iterate_impl(mapsm_grid_s* g, int64_t n) {
    if (g->state < ST_BOUND) return fail(MAPSM_ESTATE, "iterate before bind");
    if (n < 0) return fail(MAPSM_EINVAL, "n < 0");
    if (n == 0) return MAPSM_OK;
    if (g->op == MAPSM_OP_HISTOGRAM) return fail(MAPSM_EUNSUPPORTED, "a Reductive (histogram) grid is not iterated");
    g->lm_dirty = true;  // a new version of the datum (Alg 2's lastOutput changes)
    DeviceGuard dg;
    const bool graphs = g->opt_graphs && !g->opt_timing && !g->ctx->local;
    // Deep halos: K generations per pass (one halo exchange of K*r rows per
    // pass), then any remainder with the per-generation path below.
    if (tb_active(g) && n >= g->tb_k) {
        const int K = g->tb_k;
        int64_t passes = n / K;
        if (!g->deep_valid) TRY(refresh_deep_halos(g));
        Slab& s0 = g->slabs[0];
        int64_t per_pass_launches = 1, per_pass_exch = 0;
        {
            RowBands bnd, inner;
            split_bands(s0, g->halo, bnd, inner);
            if (has_exchange(s0)) per_pass_launches = 1 + ((inner.nbands > 0 && inner.end[0] > inner.begin[0]) ? 1 : 0);
            if (g->op == MAPSM_OP_CONV && !conv_tb2_ok(g)) per_pass_launches += K - 1;  // the trapezoid generations
            per_pass_exch = (has_exchange(s0) && !g->opt_no_exchange) ? s0.plan.n_recv : 0;
        }
        if (graphs) {
            int64_t gp = g->opt_graph_iters / K;  // passes per graph (even)
            if (gp < 2) gp = 2;
            if (gp % 2) gp++;
            if (s0.graph_tb_passes != gp)
                for (int b = 0; b < 2; ++b)
                    if (s0.graph_tb[b]) { cudaGraphExecDestroy(s0.graph_tb[b]); s0.graph_tb[b] = nullptr; }
            while (passes >= gp) {
                if (!s0.graph_tb[g->cur]) TRY(capture_graph(g, s0, g->cur, gp, K));
                CK(cudaSetDevice(s0.device));
                CK(cudaGraphLaunch(s0.graph_tb[g->cur], s0.main));
                passes -= gp;
                n -= gp * K;
                g->launches += per_pass_launches * gp;
                g->exchanges += per_pass_exch * gp;
                g->gen += gp * K;
                g->used_graphs = true;
            }
        }
        for (; passes > 0; --passes) {
            TRY(iterate_once(g, g->cur, K));
            g->cur ^= pass_flips(g, K);
            g->gen += K;
            n -= K;
        }
        g->deep_valid = true;
        if (n == 0) return MAPSM_OK;
    }
    if (n > 0) g->deep_valid = false;  // per-generation steps exchange only r rows
    // Life slabs with no exchanged halos (one slab): if the double-buffered
    // slab fits in the SMs' shared memory, ONE cooperative launch of the
    // SMEM-resident temporally blocked kernel runs all n generations
    // (life_resident.cu); else, if it fits in L2, the grid-barrier persistent
    // kernel, up to kPersistChunk generations per launch.
    const bool one_slab = g->op == MAPSM_OP_LIFE && g->opt_persistent && !g->opt_timing && g->slabs.size() == 1 &&
                          g->tb_k <= 1 && !has_exchange(g->slabs[0]) && g->w % 64 == 0;
    if (one_slab) {
        Slab& s = g->slabs[0];
        CK(cudaSetDevice(s.device));
        StencilGeom geom;
        geom.in = row_ptr(g, s, g->cur, 0);
        geom.out = row_ptr(g, s, g->cur ^ 1, 0);
        geom.pitch = g->pitch;
        geom.rows = s.plan.rows;
        geom.w = g->w;
        geom.top_map = rowmap_of(s.plan.top_kind);
        geom.bot_map = rowmap_of(s.plan.bottom_kind);
        geom.col_mode = g->boundary == MAPSM_WRAP ? COL_WRAP : g->boundary == MAPSM_CLAMP ? COL_CLAMP : COL_ZERO;
        geom.rec = &s.rec_bulk;
        int rctas = 0, rk = 0, rsmem = 0;
        if (g->opt_persistent_mode != 2 && life_resident_plan(g->w, s.plan.rows, s.num_sms, &rctas, &rk, &rsmem)) {
            const int64_t xb = life_resident_xbuf_bytes(g->w, rctas, rk);
            if (s.rxbytes < xb) {
                if (s.rxbuf) cudaFree(s.rxbuf);
                if (s.rflags) cudaFree(s.rflags);
                s.rxbuf = nullptr;
                s.rflags = nullptr;
                s.rxbytes = 0;
                CK(cudaMalloc(&s.rxbuf, (size_t)xb));
                CK(cudaMalloc(&s.rflags, sizeof(unsigned int) * (size_t)s.num_sms));
                s.rxbytes = xb;
            }
            cudaError_t e = launch_life_resident(geom, n, rctas, rk, rsmem, s.rxbuf, s.rflags, s.main);
            if (e != cudaSuccess) return fail(MAPSM_ECUDA, "resident Life launch: %s", cudaGetErrorString(e));
            g->launches++;
            g->cur ^= 1;  // generation n is in the other buffer, whatever the parity of n
            g->gen += n;
            return MAPSM_OK;
        }
        if (2 * s.plan.alloc_rows * g->pitch <= (64ll << 20)) {
            if (!s.gbar) CK(cudaMalloc(&s.gbar, sizeof(unsigned int)));
            const int64_t kPersistChunk = 1024;
            for (int64_t done = 0; done < n;) {
                const int64_t k = (n - done < kPersistChunk) ? n - done : kPersistChunk;
                geom.in = row_ptr(g, s, g->cur, 0);
                geom.out = row_ptr(g, s, g->cur ^ 1, 0);
                cudaError_t e = launch_life_persistent(geom, k, s.gbar, s.num_sms, s.main);
                if (e != cudaSuccess) return fail(MAPSM_ECUDA, "persistent Life launch: %s", cudaGetErrorString(e));
                g->launches++;
                if (k & 1) g->cur ^= 1;
                g->gen += k;
                done += k;
            }
            return MAPSM_OK;
        }
    }
    // CUDA graphs for the single-stream-per-process modes (g == 1 and NCCL);
    // local multi-slab mode issues directly (it is the single-GPU test vehicle).
    int64_t done = 0;
    if (graphs) {
        Slab& s = g->slabs[0];
        int64_t gi = g->opt_graph_iters;
        if (gi < 2) gi = 2;
        if (gi % 2) gi++;
        if (s.graph_iters != gi) {
            for (int b = 0; b < 2; ++b)
                if (s.graph[b]) { cudaGraphExecDestroy(s.graph[b]); s.graph[b] = nullptr; }
        }
        int64_t per_graph_launches = 0, per_graph_exch = 0;
        {
            // launches per iteration (for the counters; graphs replay them)
            RowBands bnd, inner;
            split_bands(s, g->r, bnd, inner);
            per_graph_launches = (has_exchange(s) && (!fused_now(g) || concurrent_p2p(g) || g->opt_ce))
                                     ? (1 + ((inner.nbands > 0 && inner.end[0] > inner.begin[0]) ? 1 : 0))
                                     : 1;
            per_graph_exch = (has_exchange(s) && !g->opt_no_exchange) ? s.plan.n_recv : 0;
        }
        while (n - done >= gi) {
            if (!s.graph[g->cur]) TRY(capture_graph(g, s, g->cur, gi));
            CK(cudaSetDevice(s.device));
            CK(cudaGraphLaunch(s.graph[g->cur], s.main));
            done += gi;
            g->launches += per_graph_launches * gi;
            g->exchanges += per_graph_exch * gi;
            g->gen += gi;
            g->used_graphs = true;
            // gi is even: cur unchanged
        }
    }
    for (; done < n; ++done) {
        TRY(step_all(g, g->cur));
        g->cur ^= 1;
        g->gen++;
    }
    return MAPSM_OK;
}

static mapsm_status check_async(mapsm_grid_s* g) {
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaStreamSynchronize(s.main));
        CK(cudaStreamSynchronize(s.side));
    }
    if (g->ctx->comm) {
        ncclResult_t ar = ncclSuccess;
        NK(g_nccl.commGetAsyncError(g->ctx->comm, &ar));
        if (ar != ncclSuccess) return fail(MAPSM_ENCCL, "NCCL async error: %s", g_nccl.errStr(ar));
    }
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_sync(mapsm_grid g) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    DeviceGuard dg;
    return check_async(g);
}

// ------------------------------------------------------------- bind / read

// Device memory only (not managed): results written here are stream-ordered;
// managed and host memory are host-readable, so calls writing there return
// with the data in place.
static bool is_device_only_ptr(const void* p, int* dev) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (a.type == cudaMemoryTypeDevice) {
        *dev = a.device;
        return true;
    }
    return false;
}

static bool is_device_ptr(const void* p, int* dev) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
        *dev = a.device;
        return true;
    }
    return false;
}

static mapsm_status ensure_staging(Slab& s, int64_t bytes) {
    if (s.staging_bytes >= bytes) return MAPSM_OK;
    if (s.staging) cudaFree(s.staging);
    s.staging = nullptr;
    s.staging_bytes = 0;
    CK(cudaMalloc(&s.staging, (size_t)bytes));
    s.staging_bytes = bytes;
    return MAPSM_OK;
}

static const int64_t kStagingBytes = 64ll << 20;

// Host transfers of own-stream grids (MAPSM_OPT_OWN_STREAM) of a one-device
// ctx are ordered FIFO across the grids: a grid's copies start after the
// previously issued transfer in the same direction completed.  With several
// grids pipelined (one uploading, one computing, one downloading) this keeps
// each grid's data arriving as early as possible instead of all in-flight
// uploads sharing the copy engine and finishing together — which serialised
// the uploads against the downloads (measured, profiles/r02_e2e_pipeline.txt).
static mapsm_status xfer_begin(mapsm_grid_s* g, Slab& s, bool h2d) {
    mapsm_ctx c = g->ctx;
    if (c->local || !g->opt_own_stream) return MAPSM_OK;
    cudaEvent_t& ev = h2d ? c->ev_h2d : c->ev_d2h;
    if (!ev) {
        CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        return MAPSM_OK;  // nothing recorded yet
    }
    CK(cudaStreamWaitEvent(s.main, ev, 0));
    return MAPSM_OK;
}
static mapsm_status xfer_end(mapsm_grid_s* g, Slab& s, bool h2d) {
    mapsm_ctx c = g->ctx;
    if (c->local || !g->opt_own_stream) return MAPSM_OK;
    CK(cudaEventRecord(h2d ? c->ev_h2d : c->ev_d2h, s.main));
    return MAPSM_OK;
}

// Bytes of one host row: w cells of elem bytes, or (MAPSM_OPT_HOST_PACKED)
// w / 32 little-endian u32 words of cells, bit j of word k = column 32k + j.
static int64_t host_row_bytes(const mapsm_grid_s* g) { return g->opt_host_packed ? g->w / 8 : g->w * g->elem; }

static mapsm_status bind_impl(mapsm_grid_s* g, const void* ptr, int64_t pitch, bool async) {
    if (!g || !ptr) return fail(MAPSM_EINVAL, "NULL argument");
    if (g->state < ST_OP) return fail(MAPSM_ESTATE, "bind before window_set/op_set");
    if (pitch < host_row_bytes(g)) return fail(MAPSM_EINVAL, "row pitch %lld < row bytes", (long long)pitch);
    DeviceGuard dg;
    int pdev = -1;
    const bool on_dev = is_device_ptr(ptr, &pdev);
    const int64_t y_first = g->slabs[0].plan.y0;
    TRY(upload_conv_weights(g));
    // (captured iteration graphs stay valid: they hold the slab buffers, which
    // a Bind refills in place, and start from buffer 0 like every Bind)
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        if (!on_dev) TRY(xfer_begin(g, s, true));
        const char* src = static_cast<const char*>(ptr) + (s.plan.y0 - y_first) * g->rows_per_unit() * pitch;
        const int64_t rows = s.plan.rows;
        if (!g->packed()) {  // planes of a 3-D slab are rows_per_unit contiguous device rows each
            CK(cudaMemcpy2DAsync(row_ptr(g, s, 0, 0), g->rpitch, src, pitch, g->w * g->elem, rows * g->rows_per_unit(),
                                 cudaMemcpyDefault, s.main));
        } else if (g->opt_host_packed) {  // already the device row format: one 2-D copy
            CK(cudaMemcpy2DAsync(row_ptr(g, s, 0, 0), g->pitch, src, pitch, g->w / 8, rows, cudaMemcpyDefault, s.main));
        } else if (on_dev && pdev == s.device) {
            CK(launch_pack_life(reinterpret_cast<const uint8_t*>(src), pitch, row_ptr(g, s, 0, 0), g->pitch, rows,
                                g->w, s.main));
        } else {
            const int64_t spitch = (g->w + 15) / 16 * 16;
            int64_t chunk = kStagingBytes / spitch;
            if (chunk < 1) chunk = 1;
            if (chunk > rows) chunk = rows;
            TRY(ensure_staging(s, chunk * spitch));
            for (int64_t y = 0; y < rows; y += chunk) {
                const int64_t nr = (rows - y < chunk) ? rows - y : chunk;
                CK(cudaMemcpy2DAsync(s.staging, spitch, src + y * pitch, pitch, g->w, nr, cudaMemcpyDefault, s.main));
                CK(launch_pack_life(static_cast<const uint8_t*>(s.staging), spitch, row_ptr(g, s, 0, y), g->pitch, nr,
                                    g->w, s.main));
            }
        }
    }
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        if (!on_dev) TRY(xfer_end(g, s, true));
        if (!async) CK(cudaStreamSynchronize(s.main));
        CK(cudaEventRecord(s.ev_b, s.main));  // the uploaded rows, for the first exchange
    }
    g->cur = 0;
    g->gen = 0;
    g->launches = 0;
    g->exchanges = 0;
    g->lm_dirty = true;
    g->state = ST_BOUND;
    if (g->opt_p2p) {
        if (!p2p_eligible(g))
            return fail(MAPSM_EUNSUPPORTED, "P2P exchange needs the TMA kernels (Life w %% 128, conv w %% 4) and slabs > 2r rows");
        TRY(p2p_link(g));
        // reset the mailboxes BEFORE the initial exchange: a neighbour cannot
        // deliver generation 1 until that exchange (which needs us) completed
        for (auto& s : g->slabs) {
            CK(cudaSetDevice(s.device));
            CK(cudaMemsetAsync(s.mailbox, 0, kMailboxBytes, s.main));
            CK(cudaStreamSynchronize(s.main));
        }
    }
    // Fill the halos of the current buffer once (the first exchange), after
    // every slab's upload (ev_b), before the next compute on the slab (ev_h).
    bool any = false;
    for (auto& s : g->slabs) any |= has_exchange(s);
    if (any) {
        if (g->ctx->local) {
            TRY(exchange_local(g, 0, true, g->halo));
        } else {
            Slab& s = g->slabs[0];
            CK(cudaStreamWaitEvent(s.side, s.ev_b, 0));
            TRY(exchange_nccl(g, 0, g->halo));
            CK(cudaEventRecord(s.ev_h, s.side));
        }
        for (auto& s : g->slabs) {
            CK(cudaSetDevice(s.device));
            CK(cudaStreamWaitEvent(s.main, s.ev_h, 0));
        }
        g->exchanges = 0;
    }
    if (g->opt_p2p && !g->ctx->local && g->ctx->world > 1) {
        // Across processes a neighbour's LAST launch of the previous run may
        // still deliver into my halo and mailbox after my reset above (its
        // kernels need not have finished when I entered this bind).  Every
        // rank's previous launches precede its part of the initial exchange
        // (stream order), so once that collective completed none is in
        // flight: reset again, then a barrier so that no neighbour starts
        // delivering the new run before every mailbox is clean.
        Slab& s = g->slabs[0];
        CK(cudaSetDevice(s.device));
        CK(cudaStreamSynchronize(s.main));
        CK(cudaMemsetAsync(s.mailbox, 0, kMailboxBytes, s.main));
        int* flag = nullptr;
        CK(cudaMallocAsync(reinterpret_cast<void**>(&flag), sizeof(int), s.main));
        CK(cudaMemsetAsync(flag, 0, sizeof(int), s.main));
        ncclResult_t nr = g_nccl.allReduce(flag, flag, 1, ncclInt32, ncclSum, g->ctx->comm, s.main);
        cudaFreeAsync(flag, s.main);
        if (nr != ncclSuccess) return fail(MAPSM_ENCCL, "P2P bind barrier: %s", g_nccl.errStr(nr));
        CK(cudaStreamSynchronize(s.main));
    }
    g->deep_valid = true;
    return async ? MAPSM_OK : check_async(g);
}

extern "C" mapsm_status mapsm_bind(mapsm_grid g, const void* ptr, int64_t pitch) {
    return bind_impl(g, ptr, pitch, false);
}

extern "C" mapsm_status mapsm_bind_async(mapsm_grid g, const void* ptr, int64_t pitch) {
    return bind_impl(g, ptr, pitch, true);
}

// Copy owned rows of the current buffer of slab s to dst (pitch dpitch).
static mapsm_status read_slab(mapsm_grid_s* g, Slab& s, char* dst, int64_t dpitch, bool dst_on_dev) {
    const int64_t rows = s.plan.rows;
    if (!g->packed()) {
        CK(cudaMemcpy2DAsync(dst, dpitch, row_ptr(g, s, g->cur, 0), g->rpitch, g->w * g->elem,
                             rows * g->rows_per_unit(), cudaMemcpyDefault, s.main));
        return MAPSM_OK;
    }
    if (g->opt_host_packed) {
        CK(cudaMemcpy2DAsync(dst, dpitch, row_ptr(g, s, g->cur, 0), g->pitch, g->w / 8, rows, cudaMemcpyDefault,
                             s.main));
        return MAPSM_OK;
    }
    if (dst_on_dev) {
        CK(launch_unpack_life(row_ptr(g, s, g->cur, 0), g->pitch, reinterpret_cast<uint8_t*>(dst), dpitch, rows, g->w,
                              s.main));
        return MAPSM_OK;
    }
    const int64_t spitch = (g->w + 15) / 16 * 16;
    int64_t chunk = kStagingBytes / spitch;
    if (chunk < 1) chunk = 1;
    if (chunk > rows) chunk = rows;
    TRY(ensure_staging(s, chunk * spitch));
    for (int64_t y = 0; y < rows; y += chunk) {
        const int64_t nr = (rows - y < chunk) ? rows - y : chunk;
        CK(launch_unpack_life(row_ptr(g, s, g->cur, y), g->pitch, static_cast<uint8_t*>(s.staging), spitch, nr, g->w,
                              s.main));
        CK(cudaMemcpy2DAsync(dst + y * dpitch, dpitch, s.staging, spitch, g->w, nr, cudaMemcpyDefault, s.main));
    }
    return MAPSM_OK;
}

static mapsm_status read_impl(mapsm_grid_s* g, void* ptr, int64_t pitch, bool async) {
    if (!g || !ptr) return fail(MAPSM_EINVAL, "NULL argument");
    if (g->state < ST_BOUND) return fail(MAPSM_ESTATE, "read before bind");
    if (pitch < host_row_bytes(g)) return fail(MAPSM_EINVAL, "row pitch too small");
    DeviceGuard dg;
    int pdev = -1;
    const bool on_dev = is_device_ptr(ptr, &pdev);
    const int64_t y_first = g->slabs[0].plan.y0;
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        char* dst = static_cast<char*>(ptr) + (s.plan.y0 - y_first) * g->rows_per_unit() * pitch;
        if (!on_dev) TRY(xfer_begin(g, s, false));
        TRY(read_slab(g, s, dst, pitch, on_dev && pdev == s.device));
        if (!on_dev) TRY(xfer_end(g, s, false));
    }
    return async ? MAPSM_OK : check_async(g);
}

extern "C" mapsm_status mapsm_read(mapsm_grid g, void* ptr, int64_t pitch) { return read_impl(g, ptr, pitch, false); }

extern "C" mapsm_status mapsm_read_async(mapsm_grid g, void* ptr, int64_t pitch) {
    return read_impl(g, ptr, pitch, true);
}

// Gather / GatherAsync (Table 2).  `async`: only enqueue (the caller
// waits with mapsm_sync); the root's receive buffer is stream-ordered memory.
static mapsm_status gather_impl(mapsm_grid_s* g, void* ptr, int64_t pitch, int root, bool async) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    if (g->state < ST_BOUND) return fail(MAPSM_ESTATE, "gather before bind");
    mapsm_ctx c = g->ctx;
    if (root < 0 || root >= c->world) return fail(MAPSM_EINVAL, "root %d", root);
    if (c->world == 1) {
        if (!ptr) return fail(MAPSM_EINVAL, "ptr is NULL");
        return read_impl(g, ptr, pitch, async);
    }
    if (c->rank == root && (!ptr || pitch < host_row_bytes(g))) return fail(MAPSM_EINVAL, "root needs ptr and pitch");
    DeviceGuard dg;
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    if (!async) TRY(check_async(g));
    const int64_t slab_bytes_row = g->pitch;
    // the gather list of plan.cpp (mapsm_gather_plan): non-root ranks send
    // their owned rows; the root receives every other slab in slab order
    std::vector<mapsm_msg> msgs(c->world > 1 ? c->world - 1 : 1);
    int nmsg = 0;
    TRY(mapsm_gather_plan(g->units(), c->g, g->r, g->boundary, c->rank, root, g->halo, g->pitch, msgs.data(),
                          (int)msgs.size(), &nmsg));
    if (c->rank != root) {
        for (int i = 0; i < nmsg; ++i)
            NK(g_nccl.send(s.base[g->cur] + msgs[i].offset, (size_t)msgs[i].bytes, ncclUint8, msgs[i].peer, c->comm,
                           s.main));
        return async ? MAPSM_OK : check_async(g);
    }
    int pdev = -1;
    const bool on_dev = is_device_ptr(ptr, &pdev) && pdev == s.device;
    // Root: its own rows, then each received slab via a temporary buffer.
    mapsm_slab_plan pk;
    compute_plan(g->units(), c->g, g->r, g->boundary, 0, &pk);
    const int64_t max_rows = pk.rows;  // slab 0 is never shorter than any other
    char* tmp = nullptr;
    CK(cudaMallocAsync(reinterpret_cast<void**>(&tmp), (size_t)(max_rows * slab_bytes_row), s.main));
    mapsm_status st = read_slab(g, s, static_cast<char*>(ptr) + s.plan.y0 * g->rows_per_unit() * pitch, pitch, on_dev);
    for (int i = 0; i < nmsg && st == MAPSM_OK; ++i) {
        const mapsm_msg& m = msgs[i];
        char* dst = static_cast<char*>(ptr) + m.global_row * g->rows_per_unit() * pitch;
        ncclResult_t r = g_nccl.recv(tmp + m.offset, (size_t)m.bytes, ncclUint8, m.peer, c->comm, s.main);
        if (r != ncclSuccess) {
            st = fail(MAPSM_ENCCL, "gather recv from %d: %s", m.peer, g_nccl.errStr(r));
            break;
        }
        // Reuse read_slab's copy-out path on a view of the received rows.
        Slab view = s;
        view.plan.y0 = m.global_row;
        view.plan.rows = m.rows;
        view.base[g->cur] = tmp - g->halo * g->pitch;
        view.staging = s.staging;
        view.staging_bytes = s.staging_bytes;
        st = read_slab(g, view, dst, pitch, on_dev);
        s.staging = view.staging;  // staging may have been (re)allocated
        s.staging_bytes = view.staging_bytes;
        view.staging = nullptr;
        view.graph[0] = view.graph[1] = nullptr;
        if (!async) {
            cudaError_t e = cudaStreamSynchronize(s.main);
            if (e != cudaSuccess && st == MAPSM_OK) st = fail(MAPSM_ECUDA, "gather: %s", cudaGetErrorString(e));
        }
    }
    cudaFreeAsync(tmp, s.main);  // stream-ordered: after the last copy-out
    if (st != MAPSM_OK) return st;
    return async ? MAPSM_OK : check_async(g);
}

extern "C" mapsm_status mapsm_gather(mapsm_grid g, void* ptr, int64_t pitch, int root) {
    return gather_impl(g, ptr, pitch, root, false);
}

extern "C" mapsm_status mapsm_gather_async(mapsm_grid g, void* ptr, int64_t pitch, int root) {
    return gather_impl(g, ptr, pitch, root, true);
}

// ---------------------------------------------------------------- histogram

extern "C" mapsm_status mapsm_histogram(mapsm_grid g, uint64_t* bins, int nbins) {
    if (!g || !bins) return fail(MAPSM_EINVAL, "NULL argument");
    if (nbins != 256) return fail(MAPSM_EINVAL, "nbins must be 256");
    if (g->state < ST_BOUND || g->op != MAPSM_OP_HISTOGRAM) return fail(MAPSM_ESTATE, "histogram needs a bound HISTOGRAM grid");
    // 1. per-slab partial histograms (shared-memory bins + one commit per CTA);
    // 2. aggregation of the duplicated outputs: local slabs summed
    //    on slab 0's device, then ncclAllReduce across processes.  This is the
    //    chained task on the grid's own partition (no data moves).
    return mapsm_task_histogram(g, 0, bins, nbins, nullptr);
}

static void free_task_bufs(mapsm_grid_s* g) {
    for (auto& t : g->tbufs) {
        cudaSetDevice(t.device);
        if (t.ptr) cudaFree(t.ptr);
        if (t.hist) cudaFree(t.hist);
    }
    g->tbufs.clear();
    g->task_slabs = 0;
}

// ------------------------------------------------------------ chained tasks
// a second task with a different access pattern over the
// same datum (stencil -> histogram of its result), its data movement inferred
// by the Segment Location Monitor (Alg 2) instead of hard-coded.

static const int kTaskLoc = 1 << 20;  // monitor location of target slab j of a re-partitioned task: kTaskLoc + j

static mapsm::Box rows_box(int64_t y0, int64_t rows, int64_t w) {
    mapsm::Box b;
    b.lo[0] = y0, b.hi[0] = y0 + rows;
    b.lo[1] = 0, b.hi[1] = w;
    b.lo[2] = 0, b.hi[2] = 1;
    return b;
}

// Local slab index of global slab k in this process, -1 if another process owns it.
static int local_of(const mapsm_grid_s* g, int k) {
    const int i = k - g->ctx->first_slab;
    return (i >= 0 && i < (int)g->slabs.size()) ? i : -1;
}

static mapsm_status launch_task_hist(mapsm_grid_s* g, const Slab& s, const char* rows0, int64_t rows,
                                     unsigned long long* out, cudaStream_t st) {
    if (g->op == MAPSM_OP_HISTOGRAM) {
        CK(launch_histogram(reinterpret_cast<const uint8_t*>(rows0), g->pitch, g->w, rows, out, s.num_sms, st));
    } else if (g->packed()) {
        CK(launch_histogram_life(rows0, g->pitch, g->w, rows, out, s.num_sms, st));
    } else {  // fp32: units of rows_per_unit rows each (3-D planes)
        CK(launch_histogram_f32(reinterpret_cast<const float*>(rows0), g->rpitch, g->w, rows * g->rows_per_unit(), out,
                                s.num_sms, st));
    }
    g->launches++;
    return MAPSM_OK;
}

// Sum the partial histograms parts[i] (device of local slab owner[i]) into
// slab 0's `hist`, all-reduce across processes, copy to `bins`.  Partials must
// be complete on their owners' main streams (ev_b recorded by the caller).
static mapsm_status aggregate_bins(mapsm_grid_s* g, const std::vector<const unsigned long long*>& parts,
                                   const std::vector<int>& owner, uint64_t* bins) {
    mapsm_ctx c = g->ctx;
    Slab& s0 = g->slabs[0];
    CK(cudaSetDevice(s0.device));
    const int n = (int)parts.size();
    for (int k = 0; k < n; ++k)
        if (owner[k] != 0) CK(cudaStreamWaitEvent(s0.main, g->slabs[owner[k]].ev_b, 0));
    if (n == 0) {
        CK(cudaMemsetAsync(s0.hist, 0, 256 * sizeof(unsigned long long), s0.main));
    } else if (n > 1 || parts[0] != s0.hist) {
        TRY(ensure_staging(s0, (int64_t)(n * sizeof(void*) + 8 + 256 * sizeof(unsigned long long))));
        auto* dparts = static_cast<const unsigned long long**>(s0.staging);
        auto* sum = reinterpret_cast<unsigned long long*>(static_cast<char*>(s0.staging) + n * sizeof(void*) +
                                                          (8 - (n * sizeof(void*)) % 8) % 8);
        CK(cudaMemcpyAsync(dparts, parts.data(), n * sizeof(void*), cudaMemcpyHostToDevice, s0.main));
        CK(launch_histogram_sum(dparts, n, sum, s0.main));
        g->launches++;
        CK(cudaMemcpyAsync(s0.hist, sum, 256 * sizeof(unsigned long long), cudaMemcpyDeviceToDevice, s0.main));
        CK(cudaStreamSynchronize(s0.main));  // `parts` is host memory read by the async copy
    }
    if (c->world > 1) NK(g_nccl.allReduce(s0.hist, s0.hist, 256, ncclUint64, ncclSum, c->comm, s0.main));
    CK(cudaMemcpyAsync(bins, s0.hist, 256 * sizeof(unsigned long long), cudaMemcpyDefault, s0.main));
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_task_histogram(mapsm_grid g, int target_slabs, uint64_t* bins, int nbins,
                                             int64_t* moved_bytes) {
    if (!g || !bins) return fail(MAPSM_EINVAL, "NULL argument");
    if (nbins != 256) return fail(MAPSM_EINVAL, "nbins must be 256");
    if (g->state < ST_BOUND) return fail(MAPSM_ESTATE, "task before bind");
    mapsm_ctx c = g->ctx;
    const int G = c->g;
    if (target_slabs < 0 || target_slabs > G)
        return fail(MAPSM_EINVAL, "target_slabs %d (0..%d)", target_slabs, G);
    // The even row split does not depend on the radius, so T == G is the grid's own partition.
    const bool same = target_slabs == 0 || target_slabs == G;
    const int T = same ? G : target_slabs;
    DeviceGuard dg;
    int64_t moved = 0;

    // Allocator: buffers of a re-partitioned task (kept while T is unchanged,
    // so a later task on the unmodified datum finds its rows up to date).
    if (!same && g->task_slabs != T) {
        free_task_bufs(g);
        g->lm_dirty = true;  // forget up-to-date instances in the freed buffers
        for (int j = 0; j < T; ++j) {
            const int li = local_of(g, j);
            if (li < 0) continue;
            mapsm_slab_plan pj;
            compute_plan(g->units(), T, 0, MAPSM_NO_CHECKS, j, &pj);
            mapsm_grid_s::TaskBuf tb;
            tb.device = g->slabs[li].device;
            tb.y0 = pj.y0;
            tb.rows = pj.rows;
            CK(cudaSetDevice(tb.device));
            g->tbufs.push_back(tb);  // pushed first so free_task_bufs releases it on failure
            CK(cudaMalloc(&g->tbufs.back().hist, 256 * sizeof(unsigned long long)));
            if (pj.rows > 0) CK(cudaMalloc(&g->tbufs.back().ptr, (size_t)(pj.rows * g->pitch)));
        }
        g->task_slabs = T;
    }
    // The monitor learns the datum's current version: slab k's owned rows at location k.
    if (g->lm_dirty) {
        std::vector<mapsm::LocEntry> segs;
        for (int k = 0; k < G; ++k) {
            mapsm_slab_plan pk;
            compute_plan(g->units(), G, 0, MAPSM_NO_CHECKS, k, &pk);
            segs.push_back({k, rows_box(pk.y0, pk.rows, g->w)});
        }
        g->lm.output(0, segs, false);
        g->lm_dirty = false;
    }
    // Alg 2 for every target slab (every process evaluates all of them, so the
    // monitors of all processes stay identical and send/recv pairs match).
    std::vector<std::vector<mapsm::CopyOp>> ops(T);
    std::vector<mapsm_slab_plan> tp(T);
    for (int j = 0; j < T; ++j) {
        compute_plan(g->units(), T, 0, MAPSM_NO_CHECKS, j, &tp[j]);
        const int loc = same ? j : kTaskLoc + j;
        mapsm_status st = g->lm.query(0, rows_box(tp[j].y0, tp[j].rows, g->w), loc, ops[j], nullptr);
        if (st != MAPSM_OK) return fail(st, "location monitor query for target slab %d", j);
    }
    auto tbuf_of = [&](int j) -> mapsm_grid_s::TaskBuf* {
        for (auto& t : g->tbufs)
            if (t.y0 == tp[j].y0 && t.rows == tp[j].rows && local_of(g, j) >= 0) return &t;
        return nullptr;
    };
    // Copies (P2P copy commands of Alg 1 line 13): the producer slab's stream
    // has the current generation; each target's stream waits for it.
    for (auto& s : g->slabs) {
        CK(cudaSetDevice(s.device));
        CK(cudaEventRecord(s.ev_b, s.main));
    }
    bool any_remote = false;
    for (int j = 0; j < T; ++j) {
        const int lj = local_of(g, j);
        for (const auto& op : ops[j]) {
            const int lk = local_of(g, op.src);
            const int64_t nr = op.box.hi[0] - op.box.lo[0];
            if (lj >= 0 && lk >= 0) {
                Slab& dst = g->slabs[lj];
                Slab& src = g->slabs[lk];
                mapsm_grid_s::TaskBuf* tb = tbuf_of(j);
                if (!tb) return fail(MAPSM_ESTATE, "no task buffer for target slab %d", j);
                CK(cudaSetDevice(dst.device));
                CK(cudaStreamWaitEvent(dst.main, src.ev_b, 0));
                CK(cudaMemcpyAsync(tb->ptr + (op.box.lo[0] - tb->y0) * g->pitch,
                                   row_ptr(g, src, g->cur, op.box.lo[0] - src.plan.y0), (size_t)(nr * g->pitch),
                                   cudaMemcpyDefault, dst.main));
                moved += nr * g->pitch;
            } else if (lj >= 0 || lk >= 0) {
                any_remote = true;
            }
        }
    }
    if (any_remote) {  // multi-process: one slab per process, NCCL point-to-point in one group
        Slab& s = g->slabs[0];
        CK(cudaSetDevice(s.device));
        NK(g_nccl.groupStart());
        for (int j = 0; j < T; ++j) {
            const int lj = local_of(g, j);
            for (const auto& op : ops[j]) {
                const int lk = local_of(g, op.src);
                if ((lj >= 0) == (lk >= 0)) continue;
                const int64_t nr = op.box.hi[0] - op.box.lo[0];
                const size_t bytes = (size_t)(nr * g->pitch);
                if (lk >= 0) {
                    NK(g_nccl.send(row_ptr(g, s, g->cur, op.box.lo[0] - s.plan.y0), bytes, ncclUint8, j, c->comm,
                                   s.main));
                } else {
                    mapsm_grid_s::TaskBuf* tb = tbuf_of(j);
                    if (!tb) {
                        g_nccl.groupEnd();
                        return fail(MAPSM_ESTATE, "no task buffer for target slab %d", j);
                    }
                    NK(g_nccl.recv(tb->ptr + (op.box.lo[0] - tb->y0) * g->pitch, bytes, ncclUint8, op.src, c->comm,
                                   s.main));
                    moved += (int64_t)bytes;
                    g->exchanges++;
                }
            }
        }
        NK(g_nccl.groupEnd());
    }
    for (int j = 0; j < T; ++j) g->lm.copied(0, ops[j]);

    // One slab in one process, u8 image on its own partition: a single launch
    // whose last CTA writes the bins (device bins on the slab's device: in
    // place; otherwise into s.hist, then one copy).
    if (same && G == 1 && c->world == 1 && g->op == MAPSM_OP_HISTOGRAM && g->slabs.size() == 1) {
        Slab& s = g->slabs[0];
        CK(cudaSetDevice(s.device));
        int bdev = -1;
        const bool dev_bins = is_device_only_ptr(bins, &bdev) && bdev == s.device;
        CK(launch_histogram_final(reinterpret_cast<const uint8_t*>(row_ptr(g, s, g->cur, 0)), g->pitch, g->w,
                                  s.plan.rows, s.hist_acc,
                                  dev_bins ? reinterpret_cast<unsigned long long*>(bins) : s.hist, s.num_sms,
                                  s.main));
        g->launches++;
        if (moved_bytes) *moved_bytes = moved;
        if (dev_bins) {
            CK(cudaGetLastError());
            return MAPSM_OK;
        }
        CK(cudaMemcpyAsync(bins, s.hist, 256 * sizeof(unsigned long long), cudaMemcpyDefault, s.main));
        return check_async(g);
    }

    // The Reductive-Static task itself, per local target slab, then aggregation.
    std::vector<const unsigned long long*> parts;
    std::vector<int> owner;
    for (int j = 0; j < T; ++j) {
        const int lj = local_of(g, j);
        if (lj < 0) continue;
        Slab& s = g->slabs[lj];
        CK(cudaSetDevice(s.device));
        if (same) {
            TRY(launch_task_hist(g, s, row_ptr(g, s, g->cur, 0), s.plan.rows, s.hist, s.main));
            parts.push_back(s.hist);
        } else {
            mapsm_grid_s::TaskBuf* tb = tbuf_of(j);
            if (!tb) return fail(MAPSM_ESTATE, "no task buffer for target slab %d", j);
            TRY(launch_task_hist(g, s, tb->ptr, tb->rows, tb->hist, s.main));
            parts.push_back(tb->hist);
        }
        owner.push_back(lj);
        CK(cudaEventRecord(s.ev_b, s.main));
    }
    TRY(aggregate_bins(g, parts, owner, bins));
    if (moved_bytes) *moved_bytes = moved;
    // Device-memory bins: stream-ordered like mapsm_iterate (complete on the
    // grid's stream; mapsm_sync surfaces async errors).  Host bins: the call
    // returns with the counts in place (the paper's Gather-then-read).
    int bdev = -1;
    if (is_device_only_ptr(bins, &bdev)) {
        CK(cudaGetLastError());
        return MAPSM_OK;
    }
    return check_async(g);
}

extern "C" mapsm_status mapsm_grid_destroy(mapsm_grid g) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    DeviceGuard dg;
    free_task_bufs(g);
    for (auto& s : g->slabs) {
        cudaSetDevice(s.device);
        cudaStreamSynchronize(s.main);
        cudaStreamSynchronize(s.side);
        free_slab(s);
    }
    wslot_release(g->wslot);
    g->ctx->live_grids--;
    delete g;
    return MAPSM_OK;
}

// ----------------------------------------------------------- introspection

extern "C" mapsm_status mapsm_get_info(mapsm_grid g, mapsm_grid_info* o) {
    if (!g || !o) return fail(MAPSM_EINVAL, "NULL argument");
    o->w = g->w;
    o->h = g->h;
    o->d = g->d;
    o->dtype = g->dtype;
    o->op = g->op;
    o->radius = g->r;
    o->boundary = g->boundary;
    o->world = g->ctx->g;
    o->local_slabs = (int)g->slabs.size();
    o->pitch_bytes = g->pitch;
    o->generation = g->gen;
    o->launches = g->launches;
    o->exchanges = g->exchanges;
    o->device_bytes = g->device_bytes;
    o->used_graphs = g->used_graphs ? 1 : 0;
    o->halo_rows = g->halo;
    o->gens_per_pass = tb_active(g) ? g->tb_k : 1;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_set_option(mapsm_grid g, mapsm_option opt, int64_t v) {
    if (!g) return fail(MAPSM_EINVAL, "grid is NULL");
    switch (opt) {
        case MAPSM_OPT_GRAPHS: g->opt_graphs = v != 0; break;
        case MAPSM_OPT_GRAPH_ITERS:
            if (v < 2) return fail(MAPSM_EINVAL, "graph iters must be >= 2");
            g->opt_graph_iters = v;
            break;
        case MAPSM_OPT_NO_EXCHANGE:
            if (g->opt_no_exchange != (v != 0)) drop_graphs(g);  // captured passes hold the old schedule
            g->opt_no_exchange = v != 0;
            break;
        case MAPSM_OPT_PERSISTENT:
            if (v < 0 || v > 2) return fail(MAPSM_EINVAL, "persistent mode %lld (0, 1, 2)", (long long)v);
            g->opt_persistent = v != 0;
            g->opt_persistent_mode = v == 2 ? 2 : 1;
            break;
        case MAPSM_OPT_EXCHANGE:
            if (v != MAPSM_EXCHANGE_COPY && v != MAPSM_EXCHANGE_P2P && v != MAPSM_EXCHANGE_CE)
                return fail(MAPSM_EINVAL, "exchange mode %lld", (long long)v);
            if (v == MAPSM_EXCHANGE_CE && g->ctx->local)
                return fail(MAPSM_EUNSUPPORTED, "MAPSM_EXCHANGE_CE needs one slab per process (NCCL context)");
            if (g->state >= ST_BOUND && ((v != MAPSM_EXCHANGE_COPY) != g->opt_p2p || (v == MAPSM_EXCHANGE_CE) != g->opt_ce))
                return fail(MAPSM_ESTATE, "set MAPSM_OPT_EXCHANGE before bind");
            g->opt_p2p = v != MAPSM_EXCHANGE_COPY;
            g->opt_ce = v == MAPSM_EXCHANGE_CE;
            break;
        case MAPSM_OPT_TIMING:
            g->opt_timing = v != 0;
            for (auto& s : g->slabs) s.t_bulk_used = s.t_bnd_used = 0;
            break;
        case MAPSM_OPT_HOST_PACKED:
            if (v != 0 && (!g->packed() || g->w % 32 != 0))
                return fail(MAPSM_EUNSUPPORTED, "host-packed rows: Life grids with w %% 32 == 0");
            g->opt_host_packed = v != 0;
            break;
        case MAPSM_OPT_EXCHANGE_SMS:
            if (v < -1 || v > 64) return fail(MAPSM_EINVAL, "exchange SMs %lld (-1..64)", (long long)v);
            g->opt_exchange_sms = (int)v;
            drop_graphs(g);
            break;
        case MAPSM_OPT_OWN_STREAM: {
            g->opt_own_stream = v != 0;
            if (!g->opt_own_stream) break;
            DeviceGuard dg;
            for (auto& s : g->slabs) {  // already allocated: switch to a private stream now
                if (s.own_main) continue;
                CK(cudaSetDevice(s.device));
                CK(cudaStreamSynchronize(s.main));
                CK(cudaStreamCreateWithFlags(&s.main, cudaStreamNonBlocking));
                s.own_main = true;
            }
            break;
        }
        case MAPSM_OPT_DEEP_HALO: {
            const int k = v <= 1 ? 1 : (int)v;
            const bool conv = g->dtype == MAPSM_F32;
            if (k > 1 && !conv && !life_tb_supported(k))
                return fail(MAPSM_EUNSUPPORTED, "deep halo (Life): K must be 1 (off) or one of 2, 3, 4, 6, 8 (got %lld)",
                            (long long)v);
            if (k > 1 && conv && k > 16)
                return fail(MAPSM_EUNSUPPORTED, "deep halo (conv): K must be 1 (off) .. 16 (got %lld)", (long long)v);
            if (k == g->tb_k) break;
            if (g->state >= ST_BOUND) return fail(MAPSM_ESTATE, "set MAPSM_OPT_DEEP_HALO before bind (it sizes the halos)");
            if (g->dtype == MAPSM_U8 && g->state >= ST_WINDOW && g->r != 1)
                return fail(MAPSM_EUNSUPPORTED, "deep halos apply to iterated grids (Life, conv)");
            const int old = g->tb_k;
            g->tb_k = k;
            if (g->state >= ST_WINDOW && g->r >= 1) {  // re-partition and re-allocate with the new halo depth
                const int st = g->state;
                mapsm_status e = alloc_slabs(g, g->r, g->boundary);
                if (e != MAPSM_OK) {
                    g->tb_k = old;
                    if (alloc_slabs(g, g->r, g->boundary) == MAPSM_OK) g->state = st;
                    return e;
                }
                g->state = st;
            }
            break;
        }
        default: return fail(MAPSM_EINVAL, "unknown option %d", (int)opt);
    }
    drop_graphs(g);
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_get_timing(mapsm_grid g, double* bulk_ms, int64_t* bulk_n, double* bnd_ms,
                                         int64_t* bnd_n) {
    if (!g || !bulk_ms || !bulk_n || !bnd_ms || !bnd_n) return fail(MAPSM_EINVAL, "NULL argument");
    if (g->slabs.empty()) return fail(MAPSM_ESTATE, "no slabs");
    DeviceGuard dg;
    Slab& s = g->slabs[0];
    CK(cudaSetDevice(s.device));
    CK(cudaStreamSynchronize(s.main));
    double t = 0;
    for (size_t i = 0; i < s.t_bulk_used; ++i) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, s.t_bulk[i].a, s.t_bulk[i].b));
        t += ms;
    }
    *bulk_ms = t;
    *bulk_n = (int64_t)s.t_bulk_used;
    t = 0;
    for (size_t i = 0; i < s.t_bnd_used; ++i) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, s.t_bnd[i].a, s.t_bnd[i].b));
        t += ms;
    }
    *bnd_ms = t;
    *bnd_n = (int64_t)s.t_bnd_used;
    s.t_bulk_used = s.t_bnd_used = 0;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_grid_stream(mapsm_grid g, int i, void** stream) {
    if (!g || !stream) return fail(MAPSM_EINVAL, "NULL argument");
    if (i < 0 || i >= (int)g->slabs.size()) return fail(MAPSM_EINVAL, "local slab %d out of range", i);
    *stream = g->slabs[i].main;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_launch_query(mapsm_grid g, int i, int which, mapsm_launch_info* o) {
    if (!g || !o) return fail(MAPSM_EINVAL, "NULL argument");
    if (i < 0 || i >= (int)g->slabs.size()) return fail(MAPSM_EINVAL, "local slab %d out of range", i);
    if (which != 0 && which != 1) return fail(MAPSM_EINVAL, "which must be 0 (bulk) or 1 (boundary)");
    const LaunchRec& r = which == 0 ? g->slabs[i].rec_bulk : g->slabs[i].rec_bnd;
    memset(o, 0, sizeof *o);
    o->kernel = r.kernel;
    o->threads = r.threads;
    o->smem_bytes = r.smem;
    o->ring_stages = r.ring_stages;
    o->rows_per_stage = r.rows_per_stage;
    o->consumer_warps = r.consumer_warps;
    o->gens_per_launch = r.gens;
    o->ctas = r.ctas;
    o->strips = r.nstrips;
    if (r.ring_stages > 0) {
        // the (strip, row) split of tma_rows.cuh seg_iter / seg_next, per CTA
        int64_t mn = INT64_MAX, mx = 0, mtot = INT64_MAX, nseg = 0;
        for (int b = 0; b < r.nbands; ++b) {
            const int64_t C = r.cta_begin[b + 1] - r.cta_begin[b];
            const int64_t nr = r.end[b] - r.begin[b];
            const int64_t T = r.nstrips * nr;
            for (int64_t c = 0; c < C; ++c) {
                int64_t pos = c * T / C;
                const int64_t hi = (c + 1) * T / C;
                if (pos >= hi) continue;
                int64_t longest = 0;
                mtot = std::min(mtot, hi - pos);
                while (pos < hi) {
                    const int64_t r0 = pos % nr;
                    const int64_t r1 = (nr - r0 < hi - pos) ? nr : r0 + (hi - pos);
                    longest = std::max(longest, r1 - r0);
                    pos += r1 - r0;
                    ++nseg;
                }
                mn = std::min(mn, longest);
                mx = std::max(mx, longest);
            }
        }
        o->min_cta_seg_rows = nseg ? mn : 0;
        o->max_cta_seg_rows = mx;
        o->min_cta_rows = nseg ? mtot : 0;
        o->segments = nseg;
    }
    return MAPSM_OK;
}

extern "C" const char* mapsm_status_string(mapsm_status s) {
    switch (s) {
        case MAPSM_OK: return "MAPSM_OK";
        case MAPSM_EINVAL: return "MAPSM_EINVAL";
        case MAPSM_ENOMEM: return "MAPSM_ENOMEM";
        case MAPSM_ECUDA: return "MAPSM_ECUDA";
        case MAPSM_ENCCL: return "MAPSM_ENCCL";
        case MAPSM_ESTATE: return "MAPSM_ESTATE";
        case MAPSM_EUNSUPPORTED: return "MAPSM_EUNSUPPORTED";
    }
    return "MAPSM_UNKNOWN";
}

extern "C" const char* mapsm_last_error(void) { return g_last_error.c_str(); }

extern "C" const char* mapsm_version(void) { return "mapsm 0.1 (sm_100a)"; }
