// unmodified.cpp — unmodified GPU routines over multi-GPU datums (SURVEY §8(f)
// NEXT-4; §4.6, §5.4).
//
// "MAPS-Multi can run external GPU routines by using wrapper functions with a
// predetermined prototype ... instead of invoking kernels, the scheduler
// calls the host-level wrapper functions for each GPU with the device ID,
// stream, buffer pointers and their corresponding memory segments".
// Here: fp32 matrix datums (mapsm_matrix), a task = (row count, routine,
// parameters with access patterns, scalars).  The task's rows are split evenly
// over the slabs; each parameter's required segment per slab follows
// its pattern (Table 1: Block(2D) = the slab's row block, Block(2D-
// Transposed) = every column of every row, i.e. the whole matrix for a row
// partition); the datum's Segment Location Monitor (Alg 2, locmon.cpp) infers
// the copies (peer cudaMemcpy, or NCCL send/recv between processes); then the
// wrapper runs per slab on the slab's stream; outputs become the datum's new
// lastOutput (Structured Injective row blocks).  Up-to-date segments are not
// moved again, which is what makes chains of unmodified calls cheap (the
// paper's point against CUBLAS-XT).  Built-in wrappers: SGEMM and
// SAXPY over cuBLAS (library calls, like the paper's Fig 5; cuBLAS is
// dlopen'ed, the one torch loaded if present).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstring>
#include <vector>

#include "locmon.h"
#include "mapsm.h"
#include "runtime.h"

using namespace mapsm;

// ------------------------------------------------------------------ cuBLAS

namespace {

typedef void* cublasHandle_t;
typedef int cublasStatus_t;
enum { CUBLAS_OP_N = 0 };
enum { CUBLAS_DEFAULT_MATH = 0 };

struct BlasApi {
    void* h = nullptr;
    cublasStatus_t (*create)(cublasHandle_t*) = nullptr;
    cublasStatus_t (*destroy)(cublasHandle_t) = nullptr;
    cublasStatus_t (*setStream)(cublasHandle_t, cudaStream_t) = nullptr;
    cublasStatus_t (*setMathMode)(cublasHandle_t, int) = nullptr;
    cublasStatus_t (*sgemm)(cublasHandle_t, int, int, int, int, int, const float*, const float*, int, const float*,
                            int, const float*, float*, int) = nullptr;
    cublasStatus_t (*saxpy)(cublasHandle_t, int, const float*, const float*, int, float*, int) = nullptr;
};
BlasApi g_blas;

mapsm_status blas_load() {
    if (g_blas.h) return MAPSM_OK;
    void* h = dlopen("libcublas.so.12", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("/usr/local/cuda/lib64/libcublas.so.12", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return fail(MAPSM_EUNSUPPORTED, "dlopen(libcublas.so.12) failed: %s", dlerror());
#define SYM(field, name)                                                          \
    g_blas.field = reinterpret_cast<decltype(g_blas.field)>(dlsym(h, name));      \
    if (!g_blas.field) return fail(MAPSM_EUNSUPPORTED, "cuBLAS symbol %s missing", name);
    SYM(create, "cublasCreate_v2");
    SYM(destroy, "cublasDestroy_v2");
    SYM(setStream, "cublasSetStream_v2");
    SYM(setMathMode, "cublasSetMathMode");
    SYM(sgemm, "cublasSgemm_v2");
    SYM(saxpy, "cublasSaxpy_v2");
#undef SYM
    g_blas.h = h;
    return MAPSM_OK;
}

// Per-context state: one stream and one cuBLAS handle per local slab.
struct CtxBlas {
    std::vector<cudaStream_t> streams;
    std::vector<cublasHandle_t> handles;
};

mapsm_status ctx_blas(mapsm_ctx c, CtxBlas** out) {
    if (!c->blas) {
        auto* b = new CtxBlas();
        c->blas = b;
        const int nloc = c->local ? c->g : 1;
        DeviceGuard dg;
        for (int i = 0; i < nloc; ++i) {
            CK(cudaSetDevice(c->devices[i]));
            cudaStream_t s = nullptr;
            if (!c->local && c->user_stream) s = c->user_stream;
            else CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
            b->streams.push_back(s);
            b->handles.push_back(nullptr);
        }
    }
    *out = static_cast<CtxBlas*>(c->blas);
    return MAPSM_OK;
}

}  // namespace

void blas_release(mapsm_ctx_s* c) {
    if (!c->blas) return;
    auto* b = static_cast<CtxBlas*>(c->blas);
    DeviceGuard dg;
    for (size_t i = 0; i < b->streams.size(); ++i) {
        cudaSetDevice(c->devices[i]);
        if (b->handles[i] && g_blas.destroy) g_blas.destroy(b->handles[i]);
        if (b->streams[i] && b->streams[i] != c->user_stream) cudaStreamDestroy(b->streams[i]);
    }
    delete b;
    c->blas = nullptr;
}

// ------------------------------------------------------------------ matrices

struct mapsm_matrix_s {
    mapsm_ctx ctx = nullptr;
    int64_t rows = 0, cols = 0;
    std::vector<float*> dev;       // per local slab: a rows x cols buffer (segments valid per the monitor)
    mapsm::LocationMonitor lm{2};  // datum 0; location = global slab index
    bool bound = false;
};

static mapsm::Box mbox(int64_t r0, int64_t r1, int64_t cols) {
    mapsm::Box b;
    b.lo[0] = r0, b.hi[0] = r1;
    b.lo[1] = 0, b.hi[1] = cols;
    b.lo[2] = 0, b.hi[2] = 1;
    return b;
}

static int local_index(mapsm_ctx c, int k) {
    const int i = k - c->first_slab;
    return (i >= 0 && i < (c->local ? c->g : 1)) ? i : -1;
}

static mapsm_status ensure_dev(mapsm_matrix m, int i) {
    if (m->dev[i]) return MAPSM_OK;
    DeviceGuard dg;
    CK(cudaSetDevice(m->ctx->devices[i]));
    CK(cudaMalloc(&m->dev[i], (size_t)(m->rows * m->cols * sizeof(float))));
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_matrix_create(mapsm_ctx ctx, int64_t rows, int64_t cols, mapsm_matrix* out) {
    if (!ctx || !out) return fail(MAPSM_EINVAL, "NULL argument");
    *out = nullptr;
    if (rows < 1 || cols < 1) return fail(MAPSM_EINVAL, "matrix must be at least 1x1");
    auto* m = new mapsm_matrix_s();
    m->ctx = ctx;
    m->rows = rows;
    m->cols = cols;
    m->dev.assign(ctx->local ? ctx->g : 1, nullptr);
    ctx->live_grids++;
    *out = m;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_matrix_destroy(mapsm_matrix m) {
    if (!m) return fail(MAPSM_EINVAL, "matrix is NULL");
    DeviceGuard dg;
    CtxBlas* b = static_cast<CtxBlas*>(m->ctx->blas);
    for (size_t i = 0; i < m->dev.size(); ++i) {
        if (!m->dev[i]) continue;
        cudaSetDevice(m->ctx->devices[i]);
        if (b) cudaStreamSynchronize(b->streams[i]);
        cudaFree(m->dev[i]);
    }
    m->ctx->live_grids--;
    delete m;
    return MAPSM_OK;
}

// Bind: every process passes the full matrix; it is uploaded to the
// process's first local slab, which becomes the datum's only location per
// process (the monitor then moves segments to the other slabs on demand).
extern "C" mapsm_status mapsm_matrix_bind(mapsm_matrix m, const float* host, int64_t ld) {
    if (!m || !host) return fail(MAPSM_EINVAL, "NULL argument");
    if (ld < m->cols) return fail(MAPSM_EINVAL, "ld %lld < cols", (long long)ld);
    mapsm_ctx c = m->ctx;
    CtxBlas* b = nullptr;
    TRY(ctx_blas(c, &b));
    DeviceGuard dg;
    TRY(ensure_dev(m, 0));
    CK(cudaSetDevice(c->devices[0]));
    for (size_t i = 0; i < m->dev.size(); ++i) {  // no routine may still read the old version
        CK(cudaSetDevice(c->devices[i]));
        CK(cudaStreamSynchronize(b->streams[i]));
    }
    CK(cudaSetDevice(c->devices[0]));
    CK(cudaMemcpy2DAsync(m->dev[0], m->cols * sizeof(float), host, ld * sizeof(float), m->cols * sizeof(float),
                         m->rows, cudaMemcpyDefault, b->streams[0]));
    CK(cudaStreamSynchronize(b->streams[0]));
    std::vector<mapsm::LocEntry> segs;
    if (c->local) {
        segs.push_back({0, mbox(0, m->rows, m->cols)});
    } else {
        for (int k = 0; k < c->world; ++k) segs.push_back({k, mbox(0, m->rows, m->cols)});  // one copy per process
    }
    m->lm.output(0, segs, false);
    m->bound = true;
    return MAPSM_OK;
}

// Execute Alg 2 copies for target slab j (all processes evaluate all targets
// in the same order; cross-process copies are NCCL send/recv in one group).
static mapsm_status run_copies(mapsm_matrix m, const std::vector<std::vector<mapsm::CopyOp>>& ops, CtxBlas* b,
                               int64_t* moved) {
    mapsm_ctx c = m->ctx;
    DeviceGuard dg;
    const size_t rowb = m->cols * sizeof(float);
    std::vector<cudaEvent_t> ev(m->dev.size(), nullptr);
    for (size_t i = 0; i < m->dev.size(); ++i) {  // producers' pending writes
        CK(cudaSetDevice(c->devices[i]));
        CK(cudaEventCreateWithFlags(&ev[i], cudaEventDisableTiming));
        CK(cudaEventRecord(ev[i], b->streams[i]));
    }
    bool remote = false;
    for (size_t j = 0; j < ops.size(); ++j) {
        for (const auto& op : ops[j]) {
            if (op.box.lo[1] != 0 || op.box.hi[1] != m->cols) return fail(MAPSM_EINVAL, "column-split segment");
            const int lj = local_index(c, op.dst), lk = local_index(c, op.src);
            if (lj < 0 || lk < 0) {
                remote = remote || lj >= 0 || lk >= 0;
                continue;
            }
            TRY(ensure_dev(m, lj));
            CK(cudaSetDevice(c->devices[lj]));
            CK(cudaStreamWaitEvent(b->streams[lj], ev[lk], 0));
            const int64_t r0 = op.box.lo[0], nr = op.box.hi[0] - op.box.lo[0];
            CK(cudaMemcpyAsync(m->dev[lj] + r0 * m->cols, m->dev[lk] + r0 * m->cols, nr * rowb, cudaMemcpyDefault,
                               b->streams[lj]));
            *moved += nr * (int64_t)rowb;
        }
    }
    for (size_t i = 0; i < ev.size(); ++i) cudaEventDestroy(ev[i]);
    if (remote) {
        CK(cudaSetDevice(c->devices[0]));
        TRY(ensure_dev(m, 0));
        NK(g_nccl.groupStart());
        for (size_t j = 0; j < ops.size(); ++j) {
            for (const auto& op : ops[j]) {
                const int lj = local_index(c, op.dst), lk = local_index(c, op.src);
                if ((lj >= 0) == (lk >= 0)) continue;
                const int64_t r0 = op.box.lo[0], nr = op.box.hi[0] - op.box.lo[0];
                if (lk >= 0) {
                    NK(g_nccl.send(m->dev[0] + r0 * m->cols, nr * rowb, ncclUint8, op.dst, c->comm, b->streams[0]));
                } else {
                    NK(g_nccl.recv(m->dev[0] + r0 * m->cols, nr * rowb, ncclUint8, op.src, c->comm, b->streams[0]));
                    *moved += nr * (int64_t)rowb;
                }
            }
        }
        NK(g_nccl.groupEnd());
    }
    for (size_t j = 0; j < ops.size(); ++j) m->lm.copied(0, ops[j]);
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_invoke_unmodified(mapsm_ctx c, int64_t task_rows, mapsm_routine routine, void* context,
                                                int nparams, const mapsm_matrix* params, const int* patterns,
                                                const float* scalars, int nscalars, int64_t* moved_bytes) {
    if (!c || !routine || nparams < 1 || nparams > MAPSM_MAX_PARAMS || !params || !patterns)
        return fail(MAPSM_EINVAL, "bad arguments");
    if (task_rows < 1) return fail(MAPSM_EINVAL, "task_rows must be >= 1");
    if (nscalars < 0 || (nscalars > 0 && !scalars)) return fail(MAPSM_EINVAL, "bad scalars");
    for (int i = 0; i < nparams; ++i) {
        if (!params[i] || params[i]->ctx != c) return fail(MAPSM_EINVAL, "parameter %d: bad matrix", i);
        const int p = patterns[i];
        if (p < MAPSM_PAT_BLOCK2D || p > MAPSM_PAT_INOUT_SI) return fail(MAPSM_EINVAL, "parameter %d: pattern %d", i, p);
        if (p != MAPSM_PAT_OUT_SI && !params[i]->bound && !params[i]->lm.known(0))
            return fail(MAPSM_ESTATE, "parameter %d is read before it was bound or written", i);
        if (p != MAPSM_PAT_BLOCK2D_T && params[i]->rows != task_rows)
            return fail(MAPSM_EINVAL, "parameter %d: row-block patterns need rows == task_rows", i);
    }
    CtxBlas* b = nullptr;
    TRY(ctx_blas(c, &b));
    const int G = c->g;
    std::vector<mapsm_slab_plan> plan(G);
    for (int k = 0; k < G; ++k) compute_plan(task_rows, G, 0, MAPSM_NO_CHECKS, k, &plan[k]);
    int64_t moved = 0;
    // 1. data movement inferred per input parameter (Alg 1 lines 3-13 with Alg 2)
    for (int i = 0; i < nparams; ++i) {
        const int p = patterns[i];
        if (p == MAPSM_PAT_OUT_SI) continue;
        mapsm_matrix m = params[i];
        bool dup = false;  // the same datum twice: move it once
        for (int q = 0; q < i; ++q) dup = dup || params[q] == m;
        if (dup) continue;
        std::vector<std::vector<mapsm::CopyOp>> ops(G);
        for (int k = 0; k < G; ++k) {
            const mapsm::Box need = p == MAPSM_PAT_BLOCK2D_T ? mbox(0, m->rows, m->cols)
                                                             : mbox(plan[k].y0, plan[k].y0 + plan[k].rows, m->cols);
            if (need.hi[0] <= need.lo[0]) continue;
            const mapsm_status st = m->lm.query(0, need, k, ops[k], nullptr);
            if (st != MAPSM_OK) return fail(st, "location monitor: parameter %d, slab %d", i, k);
        }
        TRY(run_copies(m, ops, b, &moved));
    }
    // 2. the wrapper, per local slab, on the slab's stream
    DeviceGuard dg;
    for (size_t li = 0; li < b->streams.size(); ++li) {
        const int k = c->first_slab + (int)li;
        if (plan[k].rows == 0) continue;
        mapsm_segment segs[MAPSM_MAX_PARAMS];
        for (int i = 0; i < nparams; ++i) {
            TRY(ensure_dev(params[i], (int)li));
            mapsm_matrix m = params[i];
            const bool whole = patterns[i] == MAPSM_PAT_BLOCK2D_T;
            segs[i].row0 = whole ? 0 : plan[k].y0;
            segs[i].rows = whole ? m->rows : plan[k].rows;
            segs[i].cols = m->cols;
            segs[i].ld = m->cols;
            segs[i].ptr = m->dev[li] + segs[i].row0 * m->cols;
        }
        CK(cudaSetDevice(c->devices[li]));
        const int rc = routine(context ? context : c, k, c->devices[li], b->streams[li], segs, nparams, scalars,
                               nscalars);
        if (rc != 0) return fail(MAPSM_ECUDA, "unmodified routine failed on slab %d (returned %d)", k, rc);
    }
    // 3. outputs: Structured Injective row blocks are the datum's new version
    for (int i = 0; i < nparams; ++i) {
        if (patterns[i] != MAPSM_PAT_OUT_SI && patterns[i] != MAPSM_PAT_INOUT_SI) continue;
        std::vector<mapsm::LocEntry> segs;
        for (int k = 0; k < G; ++k)
            if (plan[k].rows > 0) segs.push_back({k, mbox(plan[k].y0, plan[k].y0 + plan[k].rows, params[i]->cols)});
        params[i]->lm.output(0, segs, false);
    }
    if (moved_bytes) *moved_bytes = moved;
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_matrix_sync(mapsm_matrix m) {
    if (!m) return fail(MAPSM_EINVAL, "matrix is NULL");
    CtxBlas* b = static_cast<CtxBlas*>(m->ctx->blas);
    if (!b) return MAPSM_OK;
    DeviceGuard dg;
    for (size_t i = 0; i < b->streams.size(); ++i) {
        CK(cudaSetDevice(m->ctx->devices[i]));
        CK(cudaStreamSynchronize(b->streams[i]));
    }
    return MAPSM_OK;
}

// Gather: the current version to host memory on `root` — each row
// block from the location the monitor says holds it.  Collective; synchronises.
extern "C" mapsm_status mapsm_matrix_gather(mapsm_matrix m, float* host, int64_t ld, int root) {
    if (!m) return fail(MAPSM_EINVAL, "matrix is NULL");
    mapsm_ctx c = m->ctx;
    if (root < 0 || root >= c->world) return fail(MAPSM_EINVAL, "root %d", root);
    const bool me_root = c->rank == root;
    if (me_root && (!host || ld < m->cols)) return fail(MAPSM_EINVAL, "root needs host and ld >= cols");
    if (!m->lm.known(0)) return fail(MAPSM_ESTATE, "matrix has no data");
    TRY(mapsm_matrix_sync(m));
    CtxBlas* b = nullptr;
    TRY(ctx_blas(c, &b));
    // the root's view: which rows to take from where (Alg 2 with target = root host)
    std::vector<mapsm::CopyOp> ops;
    TRY(m->lm.query(0, mbox(0, m->rows, m->cols), -1 - root, ops, nullptr));
    DeviceGuard dg;
    const size_t rowb = m->cols * sizeof(float);
    std::vector<char> taken;  // rows already gathered (a row may be held by several locations)
    taken.assign((size_t)m->rows, 0);
    bool remote = false;
    for (const auto& op : ops) {
        const int lk = local_index(c, op.src);
        for (int64_t r = op.box.lo[0]; r < op.box.hi[0]; ++r) {
            if (taken[r]) continue;
            int64_t r1 = r;
            while (r1 < op.box.hi[0] && !taken[r1]) taken[r1++] = 1;
            if (lk >= 0 && me_root) {
                CK(cudaSetDevice(c->devices[lk]));
                CK(cudaMemcpy2DAsync(host + r * ld, ld * sizeof(float), m->dev[lk] + r * m->cols, rowb, rowb, r1 - r,
                                     cudaMemcpyDefault, b->streams[lk]));
            } else if (lk >= 0 || me_root) {
                remote = true;
            }
            r = r1 - 1;
        }
    }
    if (remote) {  // multi-process: owners send their rows to the root (one slab per process)
        taken.assign((size_t)m->rows, 0);
        CK(cudaSetDevice(c->devices[0]));
        float* tmp = nullptr;
        if (me_root) CK(cudaMalloc(&tmp, (size_t)(m->rows * rowb)));
        NK(g_nccl.groupStart());
        for (const auto& op : ops) {
            const int lk = local_index(c, op.src);
            for (int64_t r = op.box.lo[0]; r < op.box.hi[0]; ++r) {
                if (taken[r]) continue;
                int64_t r1 = r;
                while (r1 < op.box.hi[0] && !taken[r1]) taken[r1++] = 1;
                if (lk >= 0 && !me_root)
                    NK(g_nccl.send(m->dev[0] + r * m->cols, (r1 - r) * rowb, ncclUint8, root, c->comm, b->streams[0]));
                else if (lk < 0 && me_root)
                    NK(g_nccl.recv(tmp + r * m->cols, (r1 - r) * rowb, ncclUint8, op.src, c->comm, b->streams[0]));
                r = r1 - 1;
            }
        }
        NK(g_nccl.groupEnd());
        if (me_root) {
            taken.assign((size_t)m->rows, 0);
            for (const auto& op : ops) {
                if (local_index(c, op.src) >= 0) continue;
                for (int64_t r = op.box.lo[0]; r < op.box.hi[0]; ++r) {
                    if (taken[r]) continue;
                    int64_t r1 = r;
                    while (r1 < op.box.hi[0] && !taken[r1]) taken[r1++] = 1;
                    CK(cudaMemcpy2DAsync(host + r * ld, ld * sizeof(float), tmp + r * m->cols, rowb, rowb, r1 - r,
                                         cudaMemcpyDefault, b->streams[0]));
                    r = r1 - 1;
                }
            }
        }
        CK(cudaStreamSynchronize(b->streams[0]));
        if (tmp) cudaFree(tmp);
    }
    return mapsm_matrix_sync(m);
}

// ------------------------------------------------------- built-in wrappers

static mapsm_status blas_handle(mapsm_ctx c, int device, cudaStream_t s, cublasHandle_t* out) {
    TRY(blas_load());
    CtxBlas* b = nullptr;
    TRY(ctx_blas(c, &b));
    int li = -1;
    for (size_t i = 0; i < b->streams.size(); ++i)
        if (c->devices[i] == device && b->streams[i] == s) li = (int)i;
    if (li < 0) return fail(MAPSM_EINVAL, "no slab with that device and stream");
    if (!b->handles[li]) {
        if (g_blas.create(&b->handles[li]) != 0) return fail(MAPSM_ECUDA, "cublasCreate failed");
        g_blas.setMathMode(b->handles[li], CUBLAS_DEFAULT_MATH);  // plain fp32 (no TF32)
    }
    if (g_blas.setStream(b->handles[li], s) != 0) return fail(MAPSM_ECUDA, "cublasSetStream failed");
    *out = b->handles[li];
    return MAPSM_OK;
}

// C(row block) = alpha * A(row block) x B + beta * C(row block), row-major:
// computed as the column-major C^T = B^T A^T (the usual transposition trick).
extern "C" int mapsm_routine_sgemm(void* context, int slab, int device, void* stream, const mapsm_segment* segs,
                                   int nsegs, const float* scalars, int nscalars) {
    (void)slab;
    if (nsegs != 3 || nscalars != 2) return 1;
    const mapsm_segment &A = segs[0], &B = segs[1], &C = segs[2];
    if (A.cols != B.rows || C.cols != B.cols || A.rows != C.rows) return 2;
    cublasHandle_t h = nullptr;
    if (blas_handle(static_cast<mapsm_ctx>(context), device, static_cast<cudaStream_t>(stream), &h) != MAPSM_OK)
        return 3;
    return g_blas.sgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)C.cols, (int)C.rows, (int)A.cols, &scalars[0], B.ptr,
                        (int)B.ld, A.ptr, (int)A.ld, &scalars[1], C.ptr, (int)C.ld) == 0 ? 0 : 4;
}

// y(row block) = alpha * x(row block) + y(row block) (Fig 5);
// vectors are n x 1 matrices (or any matrix, element-wise over the block).
extern "C" int mapsm_routine_saxpy(void* context, int slab, int device, void* stream, const mapsm_segment* segs,
                                   int nsegs, const float* scalars, int nscalars) {
    (void)slab;
    if (nsegs != 2 || nscalars != 1) return 1;
    const mapsm_segment &X = segs[0], &Y = segs[1];
    if (X.rows != Y.rows || X.cols != Y.cols) return 2;
    cublasHandle_t h = nullptr;
    if (blas_handle(static_cast<mapsm_ctx>(context), device, static_cast<cudaStream_t>(stream), &h) != MAPSM_OK)
        return 3;
    return g_blas.saxpy(h, (int)(X.rows * X.cols), &scalars[0], X.ptr, 1, Y.ptr, 1) == 0 ? 0 : 4;
}
