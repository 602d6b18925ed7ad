/*
 * mapsm.h — C ABI of libmapsm, the B200-native Window(2D) -> Structured-
 * Injective stencil path of MAPS-Multi (Ben-Nun, Levy, Rubin, Barak, SC'15).
 *
 * Citations: "P:L<n> §<s>" = line n of the paper text, section s.
 *
 * What the library does (BASELINE.json north_star; §2.1
 * §4, Fig 2): an iterated radius-r 2D stencil over a double-
 * buffered grid ("two matrices are used as input and output buffers in
 * alternating succession"), row-slab-partitioned over g GPUs ("task
 * partitioning ... evenly distributing the thread-blocks among the devices",
 * P:L59), with the r halo rows the Window pattern implies exchanged between
 * neighbouring slabs every iteration ("two-line boundary exchanges per
 * iteration").  Three operators:
 *   - MAPSM_OP_LIFE: Conway's Game of Life, B3/S23 on the 3x3 window (P:L133,
 *     Gardner [14] P:L619), radius 1, u8 cells on the host (nonzero = alive),
 *     bit-packed 32 cells per 32-bit word on the device;
 *   - MAPSM_OP_CONV: fp32 window convolution (Table 1, "N-dimensional
 *     convolution"), cross-correlation with (2r+1)^2 row-major weights,
 *     1 <= r <= 8, one fmaf per tap in row-major (dy, dx) order starting from
 *     +0.0f (reading c11) so results are reproducible bit for bit;
 *   - MAPSM_OP_HISTOGRAM: the Reductive (Static) output pattern (P:L104,
 *     Fig 4): 256-bin histogram of a u8 image (bin = pixel value,
 *     64-bit counts) over a radius-0 NO_CHECKS window; per-slab partial
 *     histograms are aggregated across slabs.
 * Boundaries (the Window container's "boundary condition management",
 * P:L115; WRAP is the paper's GoL mode): WRAP = torus on both axes,
 * CLAMP = replicate the nearest edge cell, ZERO = constant 0 outside.
 *
 * Paper API -> this ABI (Table 2):
 *   Matrix<T> A,B + Bind            -> mapsm_grid_create + mapsm_bind
 *   Scheduler::AnalyzeCall x2       -> mapsm_window_set (partition + allocate
 *                                      both buffers with halos)
 *   Scheduler::Invoke (per iter)    -> mapsm_iterate(n)  (asynchronous)
 *   Wait / WaitAll                  -> mapsm_sync
 *   Gather (A if n even, else B)    -> mapsm_gather (always generation n)
 *
 * Conventions (all entry points):
 *   - Every call returns a mapsm_status; MAPSM_OK == 0.  No C++ exception
 *     crosses the ABI.  mapsm_last_error() gives a thread-local message for
 *     the most recent failure on the calling thread.
 *   - Handles are opaque; a ctx must outlive its grids.  A grid owns all of its
 *     device memory (two slab buffers per local slab, each (rows + 2r) rows).
 *   - Host pointers are borrowed only for the duration of the call (data is
 *     copied).  "ptr" arguments accept host memory (pageable or pinned) or
 *     device memory on the slab's device; the kind is detected with
 *     cudaPointerGetAttributes.  Row pitches are in bytes.
 *   - State machine: grid_create -> window_set -> op_set -> bind ->
 *     (iterate)* -> sync/gather/read -> destroy.  Out-of-order calls return
 *     MAPSM_ESTATE (e.g. window_set after bind: the allocation depends on r,
 *     like AnalyzeCall before Invoke).  Re-binding is allowed.
 *   - Multi-process mode (one process per GPU, NCCL over NVLink): bind,
 *     iterate, gather are collective — every rank calls them with the same
 *     arguments (n).  One host thread per ctx; no internal locking.
 *   - Asynchronous CUDA/NCCL errors surface at mapsm_sync / mapsm_gather /
 *     mapsm_read.
 */
#ifndef MAPSM_H
#define MAPSM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    MAPSM_OK = 0,
    MAPSM_EINVAL = -1,       /* bad argument (sizes, pointers, radius, pitch) */
    MAPSM_ENOMEM = -2,       /* device or host allocation failed */
    MAPSM_ECUDA = -3,        /* CUDA runtime / kernel error */
    MAPSM_ENCCL = -4,        /* NCCL missing or failed */
    MAPSM_ESTATE = -5,       /* call out of order for this handle */
    MAPSM_EUNSUPPORTED = -6  /* valid but not supported (dtype/op/radius combo) */
} mapsm_status;

typedef enum { MAPSM_U8 = 1, MAPSM_F32 = 2 } mapsm_dtype;
/* MAPSM_NO_CHECKS: the paper's boundary mode for a radius-0 window (Fig 4,
 * P:L369), used by the histogram's 1x1 Window input. */
typedef enum { MAPSM_WRAP = 0, MAPSM_CLAMP = 1, MAPSM_ZERO = 2, MAPSM_NO_CHECKS = 3 } mapsm_boundary;
typedef enum { MAPSM_OP_LIFE = 0, MAPSM_OP_CONV = 1, MAPSM_OP_HISTOGRAM = 2 } mapsm_op;

/* How a slab obtains the r rows just above (top) / below (bottom) its owned
 * rows — the Segment Location Monitor's answer (Alg 2) for this path. */
typedef enum {
    MAPSM_HALO_EXCHANGE = 0,   /* received from a neighbour slab every iteration */
    MAPSM_HALO_WRAP_LOCAL = 1, /* g == 1 under WRAP: the slab's own far rows (no copy) */
    MAPSM_HALO_CLAMP = 2,      /* global edge under CLAMP: replicate the edge row (no copy) */
    MAPSM_HALO_ZERO = 3        /* global edge under ZERO: zero rows written once at bind */
} mapsm_halo_kind;

typedef struct mapsm_ctx_s* mapsm_ctx;
typedef struct mapsm_grid_s* mapsm_grid;

/* ------------------------------------------------------------ partition plan
 * Pure host arithmetic (the Segmenter + Memory Analyzer + static Location
 * Monitor, Alg 2).  Needs no GPU.
 * For slab `rank` of g over h rows with radius r:
 *   rows = floor(h/g) + (rank < h mod g),  y0 = sum_{j<rank} rows_j
 *   up = (rank-1) mod g, down = (rank+1) mod g (WRAP); -1 at the global edge
 *   under CLAMP/ZERO.  top halo = global rows [y0-r, y0), bottom halo =
 *   [y0+rows, y0+rows+r), taken mod h under WRAP.
 * Requires g >= 1, h >= 1, 0 <= r, and when g > 1: rows_j >= r for all j
 * (so each halo row has exactly one owner, the neighbour) — else EINVAL.   */
typedef struct {
    int64_t y0, rows;              /* owned global rows [y0, y0+rows) */
    int up, down;                  /* neighbour slab ranks, -1 if none */
    int top_kind, bottom_kind;     /* mapsm_halo_kind */
    int64_t top_src_row;           /* global row of the first top-halo row's source (-1 if none) */
    int64_t bottom_src_row;        /* global row of the first bottom-halo row's source (-1 if none) */
    int n_send, n_recv;            /* halo messages per iteration (each r rows) */
    int64_t alloc_rows;            /* rows allocated per buffer = rows + 2r */
} mapsm_slab_plan;

mapsm_status mapsm_plan_query(int64_t h, int g, int radius, mapsm_boundary boundary, int rank,
                              mapsm_slab_plan* out);

/* The messages of the multi-process data plane, as the runtime issues them
 * (pure host arithmetic; the NCCL exchange and gather iterate exactly these
 * lists, so the CPU tests can replay them over another transport).
 * A message moves `rows` whole rows of `pitch` bytes between a slab buffer
 * laid out as [halo rows | owned rows | halo rows] and the peer:            */
typedef enum { MAPSM_MSG_SEND = 0, MAPSM_MSG_RECV = 1 } mapsm_msg_kind;
typedef struct {
    int kind;            /* mapsm_msg_kind */
    int peer;            /* the other slab (global rank) */
    int64_t row;         /* first slab-local row (owned row 0 = 0; top halo rows are < 0,
                          * bottom halo rows >= rows) */
    int64_t rows;        /* rows in the message */
    int64_t offset;      /* byte offset of `row` from the buffer's allocation base
                          * = (row + halo) * pitch; 0 for a gather receive (staging) */
    int64_t bytes;       /* rows * pitch */
    int64_t global_row;  /* global row index (mod h) of the message's first row */
} mapsm_msg;
/* Halo exchange of one pass of slab `rank` (Alg 1's P2P copies; "two-line
 * boundary exchanges per iteration"): `depth` rows per message (r per
 * generation, or K*r with deep halos), buffers with `halo` >= depth rows per
 * side.  Order (the contract, inside one ncclGroupStart/End): send-up (rows
 * [0, depth) to up), send-down (rows [rows-depth, rows) to down), recv-bottom
 * (rows [rows, rows+depth) from down), recv-top (rows [-depth, 0) from up);
 * messages of a global edge under CLAMP/ZERO (and all at g == 1) are absent.
 * Pair-wise issue order matching makes g == 2 WRAP (up == down) correct.
 * ENOMEM (with *n_msgs set) if max_msgs is too small (4 always suffices);
 * EINVAL as mapsm_plan_query, or depth > a slab's rows.                      */
mapsm_status mapsm_exchange_plan(int64_t h, int g, int radius, mapsm_boundary boundary, int rank, int64_t depth,
                                 int64_t halo, int64_t pitch, mapsm_msg* out, int max_msgs, int* n_msgs);
/* Gather (Table 2) to `root`: a non-root slab sends its owned rows
 * (one SEND); the root receives every other slab in slab order (g-1 RECVs,
 * offset 0 = into staging) and places message k at global_row = y0_k.       */
mapsm_status mapsm_gather_plan(int64_t h, int g, int radius, mapsm_boundary boundary, int rank, int root,
                               int64_t halo, int64_t pitch, mapsm_msg* out, int max_msgs, int* n_msgs);

/* ------------------------------------------------- segment location monitor
 * Alg 2 (§4.4): tracks, per datum, `lastOutput` (the segments the
 * last task wrote, per location, and whether they are partials that still
 * need aggregation) and `upToDate` (every location holding an unmodified
 * instance of a segment, "to avoid unnecessary memory transfers"),
 * and answers "which copies bring this segment up to date on that target".
 * Pure host code, needs no GPU.  The runtime uses one monitor per grid for
 * chained tasks (mapsm_task_histogram); these entry points expose the same
 * monitor for tests and for callers composing their own tasks.
 * Boxes are half-open N-D rectangles, dimension 0 = rows (slowest); unused
 * dimensions must be [0, 1).  Locations are caller-chosen ints (the runtime
 * uses the global slab index for slab buffers; -1 conventionally = host).
 * Readings (DESIGN.md l1-l3): "up to date on the target" is tested on the
 * union of the target's up-to-date boxes, and only the part of the segment
 * the target lacks is copied; partials awaiting aggregation are never up to
 * date, and every overlapping partial is copied with needs_aggregation = 1. */
#define MAPSM_MAX_DIMS 3
typedef struct {
    int64_t lo[MAPSM_MAX_DIMS], hi[MAPSM_MAX_DIMS];
} mapsm_box;
typedef struct {
    int src, dst;   /* locations */
    mapsm_box box;  /* the segment to copy (global coordinates) */
} mapsm_copy_op;
typedef struct mapsm_locmon_s* mapsm_locmon;

/* ndims in 1..3, else EINVAL.                                                */
mapsm_status mapsm_locmon_create(int ndims, mapsm_locmon* out);
mapsm_status mapsm_locmon_destroy(mapsm_locmon m);
/* A task wrote a new version of `datum` (>= 0): segment i at locs[i] covers
 * boxes[i] (arrays of nseg, copied).  lastOutput := these segments; upToDate
 * := the same unless needs_aggregation (duplicated partial outputs, the
 * Reductive pattern).                                            */
mapsm_status mapsm_locmon_output(mapsm_locmon m, int datum, int nseg, const int* locs, const mapsm_box* boxes,
                                 int needs_aggregation);
/* Alg 2 for segment `required` of `datum` on location `target`: writes the
 * copy list to ops[0..*n_ops) (*n_ops is set even when it exceeds max_ops, in
 * which case ENOMEM is returned and nothing is written) and the
 * needsAggregation flag.  ESTATE: unknown datum (never output).  EINVAL: part
 * of `required` lies outside every lastOutput segment.                      */
mapsm_status mapsm_locmon_query(mapsm_locmon m, int datum, const mapsm_box* required, int target,
                                mapsm_copy_op* ops, int max_ops, int* n_ops, int* needs_aggregation);
/* The copies in ops[0..nops) completed: their destinations now hold
 * up-to-date instances (the closing step of Alg 2).  No effect on a
 * datum whose lastOutput needs aggregation.                                  */
mapsm_status mapsm_locmon_copied(mapsm_locmon m, int datum, int nops, const mapsm_copy_op* ops);

/* ------------------------------------------------------------------- context */

/* Multi-process mode: one process (rank of world) per GPU.  `nccl_unique_id`
 * is the 128-byte ncclUniqueId from mapsm_nccl_unique_id() on rank 0,
 * broadcast by the caller (e.g. torch.distributed); required when world > 1.
 * world == 1 with an id (from mapsm_nccl_unique_id() in the same process)
 * creates a one-rank NCCL communicator: the WRAP row ring then closes
 * through NCCL, every pass sending the slab's first and last halo rows to
 * itself and receiving its halos with ncclSend / ncclRecv in the order of
 * mapsm_exchange_plan (send-up, send-down, recv-bottom, recv-top, peer 0) —
 * the data plane of the multi-process mode (boundary rows first, exchange on
 * the side stream, interior overlapped, CUDA graphs) executed on one GPU.
 * Results are identical to world == 1 without an id (which maps the halo
 * rows on the read side, no exchange); CLAMP / ZERO have no exchanged edge
 * at world == 1 and are unaffected.  ENCCL if NCCL fails to initialise.
 * `cuda_stream` (a cudaStream_t, e.g. torch.cuda.current_stream().cuda_stream)
 * becomes the compute stream; NULL -> the library creates its own.  The
 * exchange runs on a library-owned side stream.                             */
mapsm_status mapsm_ctx_create(int rank, int world, int device, const void* nccl_unique_id,
                              void* cuda_stream, mapsm_ctx* out);

/* Single-process mode (the paper's own model: one process driving g devices
 * with host-initiated peer copies): g slabs on devices[i]
 * (entries may repeat, e.g. g slabs on one GPU); halos move with
 * cudaMemcpyAsync peer/device copies instead of NCCL.                       */
mapsm_status mapsm_ctx_create_local(int nslabs, const int* devices, mapsm_ctx* out);

mapsm_status mapsm_ctx_destroy(mapsm_ctx ctx);

/* Writes a fresh ncclUniqueId (128 bytes) to out128.  ENCCL if NCCL cannot be
 * loaded (libnccl.so.2, the one torch ships, is dlopen'ed on first use).     */
mapsm_status mapsm_nccl_unique_id(void* out128);

/* ---------------------------------------------------------------------- grid */

/* Declare a w x h datum.  dtype U8 for Life, F32 for conv.          */
mapsm_status mapsm_grid_create(mapsm_ctx ctx, int64_t w, int64_t h, mapsm_dtype dtype,
                               mapsm_grid* out);

/* Window(3D) datum (§5.3 "convolved in three
 * dimensions ... the Window (3D) input memory access pattern", Table 1
 * P:L87-88): a d x h x w fp32 volume, plane-major (host layout: plane z, row
 * y at row index z*h + y of a row-pitched 2-D buffer of d*h rows).  Only
 * dtype F32 (EUNSUPPORTED otherwise).  The volume is partitioned in PLANES
 * over the slabs (like the rows of a 2-D grid), with r halo planes exchanged
 * per iteration; every call below then counts planes where it says rows for
 * partition purposes (mapsm_grid_slab returns (z0, planes); mapsm_bind /
 * mapsm_read take this process's planes [z0, z0+planes) as planes*h rows).
 * mapsm_window_set: radius 1..2, boundary WRAP / CLAMP / ZERO on all three
 * axes.  mapsm_op_set(CONV): (2r+1)^3 weights ordered (dz, dy, dx),
 * one fmaf per tap in that order from +0.0f (reading v1).  The
 * fused P2P exchange and deep halos are 2-D only.                           */
mapsm_status mapsm_grid_create_3d(mapsm_ctx ctx, int64_t w, int64_t h, int64_t d, mapsm_dtype dtype,
                                  mapsm_grid* out);

/* Window(2D) pattern: radius and boundary.  Partitions the rows over
 * the slabs and allocates both buffers of every local slab with 2r halo rows
 * (the Memory Analyzer's bounding box after both AnalyzeCalls, P:L167-169,
 * P:L281).  U8 grids: radius 1 = Life (bit-packed storage), radius 0 with
 * NO_CHECKS = histogram input (byte storage, one buffer).  F32: radius 1..8
 * (r <= 4: TMA row-pipeline kernels; r = 5..8: a
 * shared-memory tile kernel, not eligible for MAPSM_EXCHANGE_P2P).
 * Life takes any width w >= 1 (rows of ceil(w/32) words, the unused bits of
 * the last word kept 0); w % 128 == 0 runs the TMA kernels, w % 64 == 0 a
 * register kernel, other widths a word-per-thread kernel (SURVEY §8(f)
 * NEXT-2).  EUNSUPPORTED: any other radius/boundary combination.  EINVAL: a
 * slab would have fewer than r rows (g > 1).  ENOMEM on allocation failure. */
mapsm_status mapsm_window_set(mapsm_grid grid, int radius, mapsm_boundary boundary);

/* Operator: LIFE (weights must be NULL, dtype U8, r = 1), CONV (weights =
 * (2r+1)^2 fp32 values, row-major over (dy, dx), copied; dtype F32) or
 * HISTOGRAM (weights NULL, dtype U8, r = 0).                                 */
mapsm_status mapsm_op_set(mapsm_grid grid, mapsm_op op, const float* weights);

/* Owned rows of local slab `local_index` (0 in multi-process mode).          */
mapsm_status mapsm_grid_slab(mapsm_grid grid, int local_index, int64_t* y0, int64_t* rows);

/* Bind: upload this process's rows — global rows
 * [y0 of its first local slab, end of its last) — from `ptr` (row pitch
 * `row_pitch_bytes` >= w * elem_size) and fill the halos (one exchange).  Life
 * bytes: nonzero = alive.  Resets the generation counter to 0.  Collective.  */
mapsm_status mapsm_bind(mapsm_grid grid, const void* ptr, int64_t row_pitch_bytes);

/* Enqueue n iterations (Invoke, Alg 1) on the compute stream(s)
 * and return; n == 0 is a no-op.  Collective.                                */
mapsm_status mapsm_iterate(mapsm_grid grid, int64_t n);

/* Wait for all enqueued work (Wait/WaitAll, Table 2) and report async errors.*/
mapsm_status mapsm_sync(mapsm_grid grid);

/* Gather: write the full h x w generation-n grid
 * to `ptr` on rank `root` (other ranks pass NULL).  Life output bytes are
 * exactly 0/1.  Collective; synchronises.                                    */
mapsm_status mapsm_gather(mapsm_grid grid, void* ptr, int64_t row_pitch_bytes, int root);

/* Reductive (Static) aggregate (Fig 4; duplicate-and-aggregate
 * P:L103-105): the 256-bin histogram of the bound image (all slabs of all
 * processes: per-slab shared-memory bins, device-side sum across local slabs,
 * ncclAllReduce across processes) written to bins[0..255] (host or device
 * memory, 64-bit counts) on every process.  nbins must be 256; the grid's op
 * must be HISTOGRAM (else ESTATE).  Collective.  Host, pinned or MANAGED
 * `bins` (host-readable memory): returns with the counts written
 * (synchronises).  Device-memory `bins` (cudaMalloc): stream-ordered on the
 * grid's stream (mapsm_grid_stream), like mapsm_iterate — complete after
 * mapsm_sync or any later synchronisation of that stream.                  */
mapsm_status mapsm_histogram(mapsm_grid grid, uint64_t* bins, int nbins);

/* Chained task: a Reductive (Static) histogram task
 * over the grid's CURRENT generation, as a second task on the same datum with
 * a different access pattern (radius-0 Window in, ReductiveStatic out, Fig 4
 * P:L359-403).  The task partitions the rows over `target_slabs` slabs (0 =
 * the grid's own partition; k >= 1 = rows split evenly over k slabs, slab j
 * on the device of global slab j, k <= total slabs), and the grid's Segment
 * Location Monitor (Alg 2) infers which rows each target slab must receive
 * and from where; rows already up to date on a target (its own slab, or a
 * copy made by an earlier task on the unmodified datum) are not moved.
 * Copies: peer cudaMemcpy (one process) or NCCL send/recv (multi-process).
 * Bins (nbins must be 256, 64-bit counts, written on every process):
 *   HISTOGRAM grids (u8): bin = pixel value (as mapsm_histogram);
 *   Life grids: bin = cell state, so bins[0] = dead, bins[1] = alive cells;
 *   F32 grids: bin = floor(v * 256) for 0 <= v < 1, v < 0 (and NaN) -> 0,
 *              v >= 1 -> 255 (v * 256 is exact in fp32; DESIGN.md h4).
 * `moved_bytes` (may be NULL) receives the bytes this process received for
 * the task.  EINVAL: target_slabs out of range.  ESTATE: grid not bound.
 * Collective; synchronisation as mapsm_histogram (host / managed bins:
 * synchronises; device-memory bins: stream-ordered).                         */
mapsm_status mapsm_task_histogram(mapsm_grid grid, int target_slabs, uint64_t* bins, int nbins,
                                  int64_t* moved_bytes);

/* GatherAsync (Table 2): like mapsm_gather but returns once the
 * copies are enqueued; `ptr` is complete after mapsm_sync (Wait).  Use pinned
 * host or device memory for a truly asynchronous copy (pageable memory makes
 * the device-to-host step synchronous).  Do not iterate the grid before the
 * mapsm_sync.  Collective.                                                   */
mapsm_status mapsm_gather_async(mapsm_grid grid, void* ptr, int64_t row_pitch_bytes, int root);

/* ------------------------------------------------- unmodified GPU routines
 * SURVEY §8(f) NEXT-4; §4.6 ("the scheduler calls the host-level
 * wrapper functions for each GPU with the device ID, stream, buffer pointers
 * and their corresponding memory segments"), §5.4.
 * A matrix datum is a rows x cols fp32 row-major matrix.  A task splits
 * `task_rows` evenly over the slabs and gives every parameter an
 * access pattern (Table 1):
 *   MAPSM_PAT_BLOCK2D    input, the slab's row block (rows == task_rows)
 *   MAPSM_PAT_BLOCK2D_T  input, the whole matrix (Block (2D-Transposed): a row
 *                        block of the output needs every column of every row)
 *   MAPSM_PAT_OUT_SI     output, Structured Injective row block (write only)
 *   MAPSM_PAT_INOUT_SI   input row block that is also the output row block
 * The matrix's Segment Location Monitor (Alg 2) infers the copies each slab
 * needs (segments already up to date are not moved, so chains of calls on
 * unchanged inputs move nothing — the paper's point against CUBLAS-XT,
 * P:L497); then `routine` runs once per local slab on the slab's stream and
 * must only enqueue work on that stream.  Outputs become the datums' new
 * versions (row blocks on their slabs).  Asynchronous: mapsm_matrix_sync /
 * mapsm_matrix_gather wait.  Collective in multi-process mode.            */
#define MAPSM_MAX_PARAMS 8
typedef enum {
    MAPSM_PAT_BLOCK2D = 0,
    MAPSM_PAT_BLOCK2D_T = 1,
    MAPSM_PAT_OUT_SI = 2,
    MAPSM_PAT_INOUT_SI = 3
} mapsm_pattern;
typedef struct mapsm_matrix_s* mapsm_matrix;
/* One parameter's segment on the slab's device: rows [row0, row0+rows) of
 * the datum, `cols` columns, leading dimension `ld` (floats), `ptr` = element
 * (row0, 0) in device memory.                                               */
typedef struct {
    int64_t row0, rows, cols, ld;
    float* ptr;
} mapsm_segment;
/* The wrapper prototype (Fig 5): returns 0 on success.  `context`
 * is the caller's pointer (the ctx itself if the caller passed NULL).       */
typedef int (*mapsm_routine)(void* context, int slab, int device, void* stream, const mapsm_segment* segs,
                             int nsegs, const float* scalars, int nscalars);

mapsm_status mapsm_matrix_create(mapsm_ctx ctx, int64_t rows, int64_t cols, mapsm_matrix* out);
mapsm_status mapsm_matrix_destroy(mapsm_matrix m);
/* Bind: every process passes the FULL matrix (host or device memory,
 * leading dimension ld >= cols floats, copied).  It is uploaded to the
 * process's first slab; other slabs receive segments on demand.  Collective. */
mapsm_status mapsm_matrix_bind(mapsm_matrix m, const float* ptr, int64_t ld);
/* InvokeUnmodified (Table 2).  EINVAL: bad pattern / sizes (row-block
 * patterns need rows == task_rows), nparams outside 1..MAPSM_MAX_PARAMS.
 * ESTATE: an input was never bound or written.  ECUDA: the routine returned
 * nonzero.  `moved_bytes` (may be NULL): bytes this process moved for the task.*/
mapsm_status mapsm_invoke_unmodified(mapsm_ctx ctx, int64_t task_rows, mapsm_routine routine, void* context,
                                     int nparams, const mapsm_matrix* params, const int* patterns,
                                     const float* scalars, int nscalars, int64_t* moved_bytes);
/* Wait for the matrix's pending work (Wait, Table 2).                       */
mapsm_status mapsm_matrix_sync(mapsm_matrix m);
/* Gather the current version to `ptr` (host or device, ld floats) on `root`;
 * other processes pass NULL.  Collective; synchronises.                     */
mapsm_status mapsm_matrix_gather(mapsm_matrix m, float* ptr, int64_t ld, int root);
/* Built-in wrappers over cuBLAS (dlopen'ed libcublas.so.12, plain fp32
 * math, no TF32), for use as `routine` with context NULL:
 *   sgemm: params (A BLOCK2D m x k, B BLOCK2D_T k x n, C OUT_SI or INOUT_SI
 *          m x n), scalars (alpha, beta): C = alpha A B + beta C;
 *   saxpy: params (x BLOCK2D, y INOUT_SI, same shape), scalars (alpha):
 *          y = alpha x + y (Fig 5).                                         */
int mapsm_routine_sgemm(void* context, int slab, int device, void* stream, const mapsm_segment* segs, int nsegs,
                        const float* scalars, int nscalars);
int mapsm_routine_saxpy(void* context, int slab, int device, void* stream, const mapsm_segment* segs, int nsegs,
                        const float* scalars, int nscalars);

/* Copy only this process's own rows (same row range as mapsm_bind) to `ptr`;
 * not collective; synchronises.                                              */
mapsm_status mapsm_read(mapsm_grid grid, void* ptr, int64_t row_pitch_bytes);
/* Asynchronous Bind / read (the Bind and Gather of Table 2, P:L139/P:L157,
 * without the host waits): the copies (and the Life pack / unpack) are
 * enqueued on the grid's stream and the call returns; `ptr` must stay valid
 * and unmodified (bind) / unread (read) until mapsm_sync(grid) or any later
 * synchronisation of the grid's stream.  Use pinned host (or device) memory:
 * pageable memory makes the copies synchronous.  mapsm_bind_async is
 * collective like mapsm_bind (the first halo exchange is stream-ordered too);
 * mapsm_read_async copies this process's rows only.  Errors of the enqueued
 * work surface at mapsm_sync.                                               */
mapsm_status mapsm_bind_async(mapsm_grid grid, const void* ptr, int64_t row_pitch_bytes);
mapsm_status mapsm_read_async(mapsm_grid grid, void* ptr, int64_t row_pitch_bytes);

mapsm_status mapsm_grid_destroy(mapsm_grid grid);

/* ----------------------------------------------------------- introspection */

typedef struct {
    int64_t w, h;
    int dtype, op, radius, boundary;
    int world;               /* g: total slabs over all processes */
    int local_slabs;         /* slabs owned by this process */
    int64_t pitch_bytes;     /* device row pitch */
    int64_t generation;      /* iterations applied since bind */
    int64_t launches;        /* kernels launched by this grid since bind (all slabs) */
    int64_t exchanges;       /* halo messages received by this process since bind */
    int64_t device_bytes;    /* device memory owned by the grid */
    int used_graphs;         /* 1 if iterate replays CUDA graphs */
    int gens_per_pass;       /* generations per compute pass (K with MAPSM_OPT_DEEP_HALO, else 1) */
    int64_t halo_rows;       /* halo rows allocated above/below each slab (r, or K*r) */
    int64_t d;               /* planes of a Window(3D) grid, 0 for a 2-D grid */
} mapsm_grid_info;

mapsm_status mapsm_get_info(mapsm_grid grid, mapsm_grid_info* out);

/* Options (set before the first iterate; values are int64):
 *   MAPSM_OPT_GRAPHS      1 (default) capture iterations in CUDA graphs, 0 = direct launches
 *   MAPSM_OPT_GRAPH_ITERS iterations per captured graph (even, default 16)
 *   MAPSM_OPT_NO_EXCHANGE 1 = skip the halo exchange (bench only: measures
 *                         exchange exposure; results are then WRONG for g > 1)
 *   MAPSM_OPT_TIMING      1 = record CUDA events around every compute kernel
 *                         (forces direct launches); read with mapsm_get_timing
 *   MAPSM_OPT_PERSISTENT  1 (default) Life slabs without exchanged halos
 *                         (one slab): if the double-buffered slab fits in the
 *                         SMs' shared memory (w % 128 == 0; e.g. 8192^2), ONE
 *                         cooperative launch runs all n generations SMEM-
 *                         resident, K generations between neighbour-only halo
 *                         exchanges between SMs; else, if it fits in L2
 *                         (<= 64 MiB), up to 1024 generations per cooperative
 *                         launch with a grid barrier between generations;
 *                         2 = the grid-barrier kernel only; 0 = one launch per
 *                         generation
 *   MAPSM_OPT_EXCHANGE    MAPSM_EXCHANGE_COPY (default): boundary-row kernel,
 *                         then NCCL send/recv (multi-process) or peer
 *                         cudaMemcpyAsync (single process) on a side stream,
 *                         overlapped with the interior kernel.
 *                         MAPSM_EXCHANGE_P2P: ONE fused kernel per iteration
 *                         whose boundary CTAs store their rows straight into
 *                         the neighbours' halo rows (NVLink peer stores via
 *                         CUDA IPC, or same-process pointers) and signal them
 *                         through a device mailbox; the neighbour's CTAs that
 *                         need those rows wait on it.  Needs rows per slab >
 *                         2r and the TMA kernels (Life w % 128 == 0, conv
 *                         w % 4 == 0); set before bind.
 *   MAPSM_OPT_OWN_STREAM  1: the grid's slabs run on streams of their own
 *                         instead of the ctx stream (mapsm_grid_stream), so
 *                         several grids of one ctx overlap (e.g. one grid's
 *                         upload with another's compute and a third's
 *                         download); 0 (default): the ctx stream
 *   MAPSM_OPT_EXCHANGE_SMS  k in -1..64, one slab per process (multi-process
 *                         NCCL mode or the one-rank ring).  k > 0: the
 *                         concurrent-boundary schedule — generation t's
 *                         boundary rows and their NCCL exchange run on the
 *                         side stream on k SMs while the interior runs on
 *                         the other SMs; the interior of t waits only for
 *                         the boundary rows of t-1, the boundary rows of t
 *                         for the interior and halos of t-1.  k = 0: serial
 *                         (boundary, then exchange beside the interior — which
 *                         fills every SM, so NCCL's kernel waits for it).
 *                         -1 (default): 2 for Life, 4 for the 2-D conv r <= 4,
 *                         0 otherwise (measured).  With
 *                         MAPSM_EXCHANGE_P2P, k > 0 (explicit only) runs the
 *                         boundary launch with the fused peer stores beside
 *                         the interior instead of one fused launch.
 *   MAPSM_OPT_HOST_PACKED 1: Life grids (w % 32 == 0, else EUNSUPPORTED): the
 *                         host rows of mapsm_bind / mapsm_read / mapsm_gather
 *                         (and their _async forms) are bit-packed — w / 32
 *                         little-endian uint32 words per row, bit j of word k =
 *                         column 32k + j, nonzero bit = alive — i.e. the
 *                         device row format: one 2-D copy each way, 1/8 of
 *                         the u8 bytes over PCIe, no pack / unpack kernel.
 *                         Row pitch >= w / 8 bytes.  0 (default): u8 cells.
 *   MAPSM_OPT_DEEP_HALO   K > 1 (1 = off, default): the grid keeps K*r halo
 *                         rows per side and exchanges them once per pass of
 *                         K generations instead of r rows every generation
 *                         (the per-iteration exchange of
 *                         P:L461 made K-fold coarser).  Life: K in
 *                         {2,3,4,6,8}, ONE temporally blocked kernel per pass
 *                         (each CTA carries its rows through K generations in
 *                         registers: HBM traffic per generation drops K-fold).
 *                         fp32 conv (2-D and Window(3D)): K in 2..16, K
 *                         single-generation launches per pass over a
 *                         trapezoid of rows (the neighbours' halo rows are
 *                         recomputed locally).  Results are bit-identical to
 *                         the per-generation path.  Set before bind
 *                         (re-partitions and re-allocates: every slab needs
 *                         >= K*r rows when g > 1, else EINVAL).  n % K
 *                         trailing generations of an iterate call, slabs of
 *                         fewer than K rows, and w % 128 != 0 use the
 *                         per-generation kernels.  EUNSUPPORTED for non-Life
 *                         grids or other K; not combined with EXCHANGE_P2P
 *                         (the fused path then runs per generation).         */
typedef enum { MAPSM_EXCHANGE_COPY = 0, MAPSM_EXCHANGE_P2P = 1, MAPSM_EXCHANGE_CE = 2 } mapsm_exchange;
typedef enum {
    MAPSM_OPT_GRAPHS = 1,
    MAPSM_OPT_GRAPH_ITERS = 2,
    MAPSM_OPT_NO_EXCHANGE = 3,
    MAPSM_OPT_TIMING = 4,
    MAPSM_OPT_PERSISTENT = 5,
    MAPSM_OPT_EXCHANGE = 6,
    MAPSM_OPT_DEEP_HALO = 7,
    MAPSM_OPT_OWN_STREAM = 8,
    MAPSM_OPT_EXCHANGE_SMS = 9,
    MAPSM_OPT_HOST_PACKED = 10
} mapsm_option;

mapsm_status mapsm_set_option(mapsm_grid grid, mapsm_option opt, int64_t value);

/* With MAPSM_OPT_TIMING: summed device time (ms) and count of the bulk
 * ("interior" / whole-slab) compute kernels and of the boundary-row kernels
 * of local slab 0 since the option was set.  Synchronises.                   */
mapsm_status mapsm_get_timing(mapsm_grid grid, double* bulk_ms, int64_t* bulk_launches,
                              double* boundary_ms, int64_t* boundary_launches);

/* The compute stream of local slab `local_index` (a cudaStream_t).           */
mapsm_status mapsm_grid_stream(mapsm_grid grid, int local_index, void** stream);

/* Launch geometry of the last compute kernel launched for local slab
 * `local_index` (which = 0: the bulk / whole-slab launch, 1: the boundary-row
 * launch of Alg 1's exchange step), as the launcher issued it — so
 * tests can check that the kernel configuration they drive is the one the
 * bench times (e.g. rows per CTA >= 2 ring trips).  Pure host bookkeeping;
 * recorded at enqueue / graph-capture time.  Kernel ids: */
typedef enum {
    MAPSM_KERNEL_NONE = 0, MAPSM_KERNEL_LIFE_TMA = 1, MAPSM_KERNEL_LIFE_REG = 2, MAPSM_KERNEL_LIFE_ANYW = 3,
    MAPSM_KERNEL_LIFE_PERSIST = 4, MAPSM_KERNEL_LIFE_TB = 5, MAPSM_KERNEL_CONV_TMA = 6, MAPSM_KERNEL_CONV_REG = 7,
    MAPSM_KERNEL_CONV_GENERIC = 8, MAPSM_KERNEL_CONV_WIDE = 9, MAPSM_KERNEL_CONV3D = 10,
    MAPSM_KERNEL_LIFE_TB_PERSIST = 11, MAPSM_KERNEL_CONV_TB2 = 12
} mapsm_kernel;
typedef struct {
    int kernel;              /* mapsm_kernel */
    int threads;             /* threads per CTA */
    int smem_bytes;          /* dynamic shared memory per CTA */
    int ring_stages;         /* NS of the row ring (0: no ring) */
    int rows_per_stage;      /* input rows per ring stage */
    int consumer_warps;      /* consumer warps per CTA (ring kernels) */
    int gens_per_launch;     /* generations one launch advances */
    int64_t ctas;            /* CTAs launched */
    int64_t strips;          /* column strips per row (ring kernels) */
    /* ring kernels: over the CTAs that have work, the output rows of the
     * CTA's LONGEST (strip, row-run) segment (min and max over CTAs), the
     * CTA's total output rows (min), and the segment count over all CTAs   */
    int64_t min_cta_seg_rows, max_cta_seg_rows, min_cta_rows, segments;
} mapsm_launch_info;
mapsm_status mapsm_launch_query(mapsm_grid grid, int local_index, int which, mapsm_launch_info* out);

const char* mapsm_status_string(mapsm_status s);
const char* mapsm_last_error(void);
const char* mapsm_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MAPSM_H */
