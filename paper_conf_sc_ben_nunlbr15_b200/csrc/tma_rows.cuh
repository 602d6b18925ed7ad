// tma_rows.cuh — the row-streaming pipeline shared by the Life and conv
// kernels (sm_100a): a producer warp streams successive rows of a CTA's column
// strip into an NS-stage shared-memory ring with TMA bulk copies
// (cp.async.bulk, completion counted on one mbarrier per stage); consumer
// warps wait on the stage's "full" barrier, read, and release it on its
// "empty" barrier.  This is the Window(2D) input container of the paper
// (Shared Containers, §4; Window2D::SharedData)
// re-implemented with Blackwell's asynchronous bulk-copy engine: the data in
// flight lives in shared memory, so the pipeline depth does not cost
// registers or occupancy.
//
// Stage layout (4-byte elements, E = NC*128 elements = NC*512 bytes):
//   [0,4)        left margin: the 4 elements left of the strip (the previous
//                strip's tail, or at the row start the WRAP source = the
//                row's last 4 elements; CLAMP/ZERO: not written, the
//                consumer synthesises it)
//   [4, 4+seg)   the strip
//   [4+seg, +4)  right margin: the 4 elements right of the strip (next strip,
//                or at the row end the WRAP source = the row's first 4)
// A 16-byte margin covers every radius this path supports (Life r=1 needs one
// bit; conv r <= 4 needs <= 4 floats).
#pragma once
#include <cuda_runtime.h>
#include <stdlib.h>
#include <stdint.h>

#include "kernels.h"

namespace mapsm {
namespace tma {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done = 0;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    } while (!done);
}

// TMA bulk copy global -> shared (16-byte aligned, size a multiple of 16).
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// NC consumer warps, EPL 4-byte elements per lane (4 = one 16-byte vector).
template <int NC, int EPL = 4>
struct Geom {
    static constexpr int kStripElems = NC * 32 * EPL;         // 4-byte elements per strip
    static constexpr int kStageBytes = kStripElems * 4 + 32;  // + 16 B margin each side
};

constexpr int kMaxBands = 3;

// Fused halo exchange over peer memory (MAPSM_OPT_EXCHANGE_P2P): the CTAs
// that compute a slab's first / last r rows also store them into the
// neighbours' halo rows (NVLink peer stores, or plain stores between slabs
// on one device) and then add the number of rows delivered to the
// neighbour's mailbox; a CTA that needs a halo row waits until its own
// mailbox shows this generation's delivery.  Counters are monotonic; the
// generation is kept in device memory so CUDA-graph replays stay correct.
struct Mailbox {
    unsigned long long gen;  // iterations completed since bind (incremented by the last CTA of each launch)
    unsigned int done;       // CTAs finished in the current launch
    unsigned int recv_top;   // rows delivered into my top halo since bind (all strips)
    unsigned int recv_bot;   // rows delivered into my bottom halo since bind
    unsigned int pad[3];
};

struct HaloLink {
    Mailbox* mine;           // null: no fused exchange in this launch
    uint32_t* dst_up;        // up neighbour's `out`-parity buffer at its bottom-halo row 0 (null: no up link)
    uint32_t* dst_down;      // down neighbour's `out`-parity buffer at its top-halo row -r (null: no down link)
    unsigned int* sig_up;    // &up.mailbox.recv_bot
    unsigned int* sig_down;  // &down.mailbox.recv_top
    int wait_top, wait_bot;  // my top / bottom halo is delivered by a neighbour
    int r;                   // rows per delivery
    int ce;                  // copy-engine exchange (MAPSM_EXCHANGE_CE): recv_top / recv_bot are the
                             // neighbours' generation counts, copied after their rows; wait for >= gen
};

struct RowStream {
    const uint32_t* in;   // owned row 0 of the input slab (4-byte elements)
    void* out;            // owned row 0 of the output slab
    int64_t pitch;        // row pitch in 4-byte elements
    int64_t rows;         // owned rows of the slab
    int64_t n;            // elements per row (multiple of 4)
    int64_t nstrips;
    int nbands;
    int64_t begin[kMaxBands], end[kMaxBands];  // output-row bands of this launch
    int cta_begin[kMaxBands + 1];              // CTAs [cta_begin[b], cta_begin[b+1]) work on band b
    int link_ctas;                             // fused launches: CTAs [0, link_ctas) count the launch (gen)
    int top_map, bot_map;
    HaloLink link;
};

__device__ __forceinline__ int64_t map_row(const RowStream& p, int64_t y) {
    if (y < 0) {
        if (p.top_map == ROWMAP_WRAP) {
            y %= p.rows;
            if (y < 0) y += p.rows;
        } else if (p.top_map == ROWMAP_CLAMP) {
            y = 0;
        }
    } else if (y >= p.rows) {
        if (p.bot_map == ROWMAP_WRAP) y %= p.rows;
        else if (p.bot_map == ROWMAP_CLAMP) y = p.rows - 1;
    }
    return y;  // ROWMAP_HALO: the halo row itself (exchanged or zeroed)
}

// Work distribution.  Each band owns a range of CTAs (1-D grid).  The
// (strip, output row) space of a band is flattened strip-major and split into
// equal contiguous ranges, one per CTA of the band; a CTA's range is a short
// list of segments (one strip, a run of rows each), so every SM gets the same
// number of rows whatever the strip count (no idle SMs when 148 is not a
// multiple of the number of strips).
struct Seg {
    int64_t ys, ye;     // output rows [ys, ye)
    int64_t e0, seg;    // first element and element count of the strip
    bool first_strip, last_strip;
};

struct SegIter {
    int64_t pos, hi, nr, rb;
};

__device__ __forceinline__ SegIter seg_iter(const RowStream& p) {
    SegIter it;
    int band = 0;
    while (band + 1 < p.nbands && (int)blockIdx.x >= p.cta_begin[band + 1]) ++band;
    const int64_t c = (int64_t)blockIdx.x - p.cta_begin[band];
    const int64_t C = p.cta_begin[band + 1] - p.cta_begin[band];
    it.rb = p.begin[band];
    it.nr = p.end[band] - it.rb;
    const int64_t T = p.nstrips * it.nr;
    it.pos = C > 0 ? c * T / C : 0;
    it.hi = C > 0 ? (c + 1) * T / C : 0;
    return it;
}

// ---- fused exchange helpers -------------------------------------------------

__device__ __forceinline__ unsigned int ld_acquire_sys(const unsigned int* p) {
    unsigned int v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Producer side: before the TMA load of a halo row, wait for its delivery.
// Bounded spin: a protocol failure traps (kernel error) instead of hanging.
// The counters and the target (gen * r * nstrips) are taken mod 2^32; the
// comparison is wrap-safe because a counter is never more than one
// generation's deliveries (r * nstrips << 2^31) away from the target.
__device__ __forceinline__ void wait_delivery(const unsigned int* counter, unsigned int target) {
    unsigned int spins = 0;
    while ((int)(ld_acquire_sys(counter) - target) < 0) {
        __nanosleep(64);
        if (++spins > (1u << 26)) __trap();  // ~seconds: the neighbour never delivered
    }
    asm volatile("fence.proxy.async.global;" ::: "memory");  // make the peer's stores visible to TMA reads
}

// Consumer side, after this CTA's consumer warps stored `rows_sent` boundary
// rows into a neighbour's halo: one thread publishes them (system-scope
// release; the named barrier orders the other warps' stores before it).
__device__ __forceinline__ void publish_delivery(unsigned int* counter, unsigned int rows_sent, int consumers) {
    asm volatile("bar.sync 1, %0;" ::"r"(consumers * 32) : "memory");
    if (threadIdx.x == 0) {
        __threadfence_system();
        asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(counter), "r"(rows_sent) : "memory");
    }
}

// At exit the last of the launch's boundary-band CTAs (CTAs [0, n_link):
// the ones that read gen, at their start) advances gen; interior CTAs of a
// fused launch leave without counting.  The producer warp only arrives
// (named barrier 2) and leaves, so the consumer code stays free of CTA-wide
// divergence; the consumers wait on barrier 2, then thread 0 counts.
__device__ __forceinline__ void finish_launch_producer(int threads, int n_link) {
    if ((int)blockIdx.x >= n_link) return;
    __syncwarp();
    asm volatile("bar.arrive 2, %0;" ::"r"(threads) : "memory");
}

__device__ __forceinline__ void finish_launch_consumers(Mailbox* mb, int threads, int n_link) {
    if ((int)blockIdx.x >= n_link) return;
    asm volatile("bar.sync 2, %0;" ::"r"(threads) : "memory");
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(&mb->done, 1u) == (unsigned)n_link - 1) {
            mb->done = 0;
            __threadfence();
            atomicAdd(&mb->gen, 1ull);
        }
    }
}

template <int NC, int EPL = 4>
__device__ __forceinline__ bool seg_next(const RowStream& p, SegIter& it, Seg& s) {
    if (it.pos >= it.hi) return false;
    const int64_t strip = it.pos / it.nr, r0 = it.pos % it.nr;
    const int64_t r1 = (it.nr - r0 < it.hi - it.pos) ? it.nr : r0 + (it.hi - it.pos);
    s.ys = it.rb + r0;
    s.ye = it.rb + r1;
    it.pos += r1 - r0;
    using G = Geom<NC, EPL>;
    s.e0 = strip * G::kStripElems;
    s.seg = p.n - s.e0 < G::kStripElems ? p.n - s.e0 : G::kStripElems;
    s.first_strip = strip == 0;
    s.last_strip = s.e0 + s.seg == p.n;
    return true;
}

// Programmatic dependent launch (the stencil launches of consecutive
// generations): a CTA of generation t+1 may be scheduled while generation t
// drains; it sets up its shared memory, then waits here until generation t
// has completed and flushed (it reads t's output and overwrites t's input),
// and lets generation t+2 start launching.  A no-op for launches without the
// programmatic-serialization attribute.
__device__ __forceinline__ void pdl_wait_and_release() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" :::);
}

template <int NS>
__device__ __forceinline__ void init_barriers(uint64_t* full, uint64_t* empty, int consumers) {
    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], consumers);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
}

// Stage counter alignment between segments: every segment starts on a stage
// index that is a multiple of NS (so the consumers' unrolled trips use
// compile-time stage numbers); the skipped stages run an empty round
// (producer arrives without data, consumers just release) to keep every
// stage's barrier phases in step.
// The CTA-wide ring position: stage index and the phase parity of the
// current round (flips every NS rows).  Kept incrementally (no divisions).
struct RingPos {
    int stage = 0;
    uint32_t phase = 0;
    int64_t count = 0;  // rows (including empty alignment rounds) so far
    __device__ __forceinline__ void advance(int ns) {
        ++count;
        if (++stage == ns) {
            stage = 0;
            phase ^= 1u;
        }
    }
};

// The producer is the first PL lanes of the producer warp; lane l issues the
// rows whose ring position is l mod PL (each lane tracks the whole ring
// position, so stage and phase are always known).  Measured
// (profiles/r01_producer_lanes.txt): PL = 2 speeds up the 5x5 conv (8
// strips per row, 3 bulk copies per row at the row ends) by 6%, while Life
// (one whole-row copy per row) is fastest with PL = 1.
template <int NS, int PL>
__device__ __forceinline__ void produce_align(uint64_t* full, uint64_t* empty, RingPos& r, int plane) {
    while (r.stage != 0) {
        if ((int)(r.count % PL) == plane) {
            if (r.count >= NS) mbar_wait(&empty[r.stage], r.phase ^ 1u);
            mbar_arrive(&full[r.stage]);
        }
        r.advance(NS);
    }
}

template <int NS>
__device__ __forceinline__ void consume_align(uint64_t* full, uint64_t* empty, RingPos& r, int lane) {
    while (r.stage != 0) {
        mbar_wait(&full[r.stage], r.phase);
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[r.stage]);
        r.advance(NS);
    }
}

// Producer (one thread): stream input rows y_first .. y_first+n_in-1 of the
// segment's strip into the ring, continuing the CTA-wide row counter i.  Row
// i goes to stage i % NS; before reusing a stage it waits until all consumer
// warps released the row that occupied it.
template <int NC, int NS, bool WRAP_COLS, int EPL, int PL>
__device__ __forceinline__ void produce(const RowStream& p, const Seg& t, uint8_t* smem, uint64_t* full,
                                        uint64_t* empty, int64_t y_first, int64_t n_in, RingPos& r,
                                        unsigned int halo_target, int plane) {
    using G = Geom<NC, EPL>;
    // A strip that is the whole row needs no margin copies: under WRAP the
    // consumers read the row's other end from the stage itself.
    const bool whole = t.first_strip && t.last_strip;
    const bool wrap_l = WRAP_COLS && t.first_strip && !whole;
    const bool wrap_r = WRAP_COLS && t.last_strip && !whole;
    const uint32_t main_bytes = (uint32_t)(t.seg * 4) + (t.first_strip ? 0u : 16u) + (t.last_strip ? 0u : 16u);
    const uint32_t tx = main_bytes + (wrap_l ? 16u : 0u) + (wrap_r ? 16u : 0u);
    const int64_t src_off = t.e0 - (t.first_strip ? 0 : 4);  // element offset of the main copy in a row
    const uint32_t dst_main = t.first_strip ? 16u : 0u;
    const uint32_t dst_r = 16u + (uint32_t)(t.seg * 4);
    // this lane's first row, then every kProducerLanes-th row
    int64_t j = (plane - r.count % PL + PL) % PL;
    for (int64_t k = 0; k < j && k < n_in; ++k) r.advance(NS);
    const uint32_t* rowp = p.in + (y_first + j) * p.pitch;  // in-slab rows: pointer walk
    const int64_t rstep = (int64_t)PL * p.pitch;
    for (; j < n_in; j += PL, rowp += rstep) {
        // phase of the release we wait for = the previous round's (r.phase ^ 1)
        if (r.count >= NS) mbar_wait(&empty[r.stage], r.phase ^ 1u);
        const int64_t row = y_first + j;
        const uint32_t* rp = rowp;
        if (row < 0 || row >= p.rows) {  // halo / wrapped / clamped rows: slab edges only
            if (row < 0 && p.link.wait_top) wait_delivery(&p.link.mine->recv_top, halo_target);
            if (row >= p.rows && p.link.wait_bot) wait_delivery(&p.link.mine->recv_bot, halo_target);
            rp = p.in + map_row(p, row) * p.pitch;
        }
        uint8_t* st = smem + r.stage * G::kStageBytes;
        uint64_t* bar = &full[r.stage];
        mbar_arrive_expect_tx(bar, tx);
        bulk_g2s(st + dst_main, rp + src_off, main_bytes, bar);
        if (wrap_l) bulk_g2s(st, rp + p.n - 4, 16, bar);   // elements n-4..n-1
        if (wrap_r) bulk_g2s(st + dst_r, rp, 16, bar);     // elements 0..3
        // advance the ring position past this row and the other lanes' rows
        for (int q = 0; q < PL && j + q < n_in; ++q) r.advance(NS);
    }
}

}  // namespace tma

// Host side: copy a FusedLink (or none) into the kernel parameters.
inline void tma_set_link(tma::RowStream& p, const FusedLink* l, int r) {
    p.link.mine = l ? static_cast<tma::Mailbox*>(l->mailbox) : nullptr;
    p.link.dst_up = l ? static_cast<uint32_t*>(l->dst_up) : nullptr;
    p.link.dst_down = l ? static_cast<uint32_t*>(l->dst_down) : nullptr;
    p.link.sig_up = l ? l->sig_up : nullptr;
    p.link.sig_down = l ? l->sig_down : nullptr;
    p.link.wait_top = l ? l->wait_top : 0;
    p.link.wait_bot = l ? l->wait_bot : 0;
    p.link.r = r;
    p.link.ce = l ? l->ce : 0;
}

// The producer's wait target for halo rows: rows delivered since bind
// (peer stores) or the neighbour's generation count (copy engine).
__device__ __forceinline__ unsigned int halo_wait_target(const tma::HaloLink& L, int64_t nstrips) {
    const unsigned long long gen = L.mine->gen;
    return L.ce ? (unsigned int)gen : (unsigned int)(gen * (unsigned long long)(L.r * nstrips));
}

// Host side: fill the band table of a RowStream for a launch of
// `ctas_per_sm` CTAs per SM; returns the 1-D grid size (0 = nothing to do).
// Plain launches split the resident CTAs evenly over the bands; fused
// launches (bands = top boundary, bottom boundary, interior) put the boundary
// bands first with one CTA per 8 strips, the interior taking the rest.
inline int64_t tma_plan_grid(tma::RowStream& p, const RowBands& b, int num_sms, int ctas_per_sm, int strip_elems,
                             bool boundary_first = false) {
    p.nstrips = (p.n + strip_elems - 1) / strip_elems;
    p.nbands = b.nbands;
    // boundary-first needs an interior band last (a boundary-only launch —
    // the concurrent schedules' side-stream launch — splits evenly)
    if (boundary_first && b.nbands > 0) {
        int64_t other = 0;
        for (int i = 0; i + 1 < b.nbands; ++i)
            other = other > b.end[i] - b.begin[i] ? other : b.end[i] - b.begin[i];
        if (b.end[b.nbands - 1] - b.begin[b.nbands - 1] <= other) boundary_first = false;
    }
    for (int i = 0; i < tma::kMaxBands; ++i) p.begin[i] = p.end[i] = 0;
    const int64_t resident = (int64_t)num_sms * ctas_per_sm;
    int64_t total = 0;
    p.cta_begin[0] = 0;
    for (int i = 0; i < b.nbands; ++i) {
        p.begin[i] = b.begin[i];
        p.end[i] = b.end[i];
        const int64_t T = p.nstrips * (b.end[i] - b.begin[i]);
        int64_t c;
        if (boundary_first && i + 1 < b.nbands) {
            // few CTAs for the r boundary rows (they finish long before the
            // interior: a neighbour's next launch never waits on them), so
            // the interior keeps almost every SM (one CTA per strip took 16
            // of 148 SMs from the conv 5x5 interior: 481 us vs 381 plain)
            c = (p.nstrips + 7) / 8;
        } else if (boundary_first) {
            c = resident - total;
        } else {
            c = resident / (b.nbands > 0 ? b.nbands : 1);
        }
        if (c > T) c = T;
        if (c < 1 && T > 0) c = 1;
        if (T <= 0) c = 0;
        total += c;
        p.cta_begin[i + 1] = (int)total;
    }
    for (int i = b.nbands; i < tma::kMaxBands; ++i) p.cta_begin[i + 1] = (int)total;
    // who counts a fused launch: the boundary bands' CTAs (all of them when
    // the launch has no interior band)
    p.link_ctas = boundary_first && b.nbands > 1 ? p.cta_begin[b.nbands - 1] : (int)total;
    return total;
}

// Host side: launch a ring kernel with programmatic dependent launch (the
// kernel calls tma::pdl_wait_and_release() after its shared-memory setup),
// so generation t+1's CTAs are scheduled while generation t drains.
// MAPSM_NO_PDL=1 turns it off (A/B measurements).
inline bool tma_pdl_enabled() {
    static const bool on = getenv("MAPSM_NO_PDL") == nullptr;
    return on;
}

template <typename Kernel, typename Param>
inline cudaError_t tma_launch(Kernel kernel, unsigned grid, unsigned block, int smem, cudaStream_t s,
                              const Param& p, bool pdl = true) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = (size_t)smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl && tma_pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, p);
}

// Host side: describe a ring-kernel launch for mapsm_launch_query.
inline void tma_record(LaunchRec* rec, int kernel, const tma::RowStream& p, int64_t ctas, int threads, int smem,
                       int ns, int rows_per_stage, int consumer_warps, int gens = 1) {
    if (!rec) return;
    rec->kernel = kernel;
    rec->ctas = ctas;
    rec->threads = threads;
    rec->smem = smem;
    rec->ring_stages = ns;
    rec->rows_per_stage = rows_per_stage;
    rec->consumer_warps = consumer_warps;
    rec->nstrips = p.nstrips;
    rec->nbands = p.nbands;
    for (int i = 0; i < 3; ++i) {
        rec->begin[i] = p.begin[i];
        rec->end[i] = p.end[i];
    }
    for (int i = 0; i < 4; ++i) rec->cta_begin[i] = p.cta_begin[i];
    rec->gens = gens;
}

}  // namespace mapsm
