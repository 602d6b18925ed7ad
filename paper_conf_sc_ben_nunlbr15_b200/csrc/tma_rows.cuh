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

struct RowStream {
    const uint32_t* in;   // owned row 0 of the input slab (4-byte elements)
    void* out;            // owned row 0 of the output slab
    int64_t pitch;        // row pitch in 4-byte elements
    int64_t rows;         // owned rows of the slab
    int64_t n;            // elements per row (multiple of 4)
    int64_t nstrips;
    int64_t begin[2], end[2];  // output-row bands of this launch
    int top_map, bot_map;
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

// Work distribution.  The (strip, output row) space of a band is flattened
// strip-major and split into gridDim.x equal contiguous ranges; a CTA's range
// is a short list of segments (one strip, a run of rows each), so every SM
// gets the same number of rows whatever the strip count (no idle SMs when
// 148 is not a multiple of the number of strips).
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
    const int band = blockIdx.y;
    it.rb = p.begin[band];
    it.nr = p.end[band] - it.rb;
    const int64_t T = p.nstrips * it.nr;
    it.pos = (int64_t)blockIdx.x * T / gridDim.x;
    it.hi = (int64_t)(blockIdx.x + 1) * T / gridDim.x;
    return it;
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

template <int NS>
__device__ __forceinline__ void produce_align(uint64_t* full, uint64_t* empty, RingPos& r) {
    while (r.stage != 0) {
        if (r.count >= NS) mbar_wait(&empty[r.stage], r.phase ^ 1u);
        mbar_arrive(&full[r.stage]);
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
template <int NC, int NS, bool WRAP_COLS, int EPL = 4>
__device__ __forceinline__ void produce(const RowStream& p, const Seg& t, uint8_t* smem, uint64_t* full,
                                        uint64_t* empty, int64_t y_first, int64_t n_in, RingPos& r) {
    using G = Geom<NC, EPL>;
    const uint32_t main_bytes = (uint32_t)(t.seg * 4) + (t.first_strip ? 0u : 16u) + (t.last_strip ? 0u : 16u);
    uint32_t tx = main_bytes;
    if (WRAP_COLS) tx += (t.first_strip ? 16u : 0u) + (t.last_strip ? 16u : 0u);
    const uint32_t* src_main = p.in + t.e0 - (t.first_strip ? 0 : 4);
    const uint32_t dst_main = t.first_strip ? 16u : 0u;
    for (int64_t j = 0; j < n_in; ++j) {
        // phase of the release we wait for = the previous round's (r.phase ^ 1)
        if (r.count >= NS) mbar_wait(&empty[r.stage], r.phase ^ 1u);
        const int64_t row = y_first + j;
        const int64_t rr = (row >= 0 && row < p.rows) ? row : map_row(p, row);
        const int64_t roff = rr * p.pitch;
        uint8_t* st = smem + r.stage * G::kStageBytes;
        uint64_t* bar = &full[r.stage];
        mbar_arrive_expect_tx(bar, tx);
        bulk_g2s(st + dst_main, src_main + roff, main_bytes, bar);
        if (WRAP_COLS) {
            if (t.first_strip) bulk_g2s(st, p.in + roff + p.n - 4, 16, bar);            // elements n-4..n-1
            if (t.last_strip) bulk_g2s(st + 16 + t.seg * 4, p.in + roff, 16, bar);     // elements 0..3
        }
        r.advance(NS);
    }
}

}  // namespace tma

// Host side: fill the band table of a RowStream for a launch of
// `ctas_per_sm` CTAs per SM; returns the grid x size (0 = nothing to do).
inline int64_t tma_plan_grid(tma::RowStream& p, const RowBands& b, int num_sms, int ctas_per_sm, int strip_elems) {
    p.nstrips = (p.n + strip_elems - 1) / strip_elems;
    int64_t maxT = 0;
    for (int i = 0; i < 2; ++i) p.begin[i] = p.end[i] = 0;
    for (int i = 0; i < b.nbands; ++i) {
        p.begin[i] = b.begin[i];
        p.end[i] = b.end[i];
        const int64_t T = p.nstrips * (b.end[i] - b.begin[i]);
        if (T > maxT) maxT = T;
    }
    int64_t ctas = (int64_t)num_sms * ctas_per_sm / (b.nbands > 0 ? b.nbands : 1);
    if (ctas > maxT) ctas = maxT;
    return ctas;
}

}  // namespace mapsm
