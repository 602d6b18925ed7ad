// life.cu — Game of Life on bit-packed rows, sm_100a.
//
// Path row a4/a5 of SURVEY §8(a): one synchronous Life generation
// (B3/S23 on the 3x3 Window, §4, Fig 2b) over a row slab.
//
// Design.  The paper's kernel stages a 3x3 window per cell in
// shared memory and gives each thread 4x2 cells of ILP.
// On B200 the path is HBM-bound, so this kernel instead:
//   * stores 32 cells per 32-bit word (0.25 B/cell moved per generation:
//     1 bit read + 1 bit written) — 32x less traffic than a byte per cell;
//   * gives each lane V consecutive words (one 128-bit LDG/STG per row) and
//     streams a warp down a chunk of rows: each input row is loaded once,
//     its 3-cell horizontal sum (2 bit-planes, 2 funnel shifts + 2 LOP3 per
//     word) is computed once and reused by the 3 output rows that need it
//     (register blocking over rows, the paper's ILPY taken to the whole chunk);
//   * gets the neighbour bits across lane boundaries with warp shuffles and
//     across warp/row ends with one extra 4-byte load (edge lanes only);
//   * keeps P rows of loads in flight per lane (software pipeline) so that
//     ~48 KB/SM is outstanding — what HBM3e needs at ~6.5 TB/s;
//   * combines the three row sums bit-sliced: 8 LOP3 per output word.
// Rows are split into chunks so the grid is exactly one wave of resident
// warps (148 SMs x occupancy), and chunks are long (~100 rows) so the 2 extra
// input rows per chunk cost ~2% extra reads (L2 hits).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <type_traits>

#include "kernels.h"
#include "tma_rows.cuh"

namespace mapsm {
namespace {

constexpr int kThreads = 256;
constexpr unsigned kFull = 0xffffffffu;
#ifndef MAPSM_LIFE_P
#define MAPSM_LIFE_P 3
#endif
constexpr int kLifeP = MAPSM_LIFE_P;  // rows of loads in flight per lane
#ifndef MAPSM_TMA_NS
#define MAPSM_TMA_NS 24
#endif
constexpr int kTmaNS = MAPSM_TMA_NS;  // pipeline stages (rows in flight per CTA)
#ifndef MAPSM_TMA_CTAS
#define MAPSM_TMA_CTAS 0
#endif
constexpr int kTmaCtasPerSm = MAPSM_TMA_CTAS;  // 0 = 16 consumer warps per SM

struct LifeParams {
    const uint32_t* in;   // owned row 0 of input
    uint32_t* out;        // owned row 0 of output
    int64_t pitch_w;      // row pitch in 32-bit words
    int64_t rows;
    int64_t nw;           // 32-bit words per row (w / 32)
    int64_t nvec;         // nw / V
    int64_t warps_per_row;
    int64_t begin[2], end[2], nchunks[2];
    int top_map, bot_map, col_mode;
};

__device__ __forceinline__ uint32_t maj3(uint32_t a, uint32_t b, uint32_t c) {
    return (a & b) | (a & c) | (b & c);
}

template <class Prm>
__device__ __forceinline__ int64_t map_row(const Prm& p, int64_t y) {
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
    return y;
}

template <int V>
struct Fetch {
    uint32_t x[V];
    uint32_t le, re;  // edge words (only meaningful on edge lanes)
};

// COH = coherent loads (ld.global.cg, L2 only): required by the persistent
// kernel, whose input buffer was written by other SMs earlier in the same
// launch; the one-generation kernels use the read-only path (ld.global.nc).
template <bool COH>
__device__ __forceinline__ uint32_t ld_word(const uint32_t* p) {
    if constexpr (COH) return __ldcg(p);
    else return __ldg(p);
}

template <int V, bool COH = false>
__device__ __forceinline__ void load_vec(const uint32_t* ptr, uint32_t (&x)[V]) {
    if constexpr (V == 4) {
        uint4 v = COH ? __ldcg(reinterpret_cast<const uint4*>(ptr)) : __ldg(reinterpret_cast<const uint4*>(ptr));
        x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
    } else {
        uint2 v = COH ? __ldcg(reinterpret_cast<const uint2*>(ptr)) : __ldg(reinterpret_cast<const uint2*>(ptr));
        x[0] = v.x; x[1] = v.y;
    }
}

template <int V>
__device__ __forceinline__ void store_vec(uint32_t* ptr, const uint32_t (&x)[V]) {
    if constexpr (V == 4) {
        *reinterpret_cast<uint4*>(ptr) = make_uint4(x[0], x[1], x[2], x[3]);
    } else {
        *reinterpret_cast<uint2*>(ptr) = make_uint2(x[0], x[1]);
    }
}

// Per-lane constants of the column layout.  Lane l of a warp owns words
// [vi*V, vi*V+V) of every row; the bit just left of its first word comes from
// lane l-1 by shuffle (or, on lane 0 / column 0, from its own 4-byte load or
// the boundary rule), the bit right of its last word likewise from lane l+1.
struct LaneCols {
    int64_t vi;           // vector index of this lane within the row
    bool active;          // vi < nvec
    bool need_l, need_r;  // this lane supplies its own edge word instead of a shuffle
    bool load_l, load_r;  // ... and loads it (WRAP, or an interior warp edge)
    bool synth_l, synth_r;  // ... or synthesises it (CLAMP/ZERO at column 0 / w-1)
    int64_t l_off, r_off;   // word offsets of the loaded edge words within a row
};

template <int V, bool COH = false>
__device__ __forceinline__ void fetch_row(const LaneCols& c, const uint32_t* row, Fetch<V>& f) {
    if (c.active) {
        load_vec<V, COH>(row + c.vi * V, f.x);
    } else {
#pragma unroll
        for (int i = 0; i < V; ++i) f.x[i] = 0u;
    }
    f.le = c.load_l ? ld_word<COH>(row + c.l_off) : 0u;
    f.re = c.load_r ? ld_word<COH>(row + c.r_off) : 0u;
}

// Horizontal 3-cell sums of one row: s0 = parity, s1 = carry (L + x + R).
template <int V, int CM>
__device__ __forceinline__ void row_sums(const LaneCols& c, const Fetch<V>& f, uint32_t (&s0)[V],
                                         uint32_t (&s1)[V]) {
    const uint32_t up = __shfl_up_sync(kFull, f.x[V - 1], 1);
    const uint32_t dn = __shfl_down_sync(kFull, f.x[0], 1);
    uint32_t lw = c.need_l ? f.le : up;  // ZERO: f.le == 0 on the synthesising lane
    uint32_t rw = c.need_r ? f.re : dn;
    if (CM == COL_CLAMP) {
        if (c.synth_l) lw = f.x[0] << 31;       // column -1 := column 0
        if (c.synth_r) rw = f.x[V - 1] >> 31;   // column w := column w-1
    }
#pragma unroll
    for (int i = 0; i < V; ++i) {
        const uint32_t ls = (i == 0) ? lw : f.x[i - 1];
        const uint32_t rs = (i == V - 1) ? rw : f.x[i + 1];
        const uint32_t L = __funnelshift_l(ls, f.x[i], 1);  // bit j <- column j-1
        const uint32_t R = __funnelshift_r(f.x[i], rs, 1);  // bit j <- column j+1
        s0[i] = L ^ f.x[i] ^ R;
        s1[i] = maj3(L, f.x[i], R);
    }
}

// N9 = a + b + c (each a 2-bit row sum incl. the centre column), next =
// (N9 == 3) | (alive & N9 == 4)  ==  B3/S23 with N8 = N9 - alive.
//   s0 = a0^b0^c0, k = maj(a0,b0,c0)  -> N9 = s0 + 2(k + t) + 4u
//   t  = a1^b1^c1, u = maj(a1,b1,c1)
//   C  = [k + t + 2u in {1,2}] = u ^ (k|t)
//   D  = s0 ? (k^t) : alive & !(k^t)  = !(s0 ^ m) & (s0 | alive),  m = k^t
//   next = C & D
__device__ __forceinline__ uint32_t life_word(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1,
                                              uint32_t c0, uint32_t c1, uint32_t alive) {
    const uint32_t s0 = a0 ^ b0 ^ c0;
    const uint32_t k = maj3(a0, b0, c0);
    const uint32_t t = a1 ^ b1 ^ c1;
    const uint32_t u = maj3(a1, b1, c1);
    const uint32_t m = k ^ t;
    const uint32_t C = u ^ (k | t);
    const uint32_t D = ~(s0 ^ m) & (s0 | alive);
    return C & D;
}

template <int V, int CM>
struct LifeRowState {
    uint32_t a0[V], a1[V], b0[V], b1[V], alive[V];
};

// One output row: consume input row y+1 (fetch f), combine with the sums of
// rows y-1 (a) and y (b), store, rotate.
template <int V, int CM>
__device__ __forceinline__ void life_row(const LaneCols& c, const Fetch<V>& f, LifeRowState<V, CM>& st,
                                         uint32_t* out_row) {
    uint32_t c0[V], c1[V], o[V];
    row_sums<V, CM>(c, f, c0, c1);
#pragma unroll
    for (int i = 0; i < V; ++i) o[i] = life_word(st.a0[i], st.a1[i], st.b0[i], st.b1[i], c0[i], c1[i], st.alive[i]);
    if (c.active) store_vec<V>(out_row, o);
#pragma unroll
    for (int i = 0; i < V; ++i) {
        st.a0[i] = st.b0[i]; st.a1[i] = st.b1[i];
        st.b0[i] = c0[i]; st.b1[i] = c1[i];
        st.alive[i] = f.x[i];
    }
}

// One warp: output rows [ys, ye) of vector strip `strip`, reading `in`,
// writing `out` (geometry and boundary modes from p).
template <int V, int P, int CM, bool COH>
__device__ __forceinline__ void life_warp_rows(const LifeParams& p, const uint32_t* in, uint32_t* out,
                                               int64_t strip, int64_t ys, int64_t ye) {
    const int lane = threadIdx.x & 31;
    LaneCols c;
    c.vi = strip * 32 + lane;
    c.active = c.vi < p.nvec;
    const bool first = c.vi == 0, last = c.vi == p.nvec - 1;
    c.need_l = c.active && (lane == 0 || first);
    c.need_r = c.active && (lane == 31 || last);
    c.synth_l = c.need_l && first && CM != COL_WRAP;
    c.synth_r = c.need_r && last && CM != COL_WRAP;
    c.load_l = c.need_l && !c.synth_l;
    c.load_r = c.need_r && !c.synth_r;
    c.l_off = first ? p.nw - 1 : c.vi * V - 1;
    c.r_off = last ? 0 : (c.vi + 1) * V;

    // Rows ys..ye-1 lie inside the slab; only rows ys-1 and ye can be halo
    // rows (or wrapped / clamped rows), so they are resolved once here and
    // the streaming loop below is branch-free.
    const uint32_t* row_top = in + map_row(p, ys - 1) * p.pitch_w;
    const uint32_t* row_bot = in + map_row(p, ye) * p.pitch_w;
    const uint32_t* row_ys = in + ys * p.pitch_w;
    auto rowp = [&](int64_t y) { return y < ye ? row_ys + (y - ys) * p.pitch_w : row_bot; };

    Fetch<V> fa, fb;
    fetch_row<V, COH>(c, row_top, fa);
    fetch_row<V, COH>(c, row_ys, fb);
    Fetch<V> ring[P];
#pragma unroll
    for (int k = 0; k < P; ++k) fetch_row<V, COH>(c, rowp(ys + 1 + k), ring[k]);

    LifeRowState<V, CM> st;
    row_sums<V, CM>(c, fa, st.a0, st.a1);
    row_sums<V, CM>(c, fb, st.b0, st.b1);
#pragma unroll
    for (int i = 0; i < V; ++i) st.alive[i] = fb.x[i];

    uint32_t* out_row = out + ys * p.pitch_w + c.vi * V;
    int64_t y = ys;
    // Steady state: P output rows per trip, P rows of loads always in flight.
    // Fetches past row ye re-read row ye (harmless, L1/L2 hits).
    for (; y + P <= ye; y += P) {
#pragma unroll
        for (int k = 0; k < P; ++k) {
            const Fetch<V> f = ring[k];
            fetch_row<V, COH>(c, rowp(y + k + 1 + P), ring[k]);
            life_row<V, CM>(c, f, st, out_row);
            out_row += p.pitch_w;
        }
    }
    // Tail: fewer than P rows left; their input rows are already in the ring.
#pragma unroll
    for (int k = 0; k < P; ++k) {
        if (y + k < ye) {
            life_row<V, CM>(c, ring[k], st, out_row);
            out_row += p.pitch_w;
        }
    }
}

template <int V, int P, int CM>
__global__ void __launch_bounds__(kThreads) life_step_kernel(const __grid_constant__ LifeParams p) {
    const int64_t warp_gid = (int64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const int band = blockIdx.y;
    const int64_t nchunks = p.nchunks[band];
    const int64_t strip = warp_gid % p.warps_per_row;
    const int64_t chunk = warp_gid / p.warps_per_row;
    if (chunk >= nchunks) return;  // whole warp exits together
    const int64_t rb = p.begin[band], nr = p.end[band] - rb;
    const int64_t ys = rb + chunk * nr / nchunks;
    const int64_t ye = rb + (chunk + 1) * nr / nchunks;
    if (ys >= ye) return;
    life_warp_rows<V, P, CM, false>(p, p.in, p.out, strip, ys, ye);
}

// ------------------------------------------------ persistent multi-generation
// For slabs with no exchanged halo whose double buffer fits in L2 (BASELINE
// configs[0]/[1]: 64^2 and 8192^2 Life), one cooperative launch runs all n
// generations: every warp keeps its (strip, row chunk) and a grid-wide
// barrier separates generations.  This removes the per-generation launch and
// pipeline-fill latency that dominate when a generation is only ~2 us of work.
__device__ __forceinline__ void grid_barrier(unsigned int* count, unsigned int target) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(count) : "memory");
        unsigned int v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(count) : "memory");
        } while (v < target);
        __threadfence();
    }
    __syncthreads();
}

// 256-thread CTAs, as many per SM as fit (measured: one 768-thread CTA per
// SM, i.e. 3.4x fewer barrier arrivals, was 13% slower — register cap spills).
constexpr int kPersistThreads = kThreads;

template <int V, int P, int CM>
__global__ void __launch_bounds__(kPersistThreads) life_persist_kernel(const __grid_constant__ LifeParams p,
                                                                      int64_t n_gen, unsigned int* bar) {
    const int64_t warp_gid = (int64_t)blockIdx.x * (kPersistThreads / 32) + (threadIdx.x >> 5);
    const int64_t nchunks = p.nchunks[0];
    const int64_t strip = warp_gid % p.warps_per_row;
    const int64_t chunk = warp_gid / p.warps_per_row;
    const int64_t nr = p.end[0] - p.begin[0];
    const bool has = chunk < nchunks;
    const int64_t ys = p.begin[0] + (has ? chunk * nr / nchunks : 0);
    const int64_t ye = p.begin[0] + (has ? (chunk + 1) * nr / nchunks : 0);
    const uint32_t* in = p.in;
    uint32_t* out = p.out;
    for (int64_t gen = 0; gen < n_gen; ++gen) {
        if (has && ys < ye) life_warp_rows<V, P, CM, true>(p, in, out, strip, ys, ye);
        if (gen + 1 < n_gen) grid_barrier(bar, (unsigned int)((gen + 1) * gridDim.x));
        const uint32_t* t = in;
        in = out;
        out = const_cast<uint32_t*>(t);
    }
}

// ------------------------------------------------ TMA-bulk pipelined kernel
// For rows that are a multiple of 128 bits (w % 128 == 0, every BASELINE
// config): warp-specialised producer/consumer over the row-streaming pipeline
// of tma_rows.cuh.  One producer warp streams the CTA's strip (NC consumer
// warps x 512 B; the whole row when w <= 65536) of successive rows into an
// NS-stage shared-memory ring with TMA bulk copies; the NC consumer warps read
// their 16 B plus the neighbouring words (the stage's 16-byte margins hold the
// neighbouring strips' edge words, or the WRAP source at the row ends), do the
// bit-sliced update, and store straight to HBM.

template <int NC, int NS, int CM, bool FUSED>
__global__ void __launch_bounds__((NC + 1) * 32) life_tma_kernel(const __grid_constant__ tma::RowStream p) {
    using G = tma::Geom<NC>;
    extern __shared__ __align__(128) uint8_t smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * G::kStageBytes);
    uint64_t* empty = full + NS;
    tma::init_barriers<NS>(full, empty, NC);
    tma::pdl_wait_and_release();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    tma::SegIter it = tma::seg_iter(p);
    tma::Seg sg;
    tma::RingPos ring;  // CTA-wide ring position (same sequence in producer and consumers)
    const tma::HaloLink& L = p.link;

    if (warp == NC) {
        if (lane == 0) {
            while (tma::seg_next<NC>(p, it, sg)) {
                // (the mailbox is read only by segments that load halo rows)
                const unsigned int halo_target =
                    FUSED && (sg.ys < 1 || sg.ye + 1 > p.rows) ? halo_wait_target(L, p.nstrips) : 0u;
                tma::produce_align<NS, 1>(full, empty, ring, lane);
                tma::produce<NC, NS, CM == COL_WRAP, 4, 1>(p, sg, smem, full, empty, sg.ys - 1, sg.ye - sg.ys + 2, ring,
                                                     halo_target, lane);
            }
        }
        if constexpr (FUSED) tma::finish_launch_producer((NC + 1) * 32, p.link_ctas);
        return;
    }
    {
        // ------------------------------------------------------ consumers
        // Input row j of a segment (global row ys-1+j) sits in stage (base+j) % NS
        // with base a multiple of NS; the loop is unrolled by NS (a multiple of 3)
        // so stage indices and the 3-row rotation of the row sums are
        // compile-time register renames.
        static_assert(NS % 3 == 0, "NS must be a multiple of 3");
        const int t = warp * 32 + lane;  // vector index within the strip
        uint32_t r0[3][4], r1[3][4], xs[3][4];  // row sums and raw words of 3 rows
        // Per segment: the linked body (stores into the neighbours' halos and
        // signals them) only for segments that contain boundary rows; the
        // interior segments of a fused launch run the plain body, so they
        // cost what the unfused kernel costs (measured: one body for all
        // segments made the fused 65536^2 generation 212 us instead of 165).
        auto seg_body = [&](auto link_tag) {
            constexpr bool LINK = decltype(link_tag)::value;
            tma::consume_align<NS>(full, empty, ring, lane);
            uint32_t ph = ring.phase;  // segment starts at stage 0
            const int n_in = (int)(sg.ye - sg.ys + 2);  // input rows ys-1 .. ye
            const bool active = t * 4 < (int)sg.seg;
            const bool row_first = sg.first_strip && t == 0;
            const bool row_last = sg.last_strip && (t + 1) * 4 == (int)sg.seg;
            const bool whole = sg.first_strip && sg.last_strip;
            uint32_t* out_row = static_cast<uint32_t*>(p.out) + sg.ys * p.pitch + sg.e0 + t * 4;
            int64_t yo = sg.ys;  // slab row of the next output

            auto consume = [&](int j, int k, int slot) {
                // k = j % NS (static), slot = j % 3 (static)
                tma::mbar_wait(&full[k], ph);
                const uint32_t* st = reinterpret_cast<const uint32_t*>(smem + k * G::kStageBytes);
                const uint4 v = *reinterpret_cast<const uint4*>(st + 4 + t * 4);
                // neighbour words; at the row ends: WRAP -> the other end (from
                // the stage itself when the strip is the whole row, else from
                // the margin copy), CLAMP -> replicate, ZERO -> 0
                uint32_t lw = st[(CM == COL_WRAP && row_first && whole) ? 4 + (int)sg.seg - 1 : 4 + t * 4 - 1];
                uint32_t rw = st[(CM == COL_WRAP && row_last && whole) ? 4 : 4 + t * 4 + 4];
                __syncwarp();
                if (lane == 0) tma::mbar_arrive(&empty[k]);
                if (CM != COL_WRAP) {
                    if (row_first) lw = (CM == COL_CLAMP) ? (v.x << 31) : 0u;  // column -1 := column 0 / 0
                    if (row_last) rw = (CM == COL_CLAMP) ? (v.w >> 31) : 0u;   // column w := column w-1 / 0
                }
                xs[slot][0] = v.x; xs[slot][1] = v.y; xs[slot][2] = v.z; xs[slot][3] = v.w;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t ls = (q == 0) ? lw : xs[slot][q - 1];
                    const uint32_t rs = (q == 3) ? rw : xs[slot][q + 1];
                    const uint32_t Lf = __funnelshift_l(ls, xs[slot][q], 1);
                    const uint32_t Rf = __funnelshift_r(xs[slot][q], rs, 1);
                    r0[slot][q] = Lf ^ xs[slot][q] ^ Rf;
                    r1[slot][q] = maj3(Lf, xs[slot][q], Rf);
                }
            };
            auto emit = [&](int slot) {
                // centre row in slot (slot+2)%3, row above in (slot+1)%3, row below in slot
                const int A = (slot + 1) % 3, B = (slot + 2) % 3, C = slot;
                uint32_t o[4];
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    o[q] = life_word(r0[A][q], r1[A][q], r0[B][q], r1[B][q], r0[C][q], r1[C][q], xs[B][q]);
                if (active) {
                    const uint4 ov = make_uint4(o[0], o[1], o[2], o[3]);
                    *reinterpret_cast<uint4*>(out_row) = ov;
                    if constexpr (LINK) {  // boundary rows also go to the neighbours' halos
                        if (L.dst_up && yo < L.r)
                            *reinterpret_cast<uint4*>(L.dst_up + yo * p.pitch + sg.e0 + t * 4) = ov;
                        if (L.dst_down && yo >= p.rows - L.r)
                            *reinterpret_cast<uint4*>(L.dst_down + (yo - (p.rows - L.r)) * p.pitch + sg.e0 + t * 4) =
                                ov;
                    }
                }
                out_row += p.pitch;
                ++yo;
            };

            const uint32_t ph0 = ph;
            int j = 0;
            if (n_in >= NS) {
                // first trip: input rows 0,1 only fill the window
#pragma unroll
                for (int k = 0; k < NS; ++k) {
                    consume(k, k, k % 3);
                    if (k >= 2) emit(k % 3);
                }
                ph ^= 1u;
                for (j = NS; j + NS <= n_in; j += NS) {
#pragma unroll
                    for (int k = 0; k < NS; ++k) {
                        consume(j + k, k, k % 3);
                        emit(k % 3);
                    }
                    ph ^= 1u;
                }
            }
            // last (partial) trip; j is a multiple of NS (and of 3)
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                if (j + k < n_in) {
                    consume(j + k, k, k % 3);
                    if (j + k >= 2) emit(k % 3);
                }
            }
            ring.stage = n_in % NS;
            ring.phase = ph0 ^ (uint32_t)((n_in / NS) & 1);
            ring.count += n_in;
            if constexpr (LINK) {
                if (L.dst_up && sg.ys < L.r) {
                    const int64_t e = sg.ye < L.r ? sg.ye : L.r;
                    tma::publish_delivery(L.sig_up, (unsigned int)(e - sg.ys), NC);
                }
                if (L.dst_down && sg.ye > p.rows - L.r) {
                    const int64_t b0 = sg.ys > p.rows - L.r ? sg.ys : p.rows - L.r;
                    tma::publish_delivery(L.sig_down, (unsigned int)(sg.ye - b0), NC);
                }
            }
        };
        while (tma::seg_next<NC>(p, it, sg)) {
            if constexpr (FUSED) {
                if (sg.ys < L.r || sg.ye > p.rows - L.r) {
                    seg_body(std::true_type{});
                    continue;
                }
            }
            seg_body(std::false_type{});
        }
    }
    if constexpr (FUSED) tma::finish_launch_consumers(L.mine, (NC + 1) * 32, p.link_ctas);
}

template <int NC, int NS, int CM>
cudaError_t launch_life_tma_t(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s,
                              const FusedLink* link) {
    using G = tma::Geom<NC>;
    tma::RowStream p;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = g.out;
    p.pitch = g.pitch / 4;
    p.rows = g.rows;
    p.n = g.w / 32;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    const int smem = NS * G::kStageBytes + 2 * NS * 8;
    static int ctas_per_sm = 0;
    if (ctas_per_sm == 0) {
        // occupancy of the plain kernel; the fused variant is launched with the same grid
        for (auto kfn : {life_tma_kernel<NC, NS, CM, false>, life_tma_kernel<NC, NS, CM, true>}) {
            cudaError_t e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e != cudaSuccess) return e;
        }
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctas_per_sm, life_tma_kernel<NC, NS, CM, false>,
                                                                      (NC + 1) * 32, smem);
        if (e != cudaSuccess) return e;
        if (ctas_per_sm < 1) ctas_per_sm = 1;
        const int want = kTmaCtasPerSm > 0 ? kTmaCtasPerSm : (16 / NC > 0 ? 16 / NC : 1);
        if (want < ctas_per_sm) ctas_per_sm = want;
    }
    tma_set_link(p, link, 1);
    const int64_t ctas = tma_plan_grid(p, b, num_sms, ctas_per_sm, G::kStripElems, link != nullptr);
    tma_record(g.rec, LK_LIFE_TMA, p, ctas, (NC + 1) * 32, smem, NS, 1, NC);
    if (ctas == 0) return cudaSuccess;
    if (link) return tma_launch(life_tma_kernel<NC, NS, CM, true>, (unsigned)ctas, (NC + 1) * 32, smem, s, p, g.pdl);
    return tma_launch(life_tma_kernel<NC, NS, CM, false>, (unsigned)ctas, (NC + 1) * 32, smem, s, p, g.pdl);
}

template <int NC, int NS>
cudaError_t launch_life_tma_nc(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s,
                               const FusedLink* link) {
    switch (g.col_mode) {
        case COL_WRAP: return launch_life_tma_t<NC, NS, COL_WRAP>(g, b, num_sms, s, link);
        case COL_CLAMP: return launch_life_tma_t<NC, NS, COL_CLAMP>(g, b, num_sms, s, link);
        default: return launch_life_tma_t<NC, NS, COL_ZERO>(g, b, num_sms, s, link);
    }
}

// Strip width: the whole row when it fits in 16 warps x 512 B (every config:
// 65536 cells = 8 KB = 16 warps), so each CTA is ONE sequential DRAM stream;
// ~16 consumer warps per SM in total (measured best: fewer, longer streams
// keep HBM pages open — tools/membench.cu, profiles/).
template <int NS>
cudaError_t launch_life_tma(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s,
                            const FusedLink* link) {
    const int64_t nvec = g.w / 128;  // 16-byte vectors per row
    if (nvec > 8 * 32) return launch_life_tma_nc<16, NS>(g, b, num_sms, s, link);
    if (nvec > 4 * 32) return launch_life_tma_nc<8, NS>(g, b, num_sms, s, link);
    if (nvec > 2 * 32) return launch_life_tma_nc<4, NS>(g, b, num_sms, s, link);
    return launch_life_tma_nc<2, NS>(g, b, num_sms, s, link);
}

// ------------------------------------------------ any width
// Widths that are not a multiple of 64 cells: a row has nw = ceil(w/32) words,
// the last one holding b = w - 32(nw-1) cells in bits 0..b-1 (bits >= b are
// kept 0).  One thread per output word; the neighbour bits across word ends
// come from the adjacent words, and at the row ends from the boundary rule:
// WRAP pairs column w-1 (bit b-1 of the last word) with column 0.  A
// correctness path (the configs' widths all take the TMA kernel).
template <int CM>
__global__ void life_anyw_kernel(const __grid_constant__ LifeParams p, int tail_bits) {
    const int64_t m = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int band = blockIdx.z;
    if (m >= p.nw) return;
    const int64_t last = p.nw - 1;
    const uint32_t tail_mask = tail_bits == 32 ? ~0u : ((1u << tail_bits) - 1u);
    for (int64_t y = p.begin[band] + blockIdx.y; y < p.end[band]; y += gridDim.y) {
        uint32_t r0[3], r1[3], mid = 0;
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const uint32_t* row = p.in + map_row(p, y + k - 1) * p.pitch_w;
            const uint32_t x = __ldg(row + m);
            const uint32_t first = __ldg(row);
            const uint32_t lastw = __ldg(row + last);
            // cell left of bit 0 of word m, and right of the word's last cell
            uint32_t lbit;
            if (m > 0) {
                lbit = __ldg(row + m - 1) >> 31;
            } else {
                lbit = CM == COL_WRAP ? (lastw >> (tail_bits - 1)) & 1u : CM == COL_CLAMP ? (x & 1u) : 0u;
            }
            uint32_t R;
            if (m < last) {
                R = (x >> 1) | (__ldg(row + m + 1) << 31);
            } else {
                const uint32_t e = CM == COL_WRAP ? (first & 1u) : CM == COL_CLAMP ? ((x >> (tail_bits - 1)) & 1u) : 0u;
                R = (x >> 1) | (e << (tail_bits - 1));  // bits >= tail_bits of x are 0
            }
            const uint32_t L = (x << 1) | lbit;
            r0[k] = L ^ x ^ R;
            r1[k] = maj3(L, x, R);
            if (k == 1) mid = x;
        }
        uint32_t o = life_word(r0[0], r1[0], r0[1], r1[1], r0[2], r1[2], mid);
        if (m == last) o &= tail_mask;
        p.out[y * p.pitch_w + m] = o;
    }
}

template <int CM>
cudaError_t launch_life_anyw_t(const StencilGeom& g, const RowBands& b, cudaStream_t s) {
    LifeParams p;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = static_cast<uint32_t*>(g.out);
    p.pitch_w = g.pitch / 4;
    p.rows = g.rows;
    p.nw = (g.w + 31) / 32;
    p.nvec = p.nw;
    p.warps_per_row = 0;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.col_mode = g.col_mode;
    int64_t maxr = 0;
    for (int i = 0; i < 2; ++i) {
        p.begin[i] = i < b.nbands ? b.begin[i] : 0;
        p.end[i] = i < b.nbands ? b.end[i] : 0;
        p.nchunks[i] = 0;
        if (p.end[i] - p.begin[i] > maxr) maxr = p.end[i] - p.begin[i];
    }
    if (maxr <= 0) return cudaSuccess;
    const int tail = (int)(g.w - 32 * (p.nw - 1));
    dim3 grid((unsigned)((p.nw + 127) / 128), (unsigned)(maxr < 8192 ? maxr : 8192), (unsigned)b.nbands);
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_LIFE_ANYW;
        g.rec->ctas = (int64_t)grid.x * grid.y * grid.z;
        g.rec->threads = 128;
    }
    life_anyw_kernel<CM><<<grid, 128, 0, s>>>(p, tail);
    return cudaGetLastError();
}

// ------------------------------------------------------------ pack / unpack
// u8 (nonzero = alive) -> bits; one thread per 32-bit word (32 bytes in).
__global__ void pack_life_kernel(const uint8_t* __restrict__ src, int64_t src_pitch,
                                 uint32_t* __restrict__ dst, int64_t dst_pitch_w, int64_t rows,
                                 int64_t nw, int64_t w, bool vec) {
    const int64_t wi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t y = blockIdx.y + (int64_t)blockIdx.z * gridDim.y;
    if (wi >= nw || y >= rows) return;
    const uint8_t* s = src + y * src_pitch + wi * 32;
    uint32_t word = 0;
    const int64_t nb = w - wi * 32;  // cells in this word (< 32 only for the last word of an odd width)
    if (vec && nb >= 32) {
        const uint4 q0 = __ldg(reinterpret_cast<const uint4*>(s));
        const uint4 q1 = __ldg(reinterpret_cast<const uint4*>(s + 16));
        const uint32_t v[8] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w};
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            // 0x80 in every nonzero byte, then gather the 4 flags (bits 7,15,23,31)
            // into bits 28..31 with one multiply (the partial products never overlap).
            const uint32_t m = __vcmpne4(v[q], 0u) & 0x80808080u;
            word |= ((m * 0x00204081u) >> 28) << (4 * q);
        }
    } else {
        for (int j = 0; j < 32 && j < nb; ++j) word |= (uint32_t)(s[j] != 0) << j;
    }
    dst[y * dst_pitch_w + wi] = word;
}

// bits -> u8 0/1; one thread per 32-bit word (32 bytes out).
__global__ void unpack_life_kernel(const uint32_t* __restrict__ src, int64_t src_pitch_w,
                                   uint8_t* __restrict__ dst, int64_t dst_pitch, int64_t rows,
                                   int64_t nw, int64_t w, bool vec) {
    const int64_t wi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t y = blockIdx.y + (int64_t)blockIdx.z * gridDim.y;
    if (wi >= nw || y >= rows) return;
    const uint32_t word = src[y * src_pitch_w + wi];
    uint8_t* d = dst + y * dst_pitch + wi * 32;
    uint32_t v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) v[q] = (((word >> (4 * q)) & 0xFu) * 0x00204081u) & 0x01010101u;
    const int64_t nb = w - wi * 32;
    if (vec && nb >= 32) {
        *reinterpret_cast<uint4*>(d) = make_uint4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<uint4*>(d + 16) = make_uint4(v[4], v[5], v[6], v[7]);
    } else {
        for (int j = 0; j < 32 && j < nb; ++j) d[j] = (uint8_t)((word >> j) & 1u);
    }
}

template <int V, int P, int CM>
cudaError_t launch_life_t(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s) {
    LifeParams p;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = static_cast<uint32_t*>(g.out);
    p.pitch_w = g.pitch / 4;
    p.rows = g.rows;
    p.nw = g.w / 32;
    p.nvec = p.nw / V;
    p.warps_per_row = (p.nvec + 31) / 32;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.col_mode = g.col_mode;

    static int blocks_per_sm = 0;  // per (V,P) instantiation; device-independent enough
    if (blocks_per_sm == 0) {
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm,
                                                                      life_step_kernel<V, P, CM>, kThreads, 0);
        if (e != cudaSuccess) return e;
        if (blocks_per_sm < 1) blocks_per_sm = 1;
    }
    const int64_t resident_warps = (int64_t)num_sms * blocks_per_sm * (kThreads / 32);
    int64_t max_warps = 0;
    for (int i = 0; i < 2; ++i) {
        p.begin[i] = p.end[i] = 0;
        p.nchunks[i] = 0;
    }
    for (int i = 0; i < b.nbands; ++i) {
        p.begin[i] = b.begin[i];
        p.end[i] = b.end[i];
        const int64_t nr = b.end[i] - b.begin[i];
        int64_t nch = resident_warps / (p.warps_per_row * b.nbands);
        if (nch < 1) nch = 1;
        if (nch > nr) nch = nr;
        if (nr <= 0) nch = 0;
        p.nchunks[i] = nch;
        if (nch * p.warps_per_row > max_warps) max_warps = nch * p.warps_per_row;
    }
    if (max_warps == 0) return cudaSuccess;
    dim3 grid((unsigned)((max_warps + kThreads / 32 - 1) / (kThreads / 32)), (unsigned)b.nbands);
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_LIFE_REG;
        g.rec->ctas = (int64_t)grid.x * grid.y;
        g.rec->threads = kThreads;
    }
    life_step_kernel<V, P, CM><<<grid, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

template <int V, int P>
cudaError_t launch_life_cm(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s) {
    switch (g.col_mode) {
        case COL_WRAP: return launch_life_t<V, P, COL_WRAP>(g, b, num_sms, s);
        case COL_CLAMP: return launch_life_t<V, P, COL_CLAMP>(g, b, num_sms, s);
        default: return launch_life_t<V, P, COL_ZERO>(g, b, num_sms, s);
    }
}

}  // namespace

template <int V, int P, int CM>
cudaError_t launch_life_persist_t(const StencilGeom& g, int64_t n, unsigned int* bar, int num_sms, cudaStream_t s) {
    LifeParams p;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = static_cast<uint32_t*>(g.out);
    p.pitch_w = g.pitch / 4;
    p.rows = g.rows;
    p.nw = g.w / 32;
    p.nvec = p.nw / V;
    p.warps_per_row = (p.nvec + 31) / 32;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.col_mode = g.col_mode;
    static int blocks_per_sm = 0;
    if (blocks_per_sm == 0) {
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, life_persist_kernel<V, P, CM>,
                                                                      kPersistThreads, 0);
        if (e != cudaSuccess) return e;
        if (blocks_per_sm < 1) blocks_per_sm = 1;
    }
    // all CTAs co-resident (checked by the cooperative launch)
    const int64_t grid = (int64_t)num_sms * blocks_per_sm;
    int64_t nch = grid * (kPersistThreads / 32) / p.warps_per_row;
    if (nch < 1) nch = 1;
    if (nch > g.rows) nch = g.rows;
    p.begin[0] = 0;
    p.end[0] = g.rows;
    p.nchunks[0] = nch;
    p.begin[1] = p.end[1] = p.nchunks[1] = 0;
    cudaError_t e = cudaMemsetAsync(bar, 0, sizeof(unsigned int), s);
    if (e != cudaSuccess) return e;
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_LIFE_PERSIST;
        g.rec->ctas = grid;
        g.rec->threads = kPersistThreads;
        g.rec->gens = (int)n;
    }
    void* args[] = {(void*)&p, (void*)&n, (void*)&bar};
    return cudaLaunchCooperativeKernel((const void*)life_persist_kernel<V, P, CM>, dim3((unsigned)grid),
                                       dim3(kPersistThreads), args, 0, s);
}

template <int V>
cudaError_t launch_life_persist_v(const StencilGeom& g, int64_t n, unsigned int* bar, int num_sms, cudaStream_t s) {
    switch (g.col_mode) {
        case COL_WRAP: return launch_life_persist_t<V, kLifeP, COL_WRAP>(g, n, bar, num_sms, s);
        case COL_CLAMP: return launch_life_persist_t<V, kLifeP, COL_CLAMP>(g, n, bar, num_sms, s);
        default: return launch_life_persist_t<V, kLifeP, COL_ZERO>(g, n, bar, num_sms, s);
    }
}

cudaError_t launch_life_step(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s,
                             const FusedLink* link) {
    if (g.w % 128 == 0 && g.pitch % 16 == 0) return launch_life_tma<kTmaNS>(g, b, num_sms, s, link);
    if (link || b.nbands > 2) return cudaErrorInvalidValue;  // fused exchange needs the TMA kernel
    if (g.w % 64 == 0) return launch_life_cm<2, kLifeP>(g, b, num_sms, s);
    switch (g.col_mode) {
        case COL_WRAP: return launch_life_anyw_t<COL_WRAP>(g, b, s);
        case COL_CLAMP: return launch_life_anyw_t<COL_CLAMP>(g, b, s);
        default: return launch_life_anyw_t<COL_ZERO>(g, b, s);
    }
}

cudaError_t launch_life_persistent(const StencilGeom& g, int64_t n, unsigned int* bar, int num_sms, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (g.w % 64 != 0) return cudaErrorInvalidValue;  // odd widths: per-generation launches
    if (g.w % 128 == 0 && g.pitch % 16 == 0) return launch_life_persist_v<4>(g, n, bar, num_sms, s);
    return launch_life_persist_v<2>(g, n, bar, num_sms, s);
}

cudaError_t launch_pack_life(const uint8_t* src, int64_t src_pitch, void* dst, int64_t dst_pitch,
                             int64_t rows, int64_t w, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    const int64_t nw = (w + 31) / 32;
    const bool vec = (src_pitch % 16 == 0) && ((uintptr_t)src % 16 == 0);
    const unsigned ty = (unsigned)(rows < 32768 ? rows : 32768);
    dim3 grid((unsigned)((nw + 255) / 256), ty, (unsigned)((rows + ty - 1) / ty));
    pack_life_kernel<<<grid, 256, 0, s>>>(src, src_pitch, static_cast<uint32_t*>(dst), dst_pitch / 4,
                                          rows, nw, w, vec);
    return cudaGetLastError();
}

cudaError_t launch_unpack_life(const void* src, int64_t src_pitch, uint8_t* dst, int64_t dst_pitch,
                               int64_t rows, int64_t w, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    const int64_t nw = (w + 31) / 32;
    const bool vec = (dst_pitch % 16 == 0) && ((uintptr_t)dst % 16 == 0);
    const unsigned ty = (unsigned)(rows < 32768 ? rows : 32768);
    dim3 grid((unsigned)((nw + 255) / 256), ty, (unsigned)((rows + ty - 1) / ty));
    unpack_life_kernel<<<grid, 256, 0, s>>>(static_cast<const uint32_t*>(src), src_pitch / 4, dst,
                                            dst_pitch, rows, nw, w, vec);
    return cudaGetLastError();
}

}  // namespace mapsm
