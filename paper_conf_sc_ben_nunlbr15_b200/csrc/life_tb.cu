// life_tb.cu — temporally blocked ("deep halo") Game of Life, sm_100a.
//
// the Window(2D) -> Structured Injective Life step of
// the hot path (§4, Fig 2b) run K generations per pass.
// Each slab keeps H = K halo rows (instead of r = 1) and they are exchanged
// once per pass instead of every generation ("two-line boundary exchanges per
// iteration", become one K-line exchange per K iterations); inside a
// pass every CTA streams the input rows of its (strip, row range) once and
// carries them through all K generations in registers (a trapezoid in time:
// output rows [ys, ye) of generation t+K need rows [ys-K, ye+K) of
// generation t).  HBM traffic per generation drops K-fold, so the kernel is
// bound by the integer (ALU) pipe instead of HBM.  Results are bit-identical
// to K single-generation steps (same B3/S23 rule, same boundary semantics).
//
// Layout and work split.
//  * Rows stream through the TMA bulk-copy ring of tma_rows.cuh (producer
//    warp, NS stages); a stage holds the CTA's column strip (S words, S a
//    multiple of 4) plus a 4-word margin on each side.
//  * Consumer warp w, lane l holds ONE 32-bit word per row: strip word
//    x = 30w + l - 1.  Lanes 1..30 own (and store) their word; lanes 0 and 31
//    hold "ghost" words (the neighbouring warp's edge words, or the margin)
//    that are evolved with everything else so that no data crosses a warp
//    boundary inside a pass.  A ghost word gets one wrong neighbour bit per
//    generation at its outer edge; after K <= 31 generations its inner edge
//    bit — the only one its owner-lane neighbour reads — is still exact.
//  * Per generation and row each lane does 2 shuffles (the neighbour lanes'
//    words), 2 funnel shifts + 2 LOP3 (the 3-cell horizontal sum, 2 planes)
//    and the 8-LOP3 bit-sliced rule of life.cu (`life_word`): ~12 ALU ops per
//    32 cell-updates.  Level j keeps the horizontal sums and raw words of its
//    last 3 rows in registers (3-slot rotation, static under a 3-step unroll).
//
// Boundaries (identical results to the per-generation kernels):
//  * rows, WRAP with one slab: input rows are taken mod rows (periodic
//    extension commutes with the rule); exchanged halos: the H rows from the
//    neighbour; CLAMP global edge: the MIRROR image (row -1-i := row i).  A
//    mirror-symmetric grid stays mirror-symmetric under Life, so at every
//    generation row -1 equals row 0, which is exactly CLAMP;  ZERO global
//    edge: the (zeroed) halo rows, and every generation's rows outside the
//    grid are forced back to 0.
//  * columns: WRAP ghosts come from the wrap margins; CLAMP ghosts are the
//    bit-reversed edge word (the mirror image, same argument); ZERO ghosts
//    are 0 and forced to 0 at every generation.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <type_traits>

#include "kernels.h"
#include "tma_rows.cuh"

namespace mapsm {
namespace tb {

constexpr int kOut = 30;     // words stored per warp (lanes 1..30)
#ifndef MAPSM_TB_MAXNC
#define MAPSM_TB_MAXNC 15
#endif
#ifndef MAPSM_TB_REGS
#define MAPSM_TB_REGS 128
#endif
// consumer warps per CTA: 16 warps x 128 registers fill the register file
// (4 warps x 128 registers x 32 lanes = one SMSP's 16K registers)
constexpr int kMaxNC = MAPSM_TB_MAXNC;
#ifndef MAPSM_TB_NS
#define MAPSM_TB_NS 8
#endif
constexpr int kNS = MAPSM_TB_NS;  // ring stages
// rows per ring stage = rows evaluated together (a multiple of 3); 6 would
// spill at K = 8 under the 128-register cap
__host__ __device__ constexpr int rows_per_stage(int K) { return K >= 8 ? 3 : 6; }
constexpr unsigned kFull = 0xffffffffu;

struct TbParams {
    tma::RowStream s;  // s.n = words per row, bands, row maps (ROWMAP_CLAMP = mirror here)
    int64_t strip;     // strip width in words (multiple of 4); the last strip may be shorter
    int zero_top, zero_bot;  // ZERO global edges: rows outside [0, rows) forced to 0 every generation
    int pdl;                 // (host) programmatic dependent launch (StencilGeom::pdl)
};

struct TbSeg {
    int64_t ys, ye, e0, seg;
    bool first, last;
};

__device__ __forceinline__ bool tb_seg_next(const TbParams& P, tma::SegIter& it, TbSeg& s) {
    if (it.pos >= it.hi) return false;
    const int64_t strip = it.pos / it.nr, r0 = it.pos % it.nr;
    const int64_t r1 = (it.nr - r0 < it.hi - it.pos) ? it.nr : r0 + (it.hi - it.pos);
    s.ys = it.rb + r0;
    s.ye = it.rb + r1;
    it.pos += r1 - r0;
    s.e0 = strip * P.strip;
    s.seg = P.s.n - s.e0 < P.strip ? P.s.n - s.e0 : P.strip;
    s.first = strip == 0;
    s.last = s.e0 + s.seg == P.s.n;
    return true;
}

// Input row y in [-K, rows + K) -> slab row to read.
__device__ __forceinline__ int64_t tb_map_row(const tma::RowStream& p, int64_t y) {
    if (y < 0) {
        if (p.top_map == ROWMAP_WRAP) {
            y %= p.rows;
            if (y < 0) y += p.rows;
        } else if (p.top_map == ROWMAP_CLAMP) {
            y = -1 - y;  // mirror
        }
    } else if (y >= p.rows) {
        if (p.bot_map == ROWMAP_WRAP) y %= p.rows;
        else if (p.bot_map == ROWMAP_CLAMP) y = 2 * p.rows - 1 - y;  // mirror
    }
    return y;  // ROWMAP_HALO: the halo row itself (exchanged, or zero)
}

// Producer (one thread): input rows y_first .. y_first+n_in-1 of the strip,
// RPS rows per stage (one mbarrier round per RPS rows).  Stage row q:
// [margin 4 words][strip seg words][margin 4 words], row pitch P.strip + 8.
template <int NS, int RPS>
__device__ __forceinline__ void tb_produce(const TbParams& P, const TbSeg& t, uint8_t* smem, int stage_bytes,
                                           int row_bytes, uint64_t* full, uint64_t* empty, int64_t y_first,
                                           int64_t n_in, tma::RingPos& r, bool wrap_cols) {
    const tma::RowStream& p = P.s;
    const bool wrap_l = wrap_cols && t.first;
    const bool wrap_r = wrap_cols && t.last;
    const uint32_t main_bytes = (uint32_t)(t.seg * 4) + (t.first ? 0u : 16u) + (t.last ? 0u : 16u);
    const uint32_t tx = main_bytes + (wrap_l ? 16u : 0u) + (wrap_r ? 16u : 0u);
    const int64_t src_off = t.e0 - (t.first ? 0 : 4);
    const uint32_t dst_main = t.first ? 16u : 0u;
    const uint32_t dst_r = 16u + (uint32_t)(t.seg * 4);
    for (int64_t j0 = 0; j0 < n_in; j0 += RPS) {
        const int nr = n_in - j0 < RPS ? (int)(n_in - j0) : RPS;
        if (r.count >= NS) tma::mbar_wait(&empty[r.stage], r.phase ^ 1u);
        uint8_t* st = smem + r.stage * stage_bytes;
        uint64_t* bar = &full[r.stage];
        tma::mbar_arrive_expect_tx(bar, tx * (uint32_t)nr);
        for (int q = 0; q < nr; ++q, st += row_bytes) {
            const uint32_t* rp = p.in + tb_map_row(p, y_first + j0 + q) * p.pitch;
            tma::bulk_g2s(st + dst_main, rp + src_off, main_bytes, bar);
            if (wrap_l) tma::bulk_g2s(st, rp + p.n - 4, 16, bar);  // words n-4..n-1
            if (wrap_r) tma::bulk_g2s(st + dst_r, rp, 16, bar);    // words 0..3
        }
        r.advance(NS);
    }
}

__device__ __forceinline__ uint32_t maj3(uint32_t a, uint32_t b, uint32_t c) { return (a & b) | (a & c) | (b & c); }

// B3/S23 on bit-sliced 3-row sums (see life.cu: life_word); `m` masks the result.
__device__ __forceinline__ uint32_t rule(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1, uint32_t c0,
                                        uint32_t c1, uint32_t alive, uint32_t m) {
    const uint32_t s0 = a0 ^ b0 ^ c0;
    const uint32_t k = maj3(a0, b0, c0);
    const uint32_t t = a1 ^ b1 ^ c1;
    const uint32_t u = maj3(a1, b1, c1);
    const uint32_t C = u ^ (k | t);
    const uint32_t D = ~(s0 ^ k ^ t) & (s0 | alive);
    return C & D & m;
}

// Horizontal 3-cell sum of this lane's word x (2 bit-planes): the
// neighbour lanes' words by shuffle, the neighbour bits by funnel shifts.
// (Building the shifts on the FMA pipe with IMAD.WIDE instead measured 15%
// slower: the wide multiplies occupy the heavy FMA pipe and lengthen the
// per-level dependency chain.)
__device__ __forceinline__ void hsum(uint32_t x, uint32_t& n0, uint32_t& n1) {
    const uint32_t u = __shfl_up_sync(kFull, x, 1);
    const uint32_t d = __shfl_down_sync(kFull, x, 1);
    const uint32_t L = __funnelshift_l(u, x, 1);  // bit i <- column i-1
    const uint32_t R = __funnelshift_r(x, d, 1);  // bit i <- column i+1
    n0 = L ^ x ^ R;
    n1 = maj3(L, x, R);
}

// Consumer-lane state of one segment: the per-level rows and the lane's
// geometry.  Level j (generation t+j+1) keeps the horizontal sums (h0, h1)
// and raw word (cx) of the last three rows it received, slot = step mod 3.
template <int K, int CM, bool ZCHK>
struct TbLane {
    uint32_t (&h0)[K][3];
    uint32_t (&h1)[K][3];
    uint32_t (&cx)[K][3];
    uint32_t lane_mask;
    int64_t Y0, rows;
    int zero_top, zero_bot;
    bool st_ok;
    uint32_t* outp;
    int64_t pitch;

    // GG consecutive steps (input rows) s .. s+GG-1 held in xs[OFF..], slot of
    // step s = S0: the GG x K (step, level) cells in anti-diagonal order —
    // cell (g, j) needs (g-1, j) (level j's previous row) and (g, j-1) (this
    // row one generation earlier) — so up to min(GG, K) independent chains
    // are in flight; then the level-K rows are stored (from step 2K on).
    template <int OFF, int GG, int S0, int N>
    __device__ __forceinline__ void cells(uint32_t (&xs)[N], int s) {
#pragma unroll
        for (int d = 0; d < K + GG - 1; ++d) {
#pragma unroll
            for (int g = 0; g < GG; ++g) {
                const int j = d - g;
                if (j < 0 || j >= K) continue;
                const int slot = (S0 + g) % 3;
                const int A = (slot + 1) % 3, B = (slot + 2) % 3;  // rows y-2, y-1
                uint32_t m = lane_mask;
                if constexpr (ZCHK) {
                    const int64_t yj = Y0 + s + g - (j + 1);  // row emitted by level j
                    if ((zero_top && yj < 0) || (zero_bot && yj >= rows)) m = 0u;
                }
                uint32_t n0, n1;
                hsum(xs[OFF + g], n0, n1);
                const uint32_t o = rule(h0[j][A], h1[j][A], h0[j][B], h1[j][B], n0, n1, cx[j][B],
                                        (CM == COL_ZERO || ZCHK) ? m : ~0u);
                h0[j][slot] = n0;
                h1[j][slot] = n1;
                cx[j][slot] = xs[OFF + g];
                xs[OFF + g] = o;  // level j's row y-1 feeds level j+1
            }
        }
#pragma unroll
        for (int g = 0; g < GG; ++g)
            if (st_ok && s + g >= 2 * K) {
                *outp = xs[OFF + g];
                outp += pitch;
            }
    }
};

template <int K, int NS, int CM, bool ZCHK>
__device__ __forceinline__ void tb_consume_segment(const TbParams& P, const TbSeg& sg, uint8_t* smem, int stage_bytes,
                                                   int row_words, uint64_t* full, uint64_t* empty, tma::RingPos& ring,
                                                   int si, uint32_t rev, TbLane<K, CM, ZCHK>& L, int lane) {
    constexpr int RPS = rows_per_stage(K);
    const int n_in = (int)(sg.ye - sg.ys) + 2 * K;
    uint32_t xs[RPS];
    // read the next stage's first nr rows (this lane's word of each)
    auto fetch = [&](int nr) {
        tma::mbar_wait(&full[ring.stage], ring.phase);
        const uint32_t* st = reinterpret_cast<const uint32_t*>(smem + ring.stage * stage_bytes) + si;
#pragma unroll
        for (int q = 0; q < RPS; ++q) {
            if (q < nr) {
                uint32_t x = st[q * row_words];
                if (CM == COL_CLAMP) x = rev ? __brev(x) : x;
                if (CM == COL_ZERO) x &= L.lane_mask;
                xs[q] = x;
            }
        }
        __syncwarp();
        if (lane == 0) tma::mbar_arrive(&empty[ring.stage]);
        ring.advance(NS);
    };
    int s = 0;
    for (; s + RPS <= n_in; s += RPS) {  // RPS is a multiple of 3: the slot of step s is 0
        fetch(RPS);
        L.template cells<0, RPS, 0>(xs, s);
    }
    const int rem = n_in - s;  // < RPS rows, all in one stage
    if (rem > 0) {
        fetch(rem);
        if (RPS > 3 && rem >= 3) {
            L.template cells<0, 3, 0>(xs, s);
            if (rem > 3) L.template cells<(RPS > 3 ? 3 : 0), 1, 0>(xs, s + 3);
            if (rem > 4) L.template cells<(RPS > 4 ? 4 : 0), 1, 1>(xs, s + 4);
        } else {
            L.template cells<0, 1, 0>(xs, s);
            if (rem > 1) L.template cells<1, 1, 1>(xs, s + 1);
        }
    }
}

template <int K, int NS, int CM>
__global__ void __maxnreg__(MAPSM_TB_REGS) life_tb_kernel(const __grid_constant__ TbParams P) {
    static_assert(K >= 1 && K <= 31, "ghost words stay exact for at most 31 generations");
    constexpr int RPS = rows_per_stage(K);
    const tma::RowStream& p = P.s;
    const int NC = (int)(blockDim.x >> 5) - 1;
    const int row_words = (int)P.strip + 8;
    const int row_bytes = row_words * 4;
    const int stage_bytes = RPS * row_bytes;
    extern __shared__ __align__(128) uint8_t smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * stage_bytes);
    uint64_t* empty = full + NS;
    tma::init_barriers<NS>(full, empty, NC);
    tma::pdl_wait_and_release();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    tma::SegIter it = tma::seg_iter(p);
    TbSeg sg;
    tma::RingPos ring;

    if (warp == NC) {
        if (lane == 0) {
            while (tb_seg_next(P, it, sg))
                tb_produce<NS, RPS>(P, sg, smem, stage_bytes, row_bytes, full, empty, sg.ys - K,
                                    sg.ye - sg.ys + 2 * K, ring, CM == COL_WRAP);
        }
        return;
    }

    uint32_t h0[K][3], h1[K][3], cx[K][3];
#pragma unroll
    for (int j = 0; j < K; ++j)
#pragma unroll
        for (int q = 0; q < 3; ++q) h0[j][q] = h1[j][q] = cx[j][q] = 0u;

    const int xi = warp * kOut + lane - 1;  // strip word of this lane (-1: left ghost)
    while (tb_seg_next(P, it, sg)) {
        const int seg = (int)sg.seg;
        int si = 4 + xi;
        if (si > 4 + seg) si = 4 + seg;  // lanes past the right ghost: any word (never stored)
        const bool gl = sg.first && xi == -1, gr = sg.last && xi == seg;
        uint32_t lane_mask = ~0u;
        uint32_t rev = 0u;
        if (CM == COL_ZERO && (gl || gr)) lane_mask = 0u;
        if (CM == COL_CLAMP) {
            if (gl) { si = 4; rev = 1u; }
            if (gr) { si = 4 + seg - 1; rev = 1u; }
        }
        const int64_t Y0 = sg.ys - K;  // input row of step 0
        const bool zseg = (P.zero_top && Y0 < 0) || (P.zero_bot && sg.ye + K > p.rows);
        // output row of step s is ys - 2K + s; stored from s = 2K on
        uint32_t* outp = static_cast<uint32_t*>(p.out) + sg.ys * p.pitch + sg.e0 + xi;
        const bool st_ok = lane >= 1 && lane <= kOut && xi < seg;
        if (zseg) {
            TbLane<K, CM, true> L{h0, h1, cx, lane_mask, Y0, p.rows, P.zero_top, P.zero_bot, st_ok, outp, p.pitch};
            tb_consume_segment<K, NS, CM, true>(P, sg, smem, stage_bytes, row_words, full, empty, ring, si, rev, L,
                                                lane);
        } else {
            TbLane<K, CM, false> L{h0, h1, cx, lane_mask, Y0, p.rows, P.zero_top, P.zero_bot, st_ok, outp, p.pitch};
            tb_consume_segment<K, NS, CM, false>(P, sg, smem, stage_bytes, row_words, full, empty, ring, si, rev, L,
                                                 lane);
        }
    }
}

template <int K, int CM>
cudaError_t launch_tb_t(const TbParams& P0, const RowBands& b, int nc, int num_sms, cudaStream_t s, LaunchRec* rec) {
    TbParams P = P0;
    const int smem = kNS * rows_per_stage(K) * (int)(P.strip * 4 + 32) + 2 * kNS * 8;
    auto kfn = life_tb_kernel<K, kNS, CM>;
    static int attr_set = 0;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        if (e != cudaSuccess) return e;
        attr_set = 1;
    }
    static int occ[kMaxNC + 1] = {0};
    static int occ_smem[kMaxNC + 1] = {0};
    if (occ[nc] == 0 || occ_smem[nc] != smem) {
        int c = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&c, kfn, (nc + 1) * 32, smem);
        if (e != cudaSuccess) return e;
        if (c < 1) c = 1;
        // up to 32 consumer warps per SM (ALU-bound: more warps hide the
        // shuffle / dependency latency of the level chain)
        const int want = 32 / nc > 0 ? 32 / nc : 1;
        occ[nc] = c < want ? c : want;
        occ_smem[nc] = smem;
    }
    const int64_t ctas = tma_plan_grid(P.s, b, num_sms, occ[nc], (int)P.strip);
    tma_record(rec, LK_LIFE_TB, P.s, ctas, (nc + 1) * 32, smem, kNS, rows_per_stage(K), nc, K);
    if (ctas == 0) return cudaSuccess;
    cudaError_t e = tma_launch(kfn, (unsigned)ctas, (nc + 1) * 32, smem, s, P, P.pdl != 0);
    if (e != cudaSuccess && getenv("MAPSM_DEBUG")) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, kfn);
        fprintf(stderr, "life_tb K=%d CM=%d: %s; regs %d maxThreads %d threads %d smem %d ctas %lld occ %d\n", K, CM,
                cudaGetErrorString(e), fa.numRegs, fa.maxThreadsPerBlock, (nc + 1) * 32, smem, (long long)ctas,
                occ[nc]);
    }
    return e;
}

template <int K>
cudaError_t launch_tb_k(const TbParams& P, const RowBands& b, int col_mode, int nc, int num_sms, cudaStream_t s,
                        LaunchRec* rec) {
    switch (col_mode) {
        case COL_WRAP: return launch_tb_t<K, COL_WRAP>(P, b, nc, num_sms, s, rec);
        case COL_CLAMP: return launch_tb_t<K, COL_CLAMP>(P, b, nc, num_sms, s, rec);
        default: return launch_tb_t<K, COL_ZERO>(P, b, nc, num_sms, s, rec);
    }
}

}  // namespace tb

bool life_tb_supported(int k) { return k == 2 || k == 3 || k == 4 || k == 6 || k == 8; }

cudaError_t launch_life_tb(const StencilGeom& g, const RowBands& b, int k, int zero_top, int zero_bot, int num_sms,
                           cudaStream_t s) {
    using namespace tb;
    const int64_t W = g.w / 32;
    if (g.w % 128 != 0 || g.pitch % 16 != 0 || !life_tb_supported(k)) return cudaErrorInvalidValue;
    TbParams P;
    tma::RowStream& p = P.s;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = g.out;
    p.pitch = g.pitch / 4;
    p.rows = g.rows;
    p.n = W;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    tma_set_link(p, nullptr, k);
    // strips of at most kMaxNC * 30 words, as equal as possible (multiples of 4 words)
    const int64_t cap = (int64_t)kMaxNC * kOut / 4 * 4;
    const int64_t nstrips = (W + cap - 1) / cap;
    P.strip = ((W + nstrips - 1) / nstrips + 3) / 4 * 4;
    P.zero_top = zero_top;
    P.zero_bot = zero_bot;
    P.pdl = g.pdl ? 1 : 0;
    const int nc = (int)((P.strip + kOut - 1) / kOut);
    switch (k) {
        case 2: return launch_tb_k<2>(P, b, g.col_mode, nc, num_sms, s, g.rec);
        case 3: return launch_tb_k<3>(P, b, g.col_mode, nc, num_sms, s, g.rec);
        case 4: return launch_tb_k<4>(P, b, g.col_mode, nc, num_sms, s, g.rec);
        case 6: return launch_tb_k<6>(P, b, g.col_mode, nc, num_sms, s, g.rec);
        default: return launch_tb_k<8>(P, b, g.col_mode, nc, num_sms, s, g.rec);
    }
}

}  // namespace mapsm
