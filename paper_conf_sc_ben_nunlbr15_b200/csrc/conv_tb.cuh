#pragma once
// conv_tb.cuh — TWO generations of the fp32 window convolution per pass in
// one kernel (temporal blocking), radius 1..2, sm_100a.  Included by
// conv_r1.cu / conv_r2.cu (it uses their translation unit's __constant__
// weight slots, conv_impl.cuh).
//
// SURVEY §8(f) NEXT-2 (deep halos, reading t4): with
// MAPSM_OPT_DEEP_HALO = 2 the slab keeps 2r halo rows, exchanged once per
// pass; this kernel then reads generation t ONCE from HBM and writes
// generation t+2 (the 5x5 convolution is HBM-bound per generation: 8 B per
// cell-update; a pass halves that).  Per output cell the arithmetic is the
// oracle's fixed fmaf chain of reading c11, twice: generation t+1 values are
// computed exactly as a single generation would (same taps, same order,
// boundary values synthesised by the same rules) and generation t+2 is the
// same chain over them — bit-identical to two single generations.
//
// Layout.  A CTA = NC consumer warps + 1 ghost warp + 1 producer warp.  The
// producer streams the input rows [ys-2r, ye+2r) of the CTA's (strip, rows)
// segments through an NS-stage TMA ring whose stages carry 8-float margins
// (level 1 of the strip's edge vectors reads 4+r floats past the strip).
// Consumer lane t owns columns [4t, 4t+4) of the strip at both levels; the
// ghost warp's lanes 0 / 1 compute the level-1 vectors just left / right of
// the strip (columns [-4, 0) / [S, S+4)), which level 2 of the edge lanes
// reads.  Per input row: level 1 advances 2r+1 rotating accumulator rows
// (FFMA2 pairs, weights from the constant slot on the uniform datapath, as
// conv_impl.cuh); the level-1 row that completes goes to a 2-row shared
// buffer; a named barrier; level 2 consumes it (2r+1 rotating accumulators)
// and stores its completed row of generation t+2.
//
// Boundaries.  Columns: level 1 synthesises inputs outside the grid (CLAMP:
// the edge column, ZERO: 0; WRAP: the producer copies the row's other end
// into the margin); level 2 synthesises generation t+1 values outside the
// grid the same way (CLAMP: the edge column of generation t+1, ZERO: 0),
// while under WRAP the ghost / neighbour lanes computed them from wrapped
// inputs.  Rows: exchanged halos and one-slab WRAP give real generation t+1
// rows outside the slab; at a global CLAMP edge level 2 consumes the
// generation t+1 edge row in place of the r rows outside (fed r+1 times),
// at a ZERO edge it consumes r zero rows (the oracle's fmaf(w, 0, acc) terms).
#include "conv_impl.cuh"

namespace mapsm {
namespace conv_detail {

constexpr int kTbMargin = 8;  // input stage margin (floats) each side

struct ConvTb2Params {
    tma::RowStream s;   // in / out / pitch / rows / n / bands / row maps (s.nstrips: strips of NC*128 floats)
    int zero_top, zero_bot;  // global ZERO edges
    int slot;                // weight slot (c_conv_wp / c_conv_w)
};

// Producer: input rows y_first .. y_first+n_in-1 of the segment's strip into
// the ring; stage = [8 margin | seg | 8 margin] floats.
template <int NS>
__device__ __forceinline__ void tb2_produce(const tma::RowStream& p, const tma::Seg& t, uint8_t* smem,
                                            int stage_bytes, uint64_t* full, uint64_t* empty, int64_t y_first,
                                            int64_t n_in, tma::RingPos& r, bool wrap_cols) {
    const int64_t lo = t.e0 - kTbMargin > 0 ? t.e0 - kTbMargin : 0;
    const int64_t hi = t.e0 + t.seg + kTbMargin < p.n ? t.e0 + t.seg + kTbMargin : p.n;
    const uint32_t main_bytes = (uint32_t)((hi - lo) * 4);
    const uint32_t dst_main = (uint32_t)((kTbMargin - (t.e0 - lo)) * 4);
    const bool wrap_l = wrap_cols && t.first_strip;
    const bool wrap_r = wrap_cols && t.last_strip;
    const uint32_t tx = main_bytes + (wrap_l ? kTbMargin * 4u : 0u) + (wrap_r ? kTbMargin * 4u : 0u);
    const uint32_t dst_r = (uint32_t)((kTbMargin + t.seg) * 4);
    for (int64_t j = 0; j < n_in; ++j) {
        if (r.count >= NS) tma::mbar_wait(&empty[r.stage], r.phase ^ 1u);
        const uint32_t* rp = p.in + tma::map_row(p, y_first + j) * p.pitch;
        uint8_t* st = smem + r.stage * stage_bytes;
        uint64_t* bar = &full[r.stage];
        tma::mbar_arrive_expect_tx(bar, tx);
        tma::bulk_g2s(st + dst_main, rp + lo, main_bytes, bar);
        if (wrap_l) tma::bulk_g2s(st, rp + p.n - kTbMargin, kTbMargin * 4, bar);
        if (wrap_r) tma::bulk_g2s(st + dst_r, rp, kTbMargin * 4, bar);
        r.advance(NS);
    }
}

// The 12 floats [c0-4, c0+8) of a row around the 4-column vector at strip
// column c0 (`base` = the row's strip column 0), with the grid's column
// boundary applied to columns outside [0, n) (global column = e0 + c):
// CLAMP -> the edge column, ZERO -> 0 (WRAP: the margins hold real data).
template <int CM>
__device__ __forceinline__ void window12(const float* base, int c0, int64_t e0, int64_t n, bool edge, float (&b)[12]) {
#pragma unroll
    for (int m = 0; m < 12; m += 4) {
        const float4 q = *reinterpret_cast<const float4*>(base + c0 - 4 + m);
        b[m] = q.x; b[m + 1] = q.y; b[m + 2] = q.z; b[m + 3] = q.w;
    }
    if (CM != COL_WRAP && edge) {
#pragma unroll
        for (int m = 0; m < 12; ++m) {
            const int64_t gcol = e0 + c0 - 4 + m;
            if (gcol < 0) b[m] = CM == COL_CLAMP ? base[-e0] : 0.f;
            else if (gcol >= n) b[m] = CM == COL_CLAMP ? base[n - 1 - e0] : 0.f;
        }
    }
}

// One input row's taps into 2R+1 rotating accumulator rows (pairs of outputs;
// hi = out(2j), lo = out(2j+1)); acc[2R] completes with this row.
template <int R>
__device__ __forceinline__ void rot_taps(Acc2 (&acc)[2 * R + 1][2], const float (&b)[12], unsigned long long cwp,
                                         unsigned long long cw) {
    constexpr int K = 2 * R + 1;
#pragma unroll
    for (int d = K - 1; d > 0; --d) {
        acc[d][0] = acc[d - 1][0];
        acc[d][1] = acc[d - 1][1];
    }
    acc[0][0] = acc[0][1] = 0ull;  // (+0.0f, +0.0f): a new output row starts
#pragma unroll
    for (int m = 0; m <= K; ++m) {
#pragma unroll
        for (int d = 0; d < K; ++d) {
            if (m == 0 || m == K) {
                const float w = ldc_one(cw + 4 * (d * K + (m == 0 ? 0 : K - 1)));
#pragma unroll
                for (int jp = 0; jp < 2; ++jp) {
                    const float v = b[4 - R + 2 * jp + m];
                    if (m == 0) fma_hi(acc[d][jp], w, v);
                    else fma_lo(acc[d][jp], w, v);
                }
            } else {
                const unsigned long long w = ldc_pair(cwp + 8 * (d * (K - 1) + m - 1));
#pragma unroll
                for (int jp = 0; jp < 2; ++jp) fma_pair(acc[d][jp], b[4 - R + 2 * jp + m], w);
            }
        }
    }
}

__device__ __forceinline__ float4 acc_row(const Acc2 (&a)[2]) {
    return make_float4(acc_hi(a[0]), acc_lo(a[0]), acc_hi(a[1]), acc_lo(a[1]));
}

template <int R, int NC, int NS, int CM>
__global__ void __launch_bounds__((NC + 2) * 32, 1) conv_tb2_kernel(const __grid_constant__ ConvTb2Params pp) {
    constexpr int K = 2 * R + 1;
    constexpr int S = NC * 128;                         // strip width (floats)
    constexpr int SB = (S + 2 * kTbMargin) * 4;         // stage bytes
    constexpr int L1W = S + 8;                          // level-1 row: [4 ghost | S | 4 ghost]
    const tma::RowStream& p = pp.s;
    extern __shared__ __align__(128) uint8_t smem[];
    float* l1 = reinterpret_cast<float*>(smem + NS * SB);          // 2 rows
    uint64_t* full = reinterpret_cast<uint64_t*>(l1 + 2 * L1W);
    uint64_t* empty = full + NS;
    tma::init_barriers<NS>(full, empty, NC + 1);
    const unsigned long long cwp = to_const(&c_conv_wp[pp.slot][0]);
    const unsigned long long cw = to_const(&c_conv_w[pp.slot][0]);
    const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
    tma::SegIter it = tma::seg_iter(p);
    tma::Seg sg;
    tma::RingPos ring;

    if (warp == NC + 1) {  // producer
        if (lane == 0) {
            while (tma::seg_next<NC, 4>(p, it, sg)) {
                tma::produce_align<NS, 1>(full, empty, ring, 0);
                tb2_produce<NS>(p, sg, smem, SB, full, empty, sg.ys - 2 * R, sg.ye - sg.ys + 4 * R, ring,
                                CM == COL_WRAP);
            }
        }
        return;
    }
    const bool ghost = warp == NC;  // lanes 0 / 1: the level-1 vectors left / right of the strip
    const int v = ghost ? (lane == 0 ? -1 : NC * 32) : warp * 32 + lane;  // level-1 vector (strip columns 4v..4v+3)
    const bool l1_on = !ghost || lane < 2;
    const bool clamp_top = p.top_map == ROWMAP_CLAMP, clamp_bot = p.bot_map == ROWMAP_CLAMP;
    const bool edge_top = clamp_top || pp.zero_top, edge_bot = clamp_bot || pp.zero_bot;
    Acc2 a1[K][2], a2[K][2];
#pragma unroll
    for (int d = 0; d < K; ++d) a1[d][0] = a1[d][1] = a2[d][0] = a2[d][1] = 0ull;

    while (tma::seg_next<NC, 4>(p, it, sg)) {
        tma::consume_align<NS>(full, empty, ring, lane);
        const int seg = (int)sg.seg;
        const int64_t ys = sg.ys, ye = sg.ye;
        const int n_in = (int)(ye - ys) + 4 * R;
        // lanes whose 12-float windows reach past a grid edge (CLAMP / ZERO synthesis)
        const bool edge1 = (sg.first_strip && 4 * v - 4 < 0) || (sg.last_strip && 4 * v + 8 > seg);
        const bool active = !ghost && 4 * v < seg;  // stores level 2
        float* out0 = reinterpret_cast<float*>(p.out) + sg.e0 + 4 * v;
        int feeds = 0;
        // level 2: consume one generation-t+1 row (or a zero row), store the completed row
        auto feed = [&](const float* row) {
            if (ghost) return;
            float b[12];
            if (row) {
                window12<CM>(row, 4 * v, sg.e0, p.n, edge1, b);
            } else {
#pragma unroll
                for (int m = 0; m < 12; ++m) b[m] = 0.f;
            }
            rot_taps<R>(a2, b, cwp, cw);
            if (feeds >= 2 * R && active) {
                const int64_t o = ys + feeds - 2 * R;
                *reinterpret_cast<float4*>(out0 + o * p.pitch) = acc_row(a2[K - 1]);
            }
            ++feeds;
        };
        int stg = ring.stage;
        uint32_t phs = ring.phase;
#pragma unroll 1
        for (int j = 0; j < n_in; ++j) {
            // ---- level 1: input row Y = ys - 2R + j
            tma::mbar_wait(&full[stg], phs);
            const float* st = reinterpret_cast<const float*>(smem + stg * SB) + kTbMargin;  // strip column 0
            float b[12];
            if (l1_on) window12<CM>(st, 4 * v, sg.e0, p.n, edge1, b);
            __syncwarp();
            if (lane == 0) tma::mbar_arrive(&empty[stg]);
            if (++stg == NS) {
                stg = 0;
                phs ^= 1u;
            }
            if (l1_on) rot_taps<R>(a1, b, cwp, cw);
            if (j < 2 * R) continue;  // generation-t+1 rows before ys - R are not needed
            // ---- the generation-t+1 row y1 = Y - R completed
            const int64_t y1 = ys - 3 * R + j;
            float* lrow = l1 + (j & 1) * L1W + 4;  // strip column 0 of the level-1 row buffer
            if (l1_on) *reinterpret_cast<float4*>(lrow + 4 * v) = acc_row(a1[K - 1]);
            asm volatile("bar.sync 1, %0;" ::"r"((NC + 1) * 32) : "memory");
            // ---- level 2
            if (edge_top && y1 < 0) continue;          // replaced (below) when row 0 is fed
            if (edge_bot && y1 >= p.rows) continue;    // replaced (below) after row rows-1
            if (edge_top && y1 == 0)
                for (int k = 0; k < R - (int)ys; ++k) feed(clamp_top ? lrow : nullptr);
            feed(lrow);
            if (edge_bot && y1 == p.rows - 1)
                for (int k = 0; k < (int)(ye + R - p.rows); ++k) feed(clamp_bot ? lrow : nullptr);
        }
        ring.stage = stg;
        ring.phase = phs;
        ring.count += n_in;
    }
}

template <int R, int NC, int NS, int CM>
cudaError_t launch_conv_tb2_t(const StencilGeom& g, const RowBands& b, int zero_top, int zero_bot, int num_sms,
                              cudaStream_t s) {
    ConvTb2Params pp;
    tma::RowStream& p = pp.s;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = g.out;
    p.pitch = g.pitch / 4;
    p.rows = g.rows;
    p.n = g.w;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    pp.zero_top = zero_top;
    pp.zero_bot = zero_bot;
    pp.slot = g.wslot;
    if (g.wslot < 0 || g.wslot >= kConvWeightSlots) return cudaErrorInvalidValue;
    tma_set_link(p, nullptr, R);
    constexpr int S = NC * 128;
    const int smem = NS * (S + 2 * kTbMargin) * 4 + 2 * (S + 8) * 4 + 2 * NS * 8;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(conv_tb2_kernel<R, NC, NS, CM>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    const int64_t ctas = tma_plan_grid(p, b, num_sms, 1, S);
    tma_record(g.rec, LK_CONV_TB2, p, ctas, (NC + 2) * 32, smem, NS, 1, NC, 2);
    if (ctas == 0) return cudaSuccess;
    conv_tb2_kernel<R, NC, NS, CM><<<(unsigned)ctas, (NC + 2) * 32, smem, s>>>(pp);
    return cudaGetLastError();
}

template <int R>
cudaError_t launch_conv_tb2_r(const StencilGeom& g, const RowBands& b, int zero_top, int zero_bot, int num_sms,
                              cudaStream_t s) {
    constexpr int NS = 12;
    const int64_t nvec = g.w / 4;
    auto go = [&](auto nc_tag) -> cudaError_t {
        constexpr int NC = decltype(nc_tag)::value;
        switch (g.col_mode) {
            case COL_WRAP: return launch_conv_tb2_t<R, NC, NS, COL_WRAP>(g, b, zero_top, zero_bot, num_sms, s);
            case COL_CLAMP: return launch_conv_tb2_t<R, NC, NS, COL_CLAMP>(g, b, zero_top, zero_bot, num_sms, s);
            default: return launch_conv_tb2_t<R, NC, NS, COL_ZERO>(g, b, zero_top, zero_bot, num_sms, s);
        }
    };
    if (nvec > 4 * 32) return go(std::integral_constant<int, 16>());
    return go(std::integral_constant<int, 4>());
}

}  // namespace conv_detail
}  // namespace mapsm
