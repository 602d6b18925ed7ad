#pragma once
// conv.cu — fp32 window convolution (cross-correlation), radius 1..4, sm_100a.
//
// Path rows a4/a5 of SURVEY §8(a), float case: Window(2D) input (Table 1
// P:L87-88, "N-dimensional convolution") -> Structured Injective output
// (P:L102).  Per output cell, exactly (reading c11):
//     acc = +0.0f; for dy=-r..r: for dx=-r..r: acc = fmaf(W[dy][dx], in[y+dy][x+dx], acc)
// so the result is bit-identical to any implementation of that definition.
//
// Design.  Each lane owns 4 consecutive output columns (one
// 128-bit load/store per row) and a warp streams down a chunk of rows.  Input
// row Y is loaded once and feeds, in the fixed tap order, the 2r+1 output rows
// y = Y-r..Y+r whose accumulators are live in registers: because rows stream
// in increasing Y, output y receives its dy = -r..r tap rows in exactly the
// required order (this is the paper's ILP over rows, taken to the
// whole chunk).  The 2r horizontal neighbours come from the adjacent lanes via
// shuffles (edge lanes load one extra float4).  Weights are a kernel parameter
// (constant bank) indexed by compile-time tap numbers, so every FFMA takes its
// weight straight from the constant bank.  No tensor cores: a 2D stencil is
// not a dense contraction and reshaping it into one would not be exact.
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

#include "kernels.h"
#include "tma_rows.cuh"

namespace mapsm {
namespace conv_detail {

#ifndef MAPSM_CONV_BIG_PL
#define MAPSM_CONV_BIG_PL 1  // TMA producer lanes for r >= 3
#endif
#ifndef MAPSM_CONV_BIG_CTAS
#define MAPSM_CONV_BIG_CTAS 1
#endif
#ifndef MAPSM_CONV_BIG_NC
#define MAPSM_CONV_BIG_NC 16
#endif
constexpr int kConvBigCtas = MAPSM_CONV_BIG_CTAS;  // CTAs per SM for r >= 3
constexpr int kConvBigNC = MAPSM_CONV_BIG_NC;      // consumer warps per CTA for r >= 3
#ifndef MAPSM_CONV_BIG_EPL
#define MAPSM_CONV_BIG_EPL 4
#endif
constexpr int kConvBigEPL = MAPSM_CONV_BIG_EPL;    // floats per lane for r >= 3

constexpr int kThreads = 256;
constexpr unsigned kFull = 0xffffffffu;

template <int R>
struct ConvParams {
    const float* in;
    float* out;
    int64_t pitch_f;  // row pitch in floats
    int64_t rows;
    int64_t w;
    int64_t nvec;     // w / 4
    int64_t warps_per_row;
    int64_t begin[2], end[2], nchunks[2];
    int top_map, bot_map, col_mode;
    float wt[(2 * R + 1) * (2 * R + 1)];
};

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

struct F4Fetch {
    float4 v, l, r;  // own vector, left/right edge vectors (edge lanes only)
};

struct ConvLane {
    int64_t vi;
    bool active, need_l, need_r;
    int64_t l_idx, r_idx;  // float index of the edge float4, -1 = synthesise (CLAMP/ZERO)
};

template <class Prm>
__device__ __forceinline__ void conv_fetch(const Prm& p, const ConvLane& c, int64_t Y, F4Fetch& f) {
    const float* row = p.in + map_row(p, Y) * p.pitch_f;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    f.v = c.active ? __ldg(reinterpret_cast<const float4*>(row + c.vi * 4)) : z;
    f.l = (c.need_l && c.l_idx >= 0) ? __ldg(reinterpret_cast<const float4*>(row + c.l_idx)) : z;
    f.r = (c.need_r && c.r_idx >= 0) ? __ldg(reinterpret_cast<const float4*>(row + c.r_idx)) : z;
}

// v[i] = in[Y][x0 - R + i], i in [0, 4 + 2R)
template <int R, class Prm>
__device__ __forceinline__ void conv_window(const Prm& p, const ConvLane& c, const F4Fetch& f,
                                            float (&v)[4 + 2 * R]) {
    const float own[4] = {f.v.x, f.v.y, f.v.z, f.v.w};
    float lft[4], rgt[4];
    lft[0] = __shfl_up_sync(kFull, f.v.x, 1);
    lft[1] = __shfl_up_sync(kFull, f.v.y, 1);
    lft[2] = __shfl_up_sync(kFull, f.v.z, 1);
    lft[3] = __shfl_up_sync(kFull, f.v.w, 1);
    rgt[0] = __shfl_down_sync(kFull, f.v.x, 1);
    rgt[1] = __shfl_down_sync(kFull, f.v.y, 1);
    rgt[2] = __shfl_down_sync(kFull, f.v.z, 1);
    rgt[3] = __shfl_down_sync(kFull, f.v.w, 1);
    if (c.need_l) {
        if (c.l_idx >= 0) {
            lft[0] = f.l.x; lft[1] = f.l.y; lft[2] = f.l.z; lft[3] = f.l.w;
        } else {
            const float e = (p.col_mode == COL_CLAMP) ? own[0] : 0.f;
            lft[0] = lft[1] = lft[2] = lft[3] = e;
        }
    }
    if (c.need_r) {
        if (c.r_idx >= 0) {
            rgt[0] = f.r.x; rgt[1] = f.r.y; rgt[2] = f.r.z; rgt[3] = f.r.w;
        } else {
            const float e = (p.col_mode == COL_CLAMP) ? own[3] : 0.f;
            rgt[0] = rgt[1] = rgt[2] = rgt[3] = e;
        }
    }
#pragma unroll
    for (int i = 0; i < R; ++i) v[i] = lft[4 - R + i];
#pragma unroll
    for (int i = 0; i < 4; ++i) v[R + i] = own[i];
#pragma unroll
    for (int i = 0; i < R; ++i) v[R + 4 + i] = rgt[i];
}

// PF = rows of loads in flight per lane; U = unroll, a multiple of both the
// accumulator ring (2R+1) and PF so every ring index is a compile-time constant.
template <int R, int PF>
__global__ void __launch_bounds__(kThreads) conv_step_kernel(const __grid_constant__ ConvParams<R> p) {
    constexpr int K = 2 * R + 1;
    constexpr int U = K * PF;
    const int lane = threadIdx.x & 31;
    const int64_t warp_gid = (int64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const int band = blockIdx.y;
    const int64_t nchunks = p.nchunks[band];
    const int64_t strip = warp_gid % p.warps_per_row;
    const int64_t chunk = warp_gid / p.warps_per_row;
    if (chunk >= nchunks) return;
    const int64_t rb = p.begin[band], nr = p.end[band] - rb;
    const int64_t ys = rb + chunk * nr / nchunks;
    const int64_t ye = rb + (chunk + 1) * nr / nchunks;
    if (ys >= ye) return;

    ConvLane c;
    c.vi = strip * 32 + lane;
    c.active = c.vi < p.nvec;
    c.need_l = c.active && (lane == 0 || c.vi == 0);
    c.need_r = c.active && (lane == 31 || c.vi == p.nvec - 1);
    c.l_idx = (c.vi == 0) ? (p.col_mode == COL_WRAP ? p.w - 4 : -1) : c.vi * 4 - 4;
    c.r_idx = (c.vi == p.nvec - 1) ? (p.col_mode == COL_WRAP ? 0 : -1) : c.vi * 4 + 4;

    const int64_t y_first = ys - R;      // first input row
    const int64_t y_last = ye + R - 1;   // last input row

    F4Fetch ring[PF];
#pragma unroll
    for (int k = 0; k < PF; ++k)
        if (y_first + k <= y_last) conv_fetch(p, c, y_first + k, ring[k]);

    float acc[K][4];
#pragma unroll
    for (int j = 0; j < K; ++j)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[j][q] = 0.f;

    for (int64_t Yb = y_first; Yb <= y_last; Yb += U) {
#pragma unroll
        for (int s = 0; s < U; ++s) {
            const int64_t Y = Yb + s;
            if (Y <= y_last) {
                const F4Fetch f = ring[s % PF];
                if (Y + PF <= y_last) conv_fetch(p, c, Y + PF, ring[s % PF]);
                float v[4 + 2 * R];
                conv_window<R>(p, c, f, v);
                // Tap row d (dy = d - R) of output y = Y + R - d; slot (s - d) mod K.
#pragma unroll
                for (int d = 0; d < K; ++d) {
                    const int64_t y = Y + R - d;
                    const int slot = ((s - d) % K + K) % K;
                    if (y >= ys && y < ye) {
                        if (d == 0) {
#pragma unroll
                            for (int q = 0; q < 4; ++q) acc[slot][q] = 0.f;
                        }
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            float a = acc[slot][q];
#pragma unroll
                            for (int e = 0; e < K; ++e) a = __fmaf_rn(p.wt[d * K + e], v[q + e], a);
                            acc[slot][q] = a;
                        }
                        if (d == K - 1 && c.active) {
                            float* o = p.out + y * p.pitch_f + c.vi * 4;
                            *reinterpret_cast<float4*>(o) =
                                make_float4(acc[slot][0], acc[slot][1], acc[slot][2], acc[slot][3]);
                        }
                    }
                }
            }
        }
    }
}

// Generic path for widths that are not a multiple of 4 (or < 4): one thread
// per output cell, per-tap boundary resolution.  Same tap order.
template <int R>
__global__ void conv_generic_kernel(const __grid_constant__ ConvParams<R> p) {
    constexpr int K = 2 * R + 1;
    const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int band = blockIdx.z;
    if (x >= p.w) return;
    for (int64_t y = p.begin[band] + blockIdx.y; y < p.end[band]; y += gridDim.y) {
    float acc = 0.f;
#pragma unroll
    for (int d = 0; d < K; ++d) {
        const float* row = p.in + map_row(p, y + d - R) * p.pitch_f;
#pragma unroll
        for (int e = 0; e < K; ++e) {
            int64_t xx = x + e - R;
            float v;
            if (xx >= 0 && xx < p.w) {
                v = __ldg(row + xx);
            } else if (p.col_mode == COL_WRAP) {
                xx %= p.w;
                if (xx < 0) xx += p.w;
                v = __ldg(row + xx);
            } else if (p.col_mode == COL_CLAMP) {
                v = __ldg(row + (xx < 0 ? 0 : p.w - 1));
            } else {
                v = 0.f;
            }
            acc = __fmaf_rn(p.wt[d * K + e], v, acc);
        }
    }
    p.out[y * p.pitch_f + x] = acc;
    }
}

// ------------------------------------------------ TMA-bulk pipelined kernel
// Rows stream through the shared-memory ring of tma_rows.cuh (producer warp +
// NC consumer warps, one CTA strip = NC x 32 x EPL floats).  Consumer lane t
// owns EPL output columns; for input row Y it reads EPL + 8 floats (its own
// plus 4 on each side, from the stage: no shuffles) and advances the 2R+1
// live accumulator rows in the fixed tap order.  The loop is unrolled by NS,
// a multiple of 2R+1, so the accumulator ring and the stage index are
// compile-time.  EPL = 4 (one 16-byte vector per lane) for every radius:
// EPL = 2 halves the unrolled code for r >= 3 but measured 12% slower on 9x9
// (profiles/r01_conv9_variants.txt), the per-row overhead doubling relative
// to the FMAs.
template <int R>
struct ConvTmaParams {
    tma::RowStream s;
    float wt[(2 * R + 1) * (2 * R + 1)];
    // weight pairs for the FFMA2 path: wp[d * 2R + m - 1] = (W[d][m-1], W[d][m]),
    // m = 1..2R, 8-byte aligned so each is one 64-bit uniform-register pair
    float2 wp[(2 * R + 1) * 2 * R];
    int slot;  // r >= kConvPairMinR: weight slot of c_conv_wp / c_conv_w
};

// FFMA2 (fma.rn.f32x2) pair accumulation, radius >= kConvPairMinR.
// Acc2 of outputs (2j, 2j+1) of a lane holds hi = out(2j), lo = out(2j+1).
// Window value m of the pair (element 2j - R + m, m = 0..2R+1) feeds out(2j)
// with tap W[m] (m <= 2R) and out(2j+1) with tap W[m-1] (m >= 1): one FFMA2
// with the value broadcast and the pair (W[m-1], W[m]) as a 64-bit uniform
// register does both for m = 1..2R; m = 0 and m = 2R+1 feed a single half
// (scalar FFMA).  Each half is an IEEE fma, RN-even, and each output still
// receives its taps in increasing dx — the oracle's fmaf chain exactly
// (reading c11).  2R FFMA2 + 2 FFMA per pair and tap row instead of
// 2(2R+1) FFMA: the r >= 3 kernels are FFMA-issue-bound.
#ifndef MAPSM_CONV_PAIR_MINR
#define MAPSM_CONV_PAIR_MINR 3
#endif
constexpr int kConvPairMinR = MAPSM_CONV_PAIR_MINR;
typedef unsigned long long Acc2;
__device__ __forceinline__ void fma_pair(Acc2& acc, float v, unsigned long long wv) {
    asm("{\n\t.reg .b64 x;\n\tmov.b64 x, {%1, %1};\n\tfma.rn.f32x2 %0, x, %2, %0;\n\t}"
        : "+l"(acc)
        : "f"(v), "l"(wv));
}
__device__ __forceinline__ void fma_lo(Acc2& acc, float w, float v) {
    asm("{\n\t.reg .f32 l, h;\n\tmov.b64 {l, h}, %0;\n\tfma.rn.f32 l, %1, %2, l;\n\tmov.b64 %0, {l, h};\n\t}"
        : "+l"(acc)
        : "f"(w), "f"(v));
}
__device__ __forceinline__ void fma_hi(Acc2& acc, float w, float v) {
    asm("{\n\t.reg .f32 l, h;\n\tmov.b64 {l, h}, %0;\n\tfma.rn.f32 h, %1, %2, h;\n\tmov.b64 %0, {l, h};\n\t}"
        : "+l"(acc)
        : "f"(w), "f"(v));
}
// The r >= 3 (FFMA2) kernels read their weights from __constant__ memory
// through a uniform slot index the compiler cannot prove loop-invariant, so
// every weight (pair) is re-loaded into a UNIFORM register (LDCU) right before
// its FFMA2s instead of being hoisted into vector registers: the FFMA2 form
// "broadcast value x uniform-register weight pair" issues at 1.91 warp-instr/
// clk/SM, the vector-register-pair form at 1.46 (tools/pipebench3.cu), and the
// hoisted weights (72 pairs = 144 registers) no longer occupy the register
// file.  Slots are per grid (mapsm_bind uploads them; kConvWeightSlots live
// r >= 3 grids at most); every translation unit has its own copy of the
// arrays (internal linkage) and its own upload function.
static __constant__ float2 c_conv_wp[kConvWeightSlots][kConvMaxPairs];
static __constant__ float c_conv_w[kConvWeightSlots][kConvMaxTaps];

// A weight (pair) load that ptxas may neither hoist nor merge; its address
// is warp-uniform, so it becomes an LDCU into a uniform register.
// `a` is a CONSTANT-space address (to_const below).
__device__ __forceinline__ unsigned long long ldc_pair(unsigned long long a) {
    unsigned long long r;
    asm volatile("ld.const.b64 %0, [%1];" : "=l"(r) : "l"(a));
    return r;
}
__device__ __forceinline__ float ldc_one(unsigned long long a) {
    float r;
    asm volatile("ld.const.f32 %0, [%1];" : "=f"(r) : "l"(a));
    return r;
}
__device__ __forceinline__ unsigned long long to_const(const void* generic) {
    unsigned long long r;
    asm("cvta.to.const.u64 %0, %1;" : "=l"(r) : "l"(generic));
    return r;
}

template <int R, int CM>
cudaError_t conv_upload_weights_t(int slot, const float* weights) {
    constexpr int K = 2 * R + 1;
    static_assert(K * K <= kConvMaxTaps && K * (K - 1) <= kConvMaxPairs, "weight slot too small");
    if (slot < 0 || slot >= kConvWeightSlots) return cudaErrorInvalidValue;
    float2 wp[K * (K - 1)];
    for (int d = 0; d < K; ++d)
        for (int m = 1; m < K; ++m) wp[d * (K - 1) + m - 1] = make_float2(weights[d * K + m - 1], weights[d * K + m]);
    cudaError_t e = cudaMemcpyToSymbol(c_conv_wp, wp, sizeof wp, sizeof(float2) * kConvMaxPairs * slot);
    if (e != cudaSuccess) return e;
    return cudaMemcpyToSymbol(c_conv_w, weights, sizeof(float) * K * K, sizeof(float) * kConvMaxTaps * slot);
}

__device__ __forceinline__ float acc_hi(Acc2 a) { return __uint_as_float((unsigned)(a >> 32)); }
__device__ __forceinline__ float acc_lo(Acc2 a) { return __uint_as_float((unsigned)a); }

template <int EPL>
struct VecF;
template <>
struct VecF<4> {
    using T = float4;
};
template <>
struct VecF<2> {
    using T = float2;
};

template <int R, int NC, int NS, int CM, int EPL, bool FUSED>
__global__ void __launch_bounds__((NC + 1) * 32, (R <= 2 ? 1 : kConvBigCtas)) conv_tma_kernel(const __grid_constant__ ConvTmaParams<R> pp) {
    constexpr int K = 2 * R + 1;
    static_assert(NS % K == 0, "NS must be a multiple of 2R+1");
    // consumer unroll: NS rows for the HBM-bound radii (static accumulator
    // slots); the FMA-bound ones rotate their accumulators and run one row
    // per iteration (their unrolled rows did not fit the instruction cache)
    constexpr int U = R >= kConvPairMinR ? 1 : NS;
    static_assert(NS % U == 0, "the unroll must divide NS");
    static_assert(R <= 4, "16-byte stage margins cover r <= 4");
    using G = tma::Geom<NC, EPL>;
    using VT = typename VecF<EPL>::T;
    // this grid's weights: constant-space addresses (warp-uniform)
    const unsigned long long cwp = to_const(&c_conv_wp[R >= kConvPairMinR ? pp.slot : 0][0]);
    const unsigned long long cw = to_const(&c_conv_w[R >= kConvPairMinR ? pp.slot : 0][0]);
    const tma::RowStream& p = pp.s;
    extern __shared__ __align__(128) uint8_t smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * G::kStageBytes);
    uint64_t* empty = full + NS;
    tma::init_barriers<NS>(full, empty, NC);
    tma::pdl_wait_and_release();
    // warp index through a full-mask shuffle: ptxas then knows the role
    // branch below is warp-uniform and may use the uniform datapath (LDCU
    // weights) inside the consumer code
    const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
    tma::SegIter it = tma::seg_iter(p);
    tma::Seg sg;
    tma::RingPos ring;

    const tma::HaloLink& Lk = p.link;
    if (warp == NC) {
        constexpr int PL = R <= 2 ? 2 : MAPSM_CONV_BIG_PL;  // producer lanes (see tma_rows.cuh)
        if (lane < PL) {
            while (tma::seg_next<NC, EPL>(p, it, sg)) {
                // (the mailbox is read only by segments that load halo rows)
                const unsigned int halo_target =
                    FUSED && (sg.ys < R || sg.ye + R > p.rows) ? halo_wait_target(Lk, p.nstrips) : 0u;
                tma::produce_align<NS, PL>(full, empty, ring, lane);
                tma::produce<NC, NS, CM == COL_WRAP, EPL, PL>(p, sg, smem, full, empty, sg.ys - R, sg.ye - sg.ys + 2 * R,
                                                         ring, halo_target, lane);
            }
        }
        if constexpr (FUSED) tma::finish_launch_producer((NC + 1) * 32, p.link_ctas);
        return;
    }
    {
    const int t = warp * 32 + lane;
    constexpr bool PAIR = R >= kConvPairMinR;
    static_assert(EPL % 2 == 0, "pairs of outputs");
    float acc[PAIR ? 1 : K][EPL];
    Acc2 acc2[PAIR ? K : 1][EPL / 2];
    // Per segment: the linked body (boundary rows also stored into the
    // neighbours' halos, then signalled) only for segments with boundary
    // rows; interior segments of a fused launch run the plain body.
    auto seg_body = [&](auto link_tag) {
        constexpr bool LINK = decltype(link_tag)::value;
        tma::consume_align<NS>(full, empty, ring, lane);
        uint32_t ph = ring.phase;  // segment starts at stage 0
        const int n_out = (int)(sg.ye - sg.ys);
        const int n_in = n_out + 2 * R;  // input rows ys-R .. ye+R-1
        const bool active = t * EPL < (int)sg.seg;
        const bool row_first = sg.first_strip && t == 0;
        const bool row_last = sg.last_strip && (t + 1) * EPL == (int)sg.seg;
        const bool whole = sg.first_strip && sg.last_strip;
        float* out0 = static_cast<float*>(p.out) + sg.ys * p.pitch + sg.e0 + t * EPL;

        // Input row j: output rows o = j - d (d = 0..2R, tap row dy = d - R)
        // take their d-th tap row from it; o starts at d == 0 and completes
        // at d == 2R.
        // Input row j lives in ring stage `stg` (= j % NS) with phase `phs`;
        // k = j % U is static (U = the unroll: a multiple of 2R+1 dividing NS).
        auto step = [&](int j, int k, int stg, uint32_t phs, bool check) {
            tma::mbar_wait(&full[stg], phs);
            const float* st = reinterpret_cast<const float*>(smem + stg * G::kStageBytes);
            // buf[m] = stage float t*EPL + m = strip element t*EPL - 4 + m
            float buf[EPL + 8];
#pragma unroll
            for (int m = 0; m < EPL + 8; m += EPL) {
                // WRAP at the ends of a whole-row strip: the other end of the row
                // is in the stage itself (no margin copy was made)
                int off = t * EPL + m;
                if (CM == COL_WRAP && whole) {
                    if (m < 4 && row_first) off = (int)sg.seg + m;           // elements seg-4+m
                    if (m >= 4 + EPL && row_last) off = m - EPL;             // elements m-4-EPL..
                }
                const VT q = *reinterpret_cast<const VT*>(st + off);
                if constexpr (EPL == 4) {
                    buf[m] = q.x; buf[m + 1] = q.y; buf[m + 2] = q.z; buf[m + 3] = q.w;
                } else {
                    buf[m] = q.x; buf[m + 1] = q.y;
                }
            }
            __syncwarp();
            if (lane == 0) tma::mbar_arrive(&empty[stg]);
            if (CM != COL_WRAP) {
                if (row_first) {
                    const float e = (CM == COL_CLAMP) ? buf[4] : 0.f;
#pragma unroll
                    for (int m = 0; m < 4; ++m) buf[m] = e;
                }
                if (row_last) {
                    const float e = (CM == COL_CLAMP) ? buf[3 + EPL] : 0.f;
#pragma unroll
                    for (int m = 4 + EPL; m < 8 + EPL; ++m) buf[m] = e;
                }
            }
            // v[q + e] = element t*EPL + q + e - R  ->  buf[4 - R + q + e]
            // Tap row d of output o = j - d lives in slot (k - d) mod K (== o mod K, NS % K == 0).
            if constexpr (PAIR) {
                // Rotating accumulators: acc2[d] is output row o = j - d.  Shift them
                // (the finished row j - 2R left at the end of the previous row), start
                // output j at +0.0f, then apply this input row's taps.  Window value m
                // outermost, then tap row d and pair jp: 2R+1 x EPL/2 independent
                // chains between dependent FFMA2s; each chain takes m (= its dx) in
                // increasing order.  No skip tests: rows outside [0, n_out) are
                // computed and never stored.
#pragma unroll
                for (int d = K - 1; d > 0; --d)
#pragma unroll
                    for (int jp = 0; jp < EPL / 2; ++jp) acc2[d][jp] = acc2[d - 1][jp];
#pragma unroll
                for (int jp = 0; jp < EPL / 2; ++jp) acc2[0][jp] = 0ull;  // (+0.0f, +0.0f)
#pragma unroll
                for (int m = 0; m <= K; ++m) {
#pragma unroll
                    for (int d = 0; d < K; ++d) {
                        if (m == 0 || m == K) {
                            const float w = ldc_one(cw + 4 * (d * K + (m == 0 ? 0 : K - 1)));
#pragma unroll
                            for (int jp = 0; jp < EPL / 2; ++jp) {
                                const float v = buf[4 - R + 2 * jp + m];
                                if (m == 0) fma_hi(acc2[d][jp], w, v);
                                else fma_lo(acc2[d][jp], w, v);
                            }
                        } else {
                            const unsigned long long w = ldc_pair(cwp + 8 * (d * (K - 1) + m - 1));
#pragma unroll
                            for (int jp = 0; jp < EPL / 2; ++jp) fma_pair(acc2[d][jp], buf[4 - R + 2 * jp + m], w);
                        }
                    }
                }
            }
#pragma unroll
            for (int d = 0; d < K; ++d) {
                const int o = j - d;
                const int slot = PAIR ? d : ((k - d) % K + K) % K;
                if (PAIR ? (d == K - 1 && o >= 0) : (!check || (o >= 0 && o < n_out))) {
                    float res[EPL];
                    if constexpr (PAIR) {
#pragma unroll
                        for (int jp = 0; jp < EPL / 2; ++jp) {
                            res[2 * jp] = acc_hi(acc2[slot][jp]);
                            res[2 * jp + 1] = acc_lo(acc2[slot][jp]);
                        }
                    } else {
#pragma unroll
                        for (int q = 0; q < EPL; ++q) {
                            float a = (d == 0) ? 0.f : acc[slot][q];
#pragma unroll
                            for (int e = 0; e < K; ++e) a = __fmaf_rn(pp.wt[d * K + e], buf[4 - R + q + e], a);
                            acc[slot][q] = a;
                            res[q] = a;
                        }
                    }
                    if (d == K - 1 && active) {
                        using OT = typename VecF<EPL>::T;
                        OT ov;
                        if constexpr (EPL == 4)
                            ov = make_float4(res[0], res[1], res[2], res[3]);
                        else
                            ov = make_float2(res[0], res[1]);
                        *reinterpret_cast<OT*>(out0 + (int64_t)o * p.pitch) = ov;
                        if constexpr (LINK) {  // boundary rows also go to the neighbours' halos
                            const int64_t yo = sg.ys + o;
                            if (Lk.dst_up && yo < R)
                                *reinterpret_cast<OT*>(reinterpret_cast<float*>(Lk.dst_up) + yo * p.pitch + sg.e0 +
                                                       t * EPL) = ov;
                            if (Lk.dst_down && yo >= p.rows - R)
                                *reinterpret_cast<OT*>(reinterpret_cast<float*>(Lk.dst_down) +
                                                       (yo - (p.rows - R)) * p.pitch + sg.e0 + t * EPL) = ov;
                        }
                    }
                }
            }
        };

        const uint32_t ph0 = ph;
        // blocks of U rows: the first and last with full checks, the steady
        // ones (every output touched lies in [0, n_out)) without
        auto block = [&](int j0, bool check) {
            const int sbase = j0 % NS;                                // a multiple of U
            const uint32_t phb = ph0 ^ (uint32_t)((j0 / NS) & 1);     // the stage's use count parity
#pragma unroll
            for (int k = 0; k < U; ++k)
                if (!check || j0 + k < n_in) step(j0 + k, k, sbase + k, phb, check);
        };
        if constexpr (PAIR) {
            // one row per iteration (rotating accumulators: no static slots),
            // so the loop body stays small enough for the instruction cache
            int stg = 0;
            uint32_t phs = ph0;
#pragma unroll 1
            for (int j = 0; j < n_in; ++j) {
                step(j, 0, stg, phs, false);
                if (++stg == NS) {
                    stg = 0;
                    phs ^= 1u;
                }
            }
        } else {
            int j = 0;
            if (n_in >= U) {
                block(0, true);  // first block: o < 0 for d > k
                for (j = U; j + U <= n_in && j + U - 1 < n_out; j += U) block(j, false);
            }
            for (; j < n_in; j += U) block(j, true);
        }
        ring.stage = n_in % NS;
        ring.phase = ph0 ^ (uint32_t)((n_in / NS) & 1);
        ring.count += n_in;
        if constexpr (LINK) {
            if (Lk.dst_up && sg.ys < R) {
                const int64_t e = sg.ye < R ? sg.ye : R;
                tma::publish_delivery(Lk.sig_up, (unsigned int)(e - sg.ys), NC);
            }
            if (Lk.dst_down && sg.ye > p.rows - R) {
                const int64_t b0 = sg.ys > p.rows - R ? sg.ys : p.rows - R;
                tma::publish_delivery(Lk.sig_down, (unsigned int)(sg.ye - b0), NC);
            }
        }
    };
    while (tma::seg_next<NC, EPL>(p, it, sg)) {
        if constexpr (FUSED) {
            if (sg.ys < R || sg.ye > p.rows - R) {
                seg_body(std::true_type{});
                continue;
            }
        }
        seg_body(std::false_type{});
    }
    }
    if constexpr (FUSED) tma::finish_launch_consumers(Lk.mine, (NC + 1) * 32, p.link_ctas);
}

template <int R, int NC, int NS, int CM, int EPL>
cudaError_t launch_conv_tma_t(const StencilGeom& g, const RowBands& b, const float* weights, int num_sms,
                              cudaStream_t s, const FusedLink* link) {
    using G = tma::Geom<NC, EPL>;
    constexpr int K = 2 * R + 1;
    ConvTmaParams<R> pp;
    tma::RowStream& p = pp.s;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = g.out;
    p.pitch = g.pitch / 4;
    p.rows = g.rows;
    p.n = g.w;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    for (int j = 0; j < K * K; ++j) pp.wt[j] = weights[j];
    for (int d = 0; d < K; ++d)
        for (int m = 1; m < K; ++m) pp.wp[d * (K - 1) + m - 1] = make_float2(weights[d * K + m - 1], weights[d * K + m]);
    pp.slot = g.wslot;
    if (R >= kConvPairMinR && (g.wslot < 0 || g.wslot >= kConvWeightSlots)) return cudaErrorInvalidValue;
    const int smem = NS * G::kStageBytes + 2 * NS * 8;
    static int ctas_per_sm = 0;
    if (ctas_per_sm == 0) {
        auto kfn = conv_tma_kernel<R, NC, NS, CM, EPL, false>;
        for (auto kf : {conv_tma_kernel<R, NC, NS, CM, EPL, false>, conv_tma_kernel<R, NC, NS, CM, EPL, true>}) {
            cudaError_t e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e != cudaSuccess) return e;
        }
        cudaError_t e;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctas_per_sm, kfn, (NC + 1) * 32, smem);
        if (e != cudaSuccess) return e;
        if (ctas_per_sm < 1) ctas_per_sm = 1;
        // HBM-bound radii: ~16 consumer warps per SM; FMA-bound radii (r >= 3,
        // 49-81 taps): kConvBigCtas CTAs per SM.
        const int want = R <= 2 ? (16 / NC > 0 ? 16 / NC : 1) : kConvBigCtas;
        if (want < ctas_per_sm) ctas_per_sm = want;
    }
    tma_set_link(p, link, R);
    const int64_t ctas = tma_plan_grid(p, b, num_sms, ctas_per_sm, G::kStripElems, link != nullptr);
    tma_record(g.rec, LK_CONV_TMA, p, ctas, (NC + 1) * 32, smem, NS, 1, NC);
    if (ctas == 0) return cudaSuccess;
    if (link)
        return tma_launch(conv_tma_kernel<R, NC, NS, CM, EPL, true>, (unsigned)ctas, (NC + 1) * 32, smem, s, pp,
                          false);  // (measured: PDL costs the fused conv launch ~2 us per generation)
    else
        return tma_launch(conv_tma_kernel<R, NC, NS, CM, EPL, false>, (unsigned)ctas, (NC + 1) * 32, smem, s, pp,
                          g.pdl);
}

// The FMA-bound radii (r >= 3) are compiled one column mode per translation
// unit (conv_r<R>_cm<CM>.cu) so their large unrolled kernels build in
// parallel; conv_r<R>.cu declares them extern.
#define MAPSM_CONV_BIG_INST(KW, R, NS, CM)                                                                        \
    KW template cudaError_t conv_detail::conv_upload_weights_t<R, CM>(int, const float*);                       \
    KW template cudaError_t conv_detail::launch_conv_tma_t<R, 2, NS, CM, conv_detail::kConvBigEPL>(               \
        const StencilGeom&, const RowBands&, const float*, int, cudaStream_t, const FusedLink*);                 \
    KW template cudaError_t                                                                                      \
    conv_detail::launch_conv_tma_t<R, conv_detail::kConvBigNC, NS, CM, conv_detail::kConvBigEPL>(                \
        const StencilGeom&, const RowBands&, const float*, int, cudaStream_t, const FusedLink*);
#define MAPSM_CONV_BIG_INST_ALL(KW, R, NS) \
    MAPSM_CONV_BIG_INST(KW, R, NS, COL_WRAP) MAPSM_CONV_BIG_INST(KW, R, NS, COL_CLAMP) MAPSM_CONV_BIG_INST(KW, R, NS, COL_ZERO)

template <int R, int NS>
cudaError_t launch_conv_tma(const StencilGeom& g, const RowBands& b, const float* weights, int num_sms,
                            cudaStream_t s, const FusedLink* link) {
    constexpr int EPL = R <= 2 ? 4 : kConvBigEPL;
    const int64_t nvec = g.w / EPL;
    auto go = [&](auto nc_tag) -> cudaError_t {
        constexpr int NC = decltype(nc_tag)::value;
        switch (g.col_mode) {
            case COL_WRAP: return launch_conv_tma_t<R, NC, NS, COL_WRAP, EPL>(g, b, weights, num_sms, s, link);
            case COL_CLAMP: return launch_conv_tma_t<R, NC, NS, COL_CLAMP, EPL>(g, b, weights, num_sms, s, link);
            default: return launch_conv_tma_t<R, NC, NS, COL_ZERO, EPL>(g, b, weights, num_sms, s, link);
        }
    };
    if constexpr (R <= 2) {
        if (nvec > 8 * 32) return go(std::integral_constant<int, 16>());
        if (nvec > 4 * 32) return go(std::integral_constant<int, 8>());
        if (nvec > 2 * 32) return go(std::integral_constant<int, 4>());
        return go(std::integral_constant<int, 2>());
    } else {
        // FMA-bound radii: kConvBigNC (16) consumer warps + the producer warp,
        // one CTA per SM.  With the weights in __constant__ slots (uniform
        // registers) and rotating accumulators the consumer needs < 120
        // registers, so 4 consumer warps per SM sub-partition hide the FFMA2
        // and LDCU latencies (measured: 7 warps 281, 12: 317, 16: 337, 20: 335 G
        // cell-updates/s on 32768 x 4096, profiles/r02_conv9_variants.txt).
        // Narrow rows: 2.
        if (nvec > (kConvBigNC / 2) * 32) return go(std::integral_constant<int, kConvBigNC>());
        return go(std::integral_constant<int, 2>());
    }
}

template <int R, int PF>
cudaError_t launch_conv_t(const StencilGeom& g, const RowBands& b, const float* weights, int num_sms,
                          cudaStream_t s) {
    constexpr int K = 2 * R + 1;
    ConvParams<R> p;
    p.in = static_cast<const float*>(g.in);
    p.out = static_cast<float*>(g.out);
    p.pitch_f = g.pitch / 4;
    p.rows = g.rows;
    p.w = g.w;
    p.nvec = g.w / 4;
    p.warps_per_row = (p.nvec + 31) / 32;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.col_mode = g.col_mode;
    for (int i = 0; i < K * K; ++i) p.wt[i] = weights[i];
    for (int i = 0; i < 2; ++i) {
        p.begin[i] = p.end[i] = 0;
        p.nchunks[i] = 0;
    }
    const bool fast = (g.w % 4 == 0) && (g.pitch % 16 == 0) && g.w >= 4;
    if (!fast) {
        int64_t maxr = 0;
        for (int i = 0; i < b.nbands; ++i) {
            p.begin[i] = b.begin[i];
            p.end[i] = b.end[i];
            if (b.end[i] - b.begin[i] > maxr) maxr = b.end[i] - b.begin[i];
        }
        if (maxr <= 0) return cudaSuccess;
        dim3 grid((unsigned)((g.w + 127) / 128), (unsigned)(maxr < 4096 ? maxr : 4096), (unsigned)b.nbands);
        if (g.rec) {
            *g.rec = LaunchRec();
            g.rec->kernel = LK_CONV_GENERIC;
            g.rec->ctas = (int64_t)grid.x * grid.y * grid.z;
            g.rec->threads = 128;
        }
        conv_generic_kernel<R><<<grid, 128, 0, s>>>(p);
        return cudaGetLastError();
    }
    static int blocks_per_sm = 0;
    if (blocks_per_sm == 0) {
        cudaError_t e =
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, conv_step_kernel<R, PF>, kThreads, 0);
        if (e != cudaSuccess) return e;
        if (blocks_per_sm < 1) blocks_per_sm = 1;
    }
    const int64_t resident_warps = (int64_t)num_sms * blocks_per_sm * (kThreads / 32);
    int64_t max_warps = 0;
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
        g.rec->kernel = LK_CONV_REG;
        g.rec->ctas = (int64_t)grid.x * grid.y;
        g.rec->threads = kThreads;
    }
    conv_step_kernel<R, PF><<<grid, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace conv_detail

template <int R>
#ifndef MAPSM_CONV_BIG_RING
#define MAPSM_CONV_BIG_RING 2
#endif
// ring stages: multiples of 2R+1; the FMA-bound radii keep MAPSM_CONV_BIG_RING
// accumulator cycles of rows in flight
constexpr int kConvNS = R == 1 ? 12 : R == 2 ? 10 : (2 * R + 1) * MAPSM_CONV_BIG_RING;

template <int R>
cudaError_t launch_conv_radius(const StencilGeom& g, const RowBands& b, const float* weights, int num_sms,
                               cudaStream_t s, const FusedLink* link) {
    constexpr int kNS = kConvNS<R>;
    constexpr int kPF = R <= 2 ? 2 : 1;
#ifndef MAPSM_CONV_REGS
    if (g.w % 4 == 0 && g.w >= 4 && g.pitch % 16 == 0) {
        return conv_detail::launch_conv_tma<R, kNS>(g, b, weights, num_sms, s, link);
    }
#endif
    if (link || b.nbands > 2) return cudaErrorInvalidValue;  // fused exchange needs the TMA kernel
    return conv_detail::launch_conv_t<R, kPF>(g, b, weights, num_sms, s);
}

}  // namespace mapsm
