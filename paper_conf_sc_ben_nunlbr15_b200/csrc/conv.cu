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

#include "kernels.h"

namespace mapsm {
namespace {

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
    conv_step_kernel<R, PF><<<grid, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_conv_step(const StencilGeom& g, const RowBands& b, int r, const float* weights,
                             int num_sms, cudaStream_t s) {
    switch (r) {
        case 1: return launch_conv_t<1, 2>(g, b, weights, num_sms, s);
        case 2: return launch_conv_t<2, 2>(g, b, weights, num_sms, s);
        case 3: return launch_conv_t<3, 1>(g, b, weights, num_sms, s);
        case 4: return launch_conv_t<4, 1>(g, b, weights, num_sms, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace mapsm
