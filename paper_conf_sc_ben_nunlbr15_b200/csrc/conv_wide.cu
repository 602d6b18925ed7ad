// conv_wide.cu — fp32 window convolution for radii 5..8 (SURVEY §8(f)
// NEXT-2, "r > 4 fp32"), sm_100a.
//
// Same operation and tap order as conv_impl.cuh (Table 1; reading
// c11: acc = +0.0f; for dy = -r..r: for dx = -r..r: acc = fmaf(W, x, acc)),
// so results are bit-identical to the oracle.  The TMA row pipeline's 16-byte
// stage margins stop at r = 4; wider windows use a shared-memory tile:
//   * a CTA (8 warps) owns a 32-row x 128-column output tile and stages the
//     (32 + 2R) x (128 + 2R) input tile once (row map for halo / WRAP /
//     CLAMP rows, column WRAP / CLAMP / ZERO resolved while staging);
//   * warp w computes rows 4w..4w+3 of the tile, lane l columns 4l..4l+3: for
//     every tap row it reads its 4 + 2R window values with 16-byte LDS into
//     registers and runs the 2R+1 taps over its 4 accumulators.
// (2R+1)^2 = 121..289 FFMA per cell, FMA-bound; the input tile is re-read
// from HBM/L2 with a (32+2R)(128+2R)/(32*128) = 1.3..1.6x halo overhead.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace mapsm {
namespace wide {

constexpr int kTX = 128, kTY = 32, kThreads = 256;

template <int R>
struct WideParams {
    const float* in;
    float* out;
    int64_t pitch_f;  // floats between rows
    int64_t rows, w;
    int64_t begin[3], end[3];  // output-row bands
    int nbands;
    int64_t tiles_x, tiles_y[3];  // tiles per band
    int top_map, bot_map, col_mode;
    float wt[(2 * R + 1) * (2 * R + 1)];
};

template <int R>
__device__ __forceinline__ int64_t map_row(const WideParams<R>& p, int64_t y) {
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
    return y;  // ROWMAP_HALO: the halo row itself (exchanged, or zero)
}

template <int R>
__global__ void __launch_bounds__(kThreads) conv_wide_kernel(const __grid_constant__ WideParams<R> p) {
    constexpr int K = 2 * R + 1;
    constexpr int SW = (kTX + 2 * R + 3) / 4 * 4 + 4;  // smem row pitch (floats, multiple of 4)
    constexpr int SH = kTY + 2 * R;
    constexpr int NV = (4 + 2 * R + 3) / 4;            // float4 loads per window row
    __shared__ __align__(16) float tile[SH * SW];

    // tile -> (band, ty, tx)
    int64_t t = blockIdx.x;
    int band = 0;
    while (band + 1 < p.nbands && t >= p.tiles_x * p.tiles_y[band]) {
        t -= p.tiles_x * p.tiles_y[band];
        ++band;
    }
    const int64_t ty = t / p.tiles_x, tx = t % p.tiles_x;
    const int64_t y0 = p.begin[band] + ty * kTY;  // first output row of the tile
    const int64_t x0 = tx * kTX;                  // first output column
    const int64_t yend = p.end[band];

    // stage the input tile: smem (i, j) <- input (y0 - R + i, x0 - R + j)
    for (int idx = threadIdx.x; idx < SH * SW; idx += kThreads) {
        const int i = idx / SW, j = idx % SW;
        const int64_t y = y0 - R + i;
        int64_t x = x0 - R + j;
        float v = 0.f;
        if (j < kTX + 2 * R && y < yend + R) {
            bool ok = true;
            if (x < 0 || x >= p.w) {
                if (p.col_mode == COL_WRAP) {
                    x %= p.w;
                    if (x < 0) x += p.w;
                } else if (p.col_mode == COL_CLAMP) {
                    x = x < 0 ? 0 : p.w - 1;
                } else {
                    ok = false;
                }
            }
            if (ok) v = __ldg(p.in + map_row(p, y) * p.pitch_f + x);
        }
        tile[idx] = v;
    }
    __syncthreads();

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll 1
    for (int rr = 0; rr < 4; ++rr) {
        const int oy = warp * 4 + rr;  // output row within the tile
        if (y0 + oy >= yend) break;
        float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll 1
        for (int d = 0; d < K; ++d) {
            // window row: smem row oy + d, columns 4*lane .. 4*lane + 3 + 2R
            const float4* src = reinterpret_cast<const float4*>(tile + (oy + d) * SW + 4 * lane);
            float v[NV * 4];
#pragma unroll
            for (int k = 0; k < NV; ++k) {
                const float4 q = src[k];
                v[4 * k] = q.x; v[4 * k + 1] = q.y; v[4 * k + 2] = q.z; v[4 * k + 3] = q.w;
            }
#pragma unroll
            for (int e = 0; e < K; ++e) {
                const float wv = p.wt[d * K + e];
#pragma unroll
                for (int q = 0; q < 4; ++q) acc[q] = __fmaf_rn(wv, v[q + e], acc[q]);
            }
        }
        const int64_t x = x0 + 4 * lane;
        float* o = p.out + (y0 + oy) * p.pitch_f + x;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (x + q < p.w) o[q] = acc[q];
    }
}

template <int R>
cudaError_t launch(const StencilGeom& g, const RowBands& b, const float* weights, cudaStream_t s) {
    constexpr int K = 2 * R + 1;
    WideParams<R> p;
    p.in = static_cast<const float*>(g.in);
    p.out = static_cast<float*>(g.out);
    p.pitch_f = g.pitch / 4;
    p.rows = g.rows;
    p.w = g.w;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.col_mode = g.col_mode;
    for (int i = 0; i < K * K; ++i) p.wt[i] = weights[i];
    p.tiles_x = (g.w + kTX - 1) / kTX;
    p.nbands = b.nbands;
    int64_t tiles = 0;
    for (int i = 0; i < 3; ++i) {
        p.begin[i] = i < b.nbands ? b.begin[i] : 0;
        p.end[i] = i < b.nbands ? b.end[i] : 0;
        const int64_t nr = p.end[i] - p.begin[i];
        p.tiles_y[i] = nr > 0 ? (nr + kTY - 1) / kTY : 0;
        tiles += p.tiles_x * p.tiles_y[i];
    }
    if (tiles == 0) return cudaSuccess;
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_CONV_WIDE;
        g.rec->ctas = tiles;
        g.rec->threads = kThreads;
    }
    conv_wide_kernel<R><<<(unsigned)tiles, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace wide

cudaError_t launch_conv_wide(const StencilGeom& g, const RowBands& b, int r, const float* weights, cudaStream_t s) {
    switch (r) {
        case 5: return wide::launch<5>(g, b, weights, s);
        case 6: return wide::launch<6>(g, b, weights, s);
        case 7: return wide::launch<7>(g, b, weights, s);
        case 8: return wide::launch<8>(g, b, weights, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace mapsm
