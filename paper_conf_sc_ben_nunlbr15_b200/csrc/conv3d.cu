// conv3d.cu — Window(3D) fp32 convolution, radius 1..2, sm_100a (SURVEY §8(f)
// NEXT-2).
//
// Paper: Window (3D) input pattern with a Structured Injective output — "each
// image in the batch is separately convolved in three dimensions ... This
// corresponds to the Window (3D) input memory access pattern, using the
// Structured Injective output access pattern" (§5.3); Table 1
// P:L87-88 "N-dimensional convolution".  Per output cell, exactly (DESIGN.md
// reading v1, the 3-D form of reading c11):
//     acc = +0.0f
//     for dz = -r..r: for dy = -r..r: for dx = -r..r:
//         acc = fmaf(W[dz][dy][dx], in[z+dz][y+dy][x+dx], acc)
// so results are bit-identical to any implementation of that definition.
//
// Design: the volume is partitioned in planes (z) over the
// slabs, exactly like the rows of the 2-D path, so the halo exchange, plane
// maps (ROWMAP_*) and double buffering are the 2-D runtime's.  A CTA owns a
// TX x TY (64 x 16) output tile of the (y, x) plane and streams a chunk of
// planes in increasing z ("2.5-D blocking"): each input plane's tile plus its
// r-wide y/x apron is staged ONCE in shared memory (y/x boundary resolved while
// staging, the next plane's loads in flight in registers during the compute),
// and feeds the 2r+1 output planes whose accumulators are live in registers.
// Because planes stream in increasing z, output plane z receives its dz =
// -r..r tap planes in order — the paper's ILP over rows taken to
// the third dimension.  Each thread owns 4 consecutive x (one 128-bit store)
// of one row, reading its (4 + 2r)-wide window rows with three 16-byte LDS.
// Weights are a kernel parameter (constant bank).  No tensor cores: a stencil
// is not a dense contraction and a GEMM reshaping would not be exact.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace mapsm {
namespace {

constexpr int TX = 64;       // output columns per CTA (16 lanes x 4 floats)
constexpr int TY = 16;       // output rows per CTA
constexpr int NT = 256;      // threads per CTA
constexpr int SW = TX + 8;   // smem row stride: tile column c in [-4, TX+4) lives at index c + 4

template <int R>
struct Conv3Params {
    const float* in;   // owned plane 0, row 0 of the input buffer
    float* out;
    int64_t ppitch;    // plane pitch (floats)
    int64_t rpitch;    // row pitch (floats)
    int64_t planes, h, w;
    int tiles_x;
    int nbands;
    int64_t zbeg[3], zend[3], nchunks[3];
    int64_t zc;        // planes per chunk
    int top_map, bot_map, mode;  // plane maps (ROWMAP_*), y/x boundary (ColMode)
    float wt[(2 * R + 1) * (2 * R + 1) * (2 * R + 1)];
};

// Index along an axis of n cells under the in-plane boundary; -1 = zero cell.
__device__ __forceinline__ int64_t axis_map(int64_t i, int64_t n, int mode) {
    if (i >= 0 && i < n) return i;
    if (mode == COL_WRAP) {
        int64_t m = i % n;
        return m < 0 ? m + n : m;
    }
    if (mode == COL_CLAMP) return i < 0 ? 0 : n - 1;
    return -1;
}

// Slab-local plane index an input plane Z reads (halo planes live at -R..-1
// and planes..planes+R-1 of the buffer).
__device__ __forceinline__ int64_t plane_map(int64_t Z, int64_t planes, int top_map, int bot_map) {
    if (Z >= 0 && Z < planes) return Z;
    const int m = Z < 0 ? top_map : bot_map;
    if (m == ROWMAP_WRAP) {
        int64_t q = Z % planes;
        return q < 0 ? q + planes : q;
    }
    if (m == ROWMAP_CLAMP) return Z < 0 ? 0 : planes - 1;
    return Z;  // ROWMAP_HALO
}

template <int R>
struct Stage {
    static constexpr int ROWS = TY + 2 * R;
    static constexpr int NV = ROWS * (TX / 4);   // float4 items (interior columns)
    static constexpr int NE = ROWS * 2 * R;      // scalar items (apron columns)
    static constexpr int KV = (NV + NT - 1) / NT;
    static constexpr int KE = (NE + NT - 1) / NT;
    float4 v[KV];
    float e[KE];
};

template <int R>
__device__ __forceinline__ void stage_load(const Conv3Params<R>& p, Stage<R>& st, int64_t Z, int64_t x0, int64_t y0) {
    const int64_t zp = plane_map(Z, p.planes, p.top_map, p.bot_map);
    const float* plane = p.in + zp * p.ppitch;
#pragma unroll
    for (int k = 0; k < Stage<R>::KV; ++k) {
        const int idx = threadIdx.x + k * NT;
        float4 val = make_float4(0.f, 0.f, 0.f, 0.f);
        if (idx < Stage<R>::NV) {
            const int row = idx / (TX / 4), vq = idx % (TX / 4);
            const int64_t y = axis_map(y0 - R + row, p.h, p.mode);
            const int64_t x = x0 + 4 * vq;
            if (y >= 0) {
                const float* rp = plane + y * p.rpitch;
                if (x + 3 < p.w) {
                    val = __ldg(reinterpret_cast<const float4*>(rp + x));
                } else {
                    float t[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int64_t xx = axis_map(x + i, p.w, p.mode);
                        t[i] = xx >= 0 ? __ldg(rp + xx) : 0.f;
                    }
                    val = make_float4(t[0], t[1], t[2], t[3]);
                }
            }
        }
        st.v[k] = val;
    }
#pragma unroll
    for (int k = 0; k < Stage<R>::KE; ++k) {
        const int idx = threadIdx.x + k * NT;
        float val = 0.f;
        if (idx < Stage<R>::NE) {
            const int row = idx / (2 * R), q = idx % (2 * R);
            const int c = q < R ? q - R : TX + (q - R);
            const int64_t y = axis_map(y0 - R + row, p.h, p.mode);
            const int64_t x = axis_map(x0 + c, p.w, p.mode);
            if (y >= 0 && x >= 0) val = __ldg(plane + y * p.rpitch + x);
        }
        st.e[k] = val;
    }
}

template <int R>
__device__ __forceinline__ void stage_store(float* sm, const Stage<R>& st) {
#pragma unroll
    for (int k = 0; k < Stage<R>::KV; ++k) {
        const int idx = threadIdx.x + k * NT;
        if (idx < Stage<R>::NV) {
            const int row = idx / (TX / 4), vq = idx % (TX / 4);
            *reinterpret_cast<float4*>(sm + row * SW + 4 + 4 * vq) = st.v[k];
        }
    }
#pragma unroll
    for (int k = 0; k < Stage<R>::KE; ++k) {
        const int idx = threadIdx.x + k * NT;
        if (idx < Stage<R>::NE) {
            const int row = idx / (2 * R), q = idx % (2 * R);
            const int c = q < R ? q - R : TX + (q - R);
            sm[row * SW + 4 + c] = st.e[k];
        }
    }
}

template <int R>
__device__ __forceinline__ void store_out(const Conv3Params<R>& p, int64_t z, int64_t y, int64_t x, const float* a) {
    if (y >= p.h || x >= p.w) return;
    float* op = p.out + z * p.ppitch + y * p.rpitch + x;
    if (x + 3 < p.w) {
        *reinterpret_cast<float4*>(op) = make_float4(a[0], a[1], a[2], a[3]);
    } else {
        for (int i = 0; i < 4 && x + i < p.w; ++i) op[i] = a[i];
    }
}

// One input plane (step j of the chunk, J = j mod K compile-time): every live
// accumulator slot takes its 9 (R=1) / 25 (R=2) taps of this plane.
template <int R, int J>
__device__ __forceinline__ void compute_plane(const Conv3Params<R>& p, const float* sm, float (&acc)[2 * R + 1][4],
                                              int lx, int ly) {
    constexpr int K = 2 * R + 1;
#pragma unroll
    for (int dy = -R; dy <= R; ++dy) {
        const float* row = sm + (ly + R + dy) * SW + 4 * lx;   // index 4*lx = tile column 4*lx - 4
        const float4 q0 = *reinterpret_cast<const float4*>(row);
        const float4 q1 = *reinterpret_cast<const float4*>(row + 4);
        const float4 q2 = *reinterpret_cast<const float4*>(row + 8);
        const float a[12] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w, q2.x, q2.y, q2.z, q2.w};
#pragma unroll
        for (int dz = -R; dz <= R; ++dz) {
            // this plane is tap plane dz of output oz = j - R - dz: slot (J - R - dz) mod K
            const int slot = ((J - R - dz) % K + K) % K;
#pragma unroll
            for (int dx = -R; dx <= R; ++dx) {
                const float wv = p.wt[((dz + R) * K + (dy + R)) * K + (dx + R)];
#pragma unroll
                for (int i = 0; i < 4; ++i) acc[slot][i] = __fmaf_rn(wv, a[i + dx + 4], acc[slot][i]);
            }
        }
    }
}

template <int R, int J>
__device__ __forceinline__ bool chunk_step(const Conv3Params<R>& p, float* sm, Stage<R>& st, float (&acc)[2 * R + 1][4],
                                           int64_t j, int64_t nsteps, int64_t zs, int64_t zlen, int64_t x0, int64_t y0,
                                           int lx, int ly) {
    constexpr int K = 2 * R + 1;
    if (j >= nsteps) return false;
    __syncthreads();              // previous plane's readers are done
    stage_store<R>(sm, st);
    __syncthreads();
    if (j + 1 < nsteps) stage_load<R>(p, st, zs - R + j + 1, x0, y0);   // next plane in flight
    compute_plane<R, J>(p, sm, acc, lx, ly);
    // output oz = j - 2R is complete (its dz = +R plane was this one)
    constexpr int done_slot = ((J - 2 * R) % K + K) % K;
    const int64_t oz = j - 2 * R;
    if (oz >= 0 && oz < zlen) store_out<R>(p, zs + oz, y0 + ly, x0 + 4 * lx, acc[done_slot]);
#pragma unroll
    for (int i = 0; i < 4; ++i) acc[done_slot][i] = 0.0f;
    return true;
}

template <int R, int... Js>
__device__ __forceinline__ void run_chunk(const Conv3Params<R>& p, float* sm, int64_t zs, int64_t ze, int64_t x0,
                                          int64_t y0, int lx, int ly) {
    constexpr int K = 2 * R + 1;
    float acc[K][4];
#pragma unroll
    for (int s = 0; s < K; ++s)
#pragma unroll
        for (int i = 0; i < 4; ++i) acc[s][i] = 0.0f;
    Stage<R> st;
    const int64_t zlen = ze - zs;
    const int64_t nsteps = zlen + 2 * R;   // input planes zs-R .. ze+R-1
    stage_load<R>(p, st, zs - R, x0, y0);
    for (int64_t j = 0; j < nsteps; j += K) {
        bool go = true;
        // unrolled K steps: J = 0..K-1 are compile-time slot phases
        ((go = go && chunk_step<R, Js>(p, sm, st, acc, j + Js, nsteps, zs, zlen, x0, y0, lx, ly)), ...);
    }
}

template <int R>
__global__ void __launch_bounds__(NT) conv3d_kernel(const __grid_constant__ Conv3Params<R> p) {
    __shared__ __align__(16) float sm[(TY + 2 * R) * SW];
    const int tile = blockIdx.x;
    const int64_t x0 = (int64_t)(tile % p.tiles_x) * TX;
    const int64_t y0 = (int64_t)(tile / p.tiles_x) * TY;
    int64_t c = blockIdx.y;
    int b = 0;
    while (b < p.nbands && c >= p.nchunks[b]) c -= p.nchunks[b++];
    if (b >= p.nbands) return;
    const int64_t zs = p.zbeg[b] + c * p.zc;
    const int64_t ze = zs + p.zc < p.zend[b] ? zs + p.zc : p.zend[b];
    const int lx = threadIdx.x % (TX / 4), ly = threadIdx.x / (TX / 4);
    if constexpr (R == 1)
        run_chunk<R, 0, 1, 2>(p, sm, zs, ze, x0, y0, lx, ly);
    else
        run_chunk<R, 0, 1, 2, 3, 4>(p, sm, zs, ze, x0, y0, lx, ly);
}

template <int R>
cudaError_t launch_t(const StencilGeom& g, const RowBands& bands, const float* weights, int num_sms, cudaStream_t s) {
    Conv3Params<R> p;
    p.in = static_cast<const float*>(g.in);
    p.out = static_cast<float*>(g.out);
    p.ppitch = g.pitch / 4;
    p.rpitch = g.rpitch / 4;
    p.planes = g.rows;
    p.h = g.plane_rows;
    p.w = g.w;
    p.tiles_x = (int)((g.w + TX - 1) / TX);
    const int64_t tiles = (int64_t)p.tiles_x * ((g.plane_rows + TY - 1) / TY);
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.mode = g.col_mode;
    constexpr int K = 2 * R + 1;
    for (int i = 0; i < K * K * K; ++i) p.wt[i] = weights[i];
    int64_t total = 0;
    for (int b = 0; b < bands.nbands; ++b) total += bands.end[b] - bands.begin[b];
    if (total <= 0 || tiles <= 0) return cudaSuccess;
    // enough CTAs to keep every SM busy (~6 resident per SM), chunks >= 2K planes
    const int64_t want = (int64_t)num_sms * 6;
    int64_t chunks = (want + tiles - 1) / tiles;
    int64_t zc = (total + chunks - 1) / chunks;
    if (zc < 2 * K) zc = 2 * K;
    p.zc = zc;
    p.nbands = bands.nbands;
    int64_t ny = 0;
    for (int b = 0; b < bands.nbands; ++b) {
        p.zbeg[b] = bands.begin[b];
        p.zend[b] = bands.end[b];
        p.nchunks[b] = bands.end[b] > bands.begin[b] ? (bands.end[b] - bands.begin[b] + zc - 1) / zc : 0;
        ny += p.nchunks[b];
    }
    if (tiles > 0x7fffffff || ny > 65535) return cudaErrorInvalidConfiguration;
    conv3d_kernel<R><<<dim3((unsigned)tiles, (unsigned)ny), NT, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_conv3d(const StencilGeom& g, const RowBands& b, int r, const float* weights, int num_sms,
                          cudaStream_t s) {
    switch (r) {
        case 1: return launch_t<1>(g, b, weights, num_sms, s);
        case 2: return launch_t<2>(g, b, weights, num_sms, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace mapsm
