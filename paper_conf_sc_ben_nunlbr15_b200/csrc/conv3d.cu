// conv3d.cu — Window(3D) fp32 convolution, radius 1..4, sm_100a (SURVEY §8(f)
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
// r-wide y/x apron is staged ONCE in shared memory by cp.async (LDGSTS) into a
// 4-deep plane ring (y/x boundary resolved by the source address, ZERO cells
// by zero-fill), and feeds the 2r+1 output planes whose accumulators are live
// in registers.
// Because planes stream in increasing z, output plane z receives its dz =
// -r..r tap planes in order — the paper's ILP over rows taken to
// the third dimension.  Each thread owns 4 consecutive x (one 128-bit store)
// of RY rows (register blocking in y: RY + 2r window rows, three 16-byte LDS
// each, serve RY x 4 outputs — without it the kernel was shared-memory bound,
// ncu: 36 wavefronts per 108 FFMA per warp and plane).
// Weights are a kernel parameter (constant bank).  No tensor cores: a stencil
// is not a dense contraction and a GEMM reshaping would not be exact.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace mapsm {
namespace {

constexpr int TX = 64;       // output columns per CTA (16 thread columns x 4 floats)
constexpr int NT = 256;      // threads per CTA: 16 x 16
constexpr int SW = TX + 8;   // smem row stride: tile column c in [-4, TX+4) lives at index c + 4
#ifndef MAPSM_C3_NBUF
#define MAPSM_C3_NBUF 4
#endif
#ifndef MAPSM_C3_RY1
#define MAPSM_C3_RY1 4
#endif
#ifndef MAPSM_C3_MINB1
#define MAPSM_C3_MINB1 2
#endif
#ifndef MAPSM_C3_RY2
#define MAPSM_C3_RY2 2
#endif
#ifndef MAPSM_C3_MINB2
#define MAPSM_C3_MINB2 2
#endif
constexpr int NBUF = MAPSM_C3_NBUF;
typedef unsigned long long Acc2;   // a pair of fp32 accumulators (see fma_pair)   // plane ring depth (NBUF - 1 planes in flight)

// rows per thread (register blocking in y) and CTAs per SM, per radius
template <int R> struct Cfg;
template <> struct Cfg<1> { static constexpr int RY = MAPSM_C3_RY1, MINB = MAPSM_C3_MINB1; };
template <> struct Cfg<2> { static constexpr int RY = MAPSM_C3_RY2, MINB = MAPSM_C3_MINB2; };
// r = 3..4 (343 / 729 FMA per cell): one output row per thread, rotating
// accumulators (one plane per loop iteration: the 2r+1-plane unroll of the
// static slots would not fit the instruction cache)
template <> struct Cfg<3> { static constexpr int RY = 1, MINB = 2; };
template <> struct Cfg<4> { static constexpr int RY = 1, MINB = 2; };

template <int R>
struct Conv3Params {
    const float* in;   // owned plane 0, row 0 of the input buffer
    float* out;
    int64_t ppitch;    // plane pitch (floats)
    int64_t rpitch;    // row pitch (floats)
    int64_t planes, h, w;
    int tiles_x;
    int64_t tiles;
    int nbands;
    int64_t zbeg[3], zend[3], zc[3];
    int64_t units;     // plane-tiles over all bands (band-major, then z-block of zc planes, then tile, then z)
    int top_map, bot_map, mode;  // plane maps (ROWMAP_*), y/x boundary (ColMode)
    float wt[(2 * R + 1) * (2 * R + 1) * (2 * R + 1)];
    // weight pairs for fma_pair, aligned so each loads as one 64-bit uniform
    // register pair: wp[((dz+R)(2R+1) + dy+R) 2R + dx+R-1] = (W[..][dx-1], W[..][dx]), dx in [1-R, R]
    float2 wp[(2 * R + 1) * (2 * R + 1) * 2 * R];
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

// Slab-local plane index an input plane Z outside [0, planes) reads (halo
// planes live at -R..-1 and planes..planes+R-1 of the buffer).  Out of line:
// the hot loop only tests the range.
__device__ __noinline__ int64_t plane_map_edge(int64_t Z, int64_t planes, int top_map, int bot_map) {
    const int m = Z < 0 ? top_map : bot_map;
    if (m == ROWMAP_WRAP) {
        int64_t q = Z % planes;
        return q < 0 ? q + planes : q;
    }
    if (m == ROWMAP_CLAMP) return Z < 0 ? 0 : planes - 1;
    return Z;  // ROWMAP_HALO
}

__device__ __forceinline__ void cp16(float* dst, const float* src, bool valid) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp4(float* dst, const float* src, bool valid) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 4 : 0) : "memory");
}
__device__ __forceinline__ int64_t plane_map(int64_t Z, int64_t planes, int top_map, int bot_map) {
    return (Z >= 0 && Z < planes) ? Z : plane_map_edge(Z, planes, top_map, bot_map);
}

__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// The tile's staging items (fixed for the CTA): in-plane source offsets of
// the thread's 16-byte interior chunks and apron floats (-1 = zero cell,
// -2 = partial vector at the right edge: per-element path).
template <int R>
struct Items {
    static constexpr int TY = 16 * Cfg<R>::RY;
    static constexpr int ROWS = TY + 2 * R;
    static constexpr int NV = ROWS * (TX / 4);
    static constexpr int NE = ROWS * 2 * R;
    static constexpr int KV = (NV + NT - 1) / NT;
    static constexpr int KE = (NE + NT - 1) / NT;
    int64_t voff[KV];
    int64_t eoff[KE];
};

template <int R>
__device__ __forceinline__ void items_init(const Conv3Params<R>& p, Items<R>& it, int64_t x0, int64_t y0) {
#pragma unroll
    for (int k = 0; k < Items<R>::KV; ++k) {
        const int idx = threadIdx.x + k * NT;
        const int row = idx / (TX / 4), vq = idx % (TX / 4);
        const int64_t y = axis_map(y0 - R + row, p.h, p.mode);
        const int64_t x = x0 + 4 * vq;
        it.voff[k] = (idx >= Items<R>::NV || y < 0) ? -1 : (x + 3 < p.w ? y * p.rpitch + x : -2);
    }
#pragma unroll
    for (int k = 0; k < Items<R>::KE; ++k) {
        const int idx = threadIdx.x + k * NT;
        const int row = idx / (2 * R), q = idx % (2 * R);
        const int c = q < R ? q - R : TX + (q - R);
        const int64_t y = axis_map(y0 - R + row, p.h, p.mode);
        const int64_t x = axis_map(x0 + c, p.w, p.mode);
        it.eoff[k] = (idx >= Items<R>::NE || y < 0 || x < 0) ? -1 : y * p.rpitch + x;
    }
}

// A 16-byte chunk that crosses the right edge of the plane (or lies past it):
// four 4-byte copies with the x boundary resolved per element.
__device__ __noinline__ void stage_partial(const float* plane, float* dst, int64_t yy, int64_t x, int64_t h, int64_t w,
                                           int64_t rpitch, int mode) {
    const int64_t y = axis_map(yy, h, mode);
    for (int i = 0; i < 4; ++i) {
        const int64_t xx = axis_map(x + i, w, mode);
        cp4(dst + i, plane + (xx >= 0 && y >= 0 ? y * rpitch + xx : 0), xx >= 0 && y >= 0);
    }
}

// Issue the cp.async copies of input plane Z's tile into buffer `sm`.
template <int R>
__device__ __forceinline__ void stage_issue(const Conv3Params<R>& p, const Items<R>& it, float* sm, int64_t Z,
                                            int64_t x0, int64_t y0) {
    const float* plane = p.in + plane_map(Z, p.planes, p.top_map, p.bot_map) * p.ppitch;
#pragma unroll
    for (int k = 0; k < Items<R>::KV; ++k) {
        const int idx = threadIdx.x + k * NT;
        if (idx < Items<R>::NV) {
            const int row = idx / (TX / 4), vq = idx % (TX / 4);
            float* dst = sm + row * SW + 4 + 4 * vq;
            const int64_t off = it.voff[k];
            if (off != -2)
                cp16(dst, plane + (off >= 0 ? off : 0), off >= 0);
            else  // right edge: per element, out of line
                stage_partial(plane, dst, y0 - R + row, x0 + 4 * vq, p.h, p.w, p.rpitch, p.mode);
        }
    }
#pragma unroll
    for (int k = 0; k < Items<R>::KE; ++k) {
        const int idx = threadIdx.x + k * NT;
        if (idx < Items<R>::NE) {
            const int row = idx / (2 * R), q = idx % (2 * R);
            const int c = q < R ? q - R : TX + (q - R);
            const int64_t off = it.eoff[k];
            cp4(sm + row * SW + 4 + c, plane + (off >= 0 ? off : 0), off >= 0);
        }
    }
}

template <int R>
__device__ __forceinline__ void store_out(const Conv3Params<R>& p, int64_t z, int64_t y, int64_t x, const Acc2* acc2) {
    if (y >= p.h || x >= p.w) return;
    const float2 p0 = *reinterpret_cast<const float2*>(&acc2[0]), p1 = *reinterpret_cast<const float2*>(&acc2[1]);
    const float a[4] = {p0.y, p0.x, p1.y, p1.x};   // (hi, lo) = (out 2j, out 2j+1)
    float* op = p.out + z * p.ppitch + y * p.rpitch + x;
    if (x + 3 < p.w) {
        *reinterpret_cast<float4*>(op) = make_float4(a[0], a[1], a[2], a[3]);
    } else {
        for (int i = 0; i < 4 && x + i < p.w; ++i) op[i] = a[i];
    }
}

// Accumulators in pairs: Acc2 of outputs (x0+2j, x0+2j+1) holds
// lo = out(x0+2j+1), hi = out(x0+2j), so that one FFMA2 with the input value
// broadcast (R.F32) and the consecutive weights (W[dx-1], W[dx]) as a
// uniform-register pair (UR.F32x2) advances both outputs by their own tap:
// out(2j) by dx, out(2j+1) by dx-1 (each half is an IEEE fma, RN-even — the
// oracle's fmaf).  The first and last value of a pair's window feed only one
// of the two outputs: a scalar FFMA on that half.  2R FFMA2 + 2 FFMA per
// pair and tap row instead of 2(2R+1) FFMA (the kernel is issue-bound, ncu:
// issue slots 72% busy, not_selected the top stall).
__device__ __forceinline__ void fma_pair(Acc2& acc, float v, const float2& wv) {
    asm("{\n\t.reg .b64 x;\n\tmov.b64 x, {%1, %1};\n\tfma.rn.f32x2 %0, x, %2, %0;\n\t}"
        : "+l"(acc)
        : "f"(v), "l"(*reinterpret_cast<const unsigned long long*>(&wv)));
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

// One input plane (chunk step j, J = j mod K compile-time): every live
// accumulator slot takes this plane's taps.  Window rows t = 0..RY+2R-1 of
// the thread (tile rows ly*RY + t) are read once each; row t is tap row
// dy = t - R - i of the thread's output row i.  For a fixed accumulator the
// taps arrive in (dy, dx) order (t increasing), planes in dz order.
// ROT: rotating accumulators, acc[R + dz] is the output plane this plane's
// tap dz goes to (static slot phases J otherwise).
template <int R, int J, bool ROT = false>
__device__ __forceinline__ void compute_plane(const Conv3Params<R>& p, const float* sm,
                                              Acc2 (&acc)[2 * R + 1][Cfg<R>::RY][2], int lx, int ly) {
    constexpr int K = 2 * R + 1;
    constexpr int RY = Cfg<R>::RY;
#pragma unroll
    for (int t = 0; t < RY + 2 * R; ++t) {
        const float* row = sm + (ly * RY + t) * SW + 4 * lx;   // index 4*lx = tile column 4*lx - 4
        const float4 q0 = *reinterpret_cast<const float4*>(row);
        const float4 q1 = *reinterpret_cast<const float4*>(row + 4);
        const float4 q2 = *reinterpret_cast<const float4*>(row + 8);
        const float a[12] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w, q2.x, q2.y, q2.z, q2.w};
#pragma unroll
        for (int i = 0; i < RY; ++i) {
            const int dy = t - R - i;
            if (dy < -R || dy > R) continue;
#pragma unroll
            for (int dz = -R; dz <= R; ++dz) {
                const int slot = ROT ? R + dz : ((J - R - dz) % K + K) % K;
                const float2* wq = p.wp + ((dz + R) * K + (dy + R)) * 2 * R + R - 1;   // wq[dx] = (W[dx-1], W[dx])
#pragma unroll
                for (int jp = 0; jp < 2; ++jp) {
                    // window values a[m], m = 4 + 2jp + dx (dx of out(2jp)); in m order
                    fma_hi(acc[slot][i][jp], wq[1 - R].x, a[4 + 2 * jp - R]);          // out(2jp) only, dx = -R
#pragma unroll
                    for (int dx = -R + 1; dx <= R; ++dx)
                        fma_pair(acc[slot][i][jp], a[4 + 2 * jp + dx], wq[dx]);
                    fma_lo(acc[slot][i][jp], wq[R].y, a[5 + 2 * jp + R]);              // out(2jp+1) only, dx' = R
                }
            }
        }
    }
}

template <int R, int J>
__device__ __forceinline__ bool chunk_step(const Conv3Params<R>& p, const Items<R>& it, float* smbase,
                                           Acc2 (&acc)[2 * R + 1][Cfg<R>::RY][2], int64_t j, int64_t nsteps,
                                           int64_t zs, int64_t zlen, int64_t x0, int64_t y0, int lx, int ly) {
    constexpr int K = 2 * R + 1;
    constexpr int RY = Cfg<R>::RY;
    constexpr int BUF = Items<R>::ROWS * SW;
    if (j >= nsteps) return false;
    __syncthreads();   // every thread finished plane j-1: its ring slot may be refilled
    if (j + NBUF - 1 < nsteps) stage_issue<R>(p, it, smbase + ((j + NBUF - 1) % NBUF) * BUF, zs - R + j + NBUF - 1, x0, y0);
    cp_commit();       // (possibly empty group: keeps the group count uniform)
    cp_wait<NBUF - 1>();   // plane j has landed (for this thread's copies)
    __syncthreads();   // ... and for everybody's
    compute_plane<R, J>(p, smbase + (j % NBUF) * BUF, acc, lx, ly);
    // output oz = j - 2R is complete (its dz = +R plane was this one)
    constexpr int done_slot = ((J - 2 * R) % K + K) % K;
    const int64_t oz = j - 2 * R;
    if (oz >= 0 && oz < zlen) {
#pragma unroll
        for (int i = 0; i < RY; ++i) store_out<R>(p, zs + oz, y0 + ly * RY + i, x0 + 4 * lx, acc[done_slot][i]);
    }
#pragma unroll
    for (int i = 0; i < RY; ++i) acc[done_slot][i][0] = acc[done_slot][i][1] = 0ull;   // +0.0f pairs
    return true;
}

template <int R, int... Js>
__device__ __forceinline__ void run_chunk(const Conv3Params<R>& p, float* smbase, int64_t zs, int64_t ze, int64_t x0,
                                          int64_t y0, int lx, int ly) {
    constexpr int K = 2 * R + 1;
    constexpr int RY = Cfg<R>::RY;
    constexpr int BUF = Items<R>::ROWS * SW;
    Acc2 acc[K][RY][2];
#pragma unroll
    for (int s = 0; s < K; ++s)
#pragma unroll
        for (int i = 0; i < RY; ++i) acc[s][i][0] = acc[s][i][1] = 0ull;
    Items<R> it;
    items_init<R>(p, it, x0, y0);
    const int64_t zlen = ze - zs;
    const int64_t nsteps = zlen + 2 * R;   // input planes zs-R .. ze+R-1
    // prologue: planes 0 .. NBUF-2 in flight
#pragma unroll
    for (int q = 0; q < NBUF - 1; ++q) {
        if (q < nsteps) stage_issue<R>(p, it, smbase + q * BUF, zs - R + q, x0, y0);
        cp_commit();
    }
    for (int64_t j = 0; j < nsteps; j += K) {
        bool go = true;
        // unrolled K steps: J = 0..K-1 are compile-time slot phases
        ((go = go && chunk_step<R, Js>(p, it, smbase, acc, j + Js, nsteps, zs, zlen, x0, y0, lx, ly)), ...);
    }
    cp_wait<0>();
}

// r >= 3: one plane per iteration; before plane j the accumulators shift
// (acc[d] <- acc[d-1], acc[0] = +0.0f starts output plane j), after it
// acc[2R] (output plane j - 2R, its dz = +R plane was this one) is complete.
template <int R>
__device__ __forceinline__ void run_chunk_rot(const Conv3Params<R>& p, float* smbase, int64_t zs, int64_t ze,
                                              int64_t x0, int64_t y0, int lx, int ly) {
    constexpr int K = 2 * R + 1;
    constexpr int RY = Cfg<R>::RY;
    constexpr int BUF = Items<R>::ROWS * SW;
    Acc2 acc[K][RY][2];
#pragma unroll
    for (int s = 0; s < K; ++s)
#pragma unroll
        for (int i = 0; i < RY; ++i) acc[s][i][0] = acc[s][i][1] = 0ull;
    Items<R> it;
    items_init<R>(p, it, x0, y0);
    const int64_t zlen = ze - zs;
    const int64_t nsteps = zlen + 2 * R;
#pragma unroll
    for (int q = 0; q < NBUF - 1; ++q) {
        if (q < nsteps) stage_issue<R>(p, it, smbase + q * BUF, zs - R + q, x0, y0);
        cp_commit();
    }
#pragma unroll 1
    for (int64_t j = 0; j < nsteps; ++j) {
        __syncthreads();
        if (j + NBUF - 1 < nsteps) stage_issue<R>(p, it, smbase + ((j + NBUF - 1) % NBUF) * BUF, zs - R + j + NBUF - 1, x0, y0);
        cp_commit();
        cp_wait<NBUF - 1>();
        __syncthreads();
#pragma unroll
        for (int d = K - 1; d > 0; --d)
#pragma unroll
            for (int i = 0; i < RY; ++i) acc[d][i][0] = acc[d - 1][i][0], acc[d][i][1] = acc[d - 1][i][1];
#pragma unroll
        for (int i = 0; i < RY; ++i) acc[0][i][0] = acc[0][i][1] = 0ull;
        compute_plane<R, 0, true>(p, smbase + (j % NBUF) * BUF, acc, lx, ly);
        const int64_t oz = j - 2 * R;
        if (oz >= 0 && oz < zlen) {
#pragma unroll
            for (int i = 0; i < RY; ++i) store_out<R>(p, zs + oz, y0 + ly * RY + i, x0 + 4 * lx, acc[K - 1][i]);
        }
    }
    cp_wait<0>();
}

template <int R>
__global__ void __launch_bounds__(NT, Cfg<R>::MINB) conv3d_kernel(const __grid_constant__ Conv3Params<R> p) {
    extern __shared__ __align__(16) float smbase[];
    constexpr int TY = Items<R>::TY;
    const int lx = threadIdx.x % (TX / 4), ly = threadIdx.x / (TX / 4);
    // Balanced split: CTA c of the (persistent, one-wave) grid owns plane-tiles
    // [c*U/P, (c+1)*U/P) and walks them as runs of consecutive planes of one
    // tile.  Units are ordered z-block-major (zc planes, ~P/tiles blocks), so
    // the CTAs running at the same time hold neighbouring tiles of the same
    // planes and the tiles' shared apron sectors hit in L2.
    const int64_t P = gridDim.x;
    int64_t u = p.units * (int64_t)blockIdx.x / P;
    const int64_t uend = p.units * ((int64_t)blockIdx.x + 1) / P;
    while (u < uend) {
        int64_t v = u;
        int b = 0;
        while (b < p.nbands && v >= p.tiles * (p.zend[b] - p.zbeg[b])) v -= p.tiles * (p.zend[b] - p.zbeg[b]), ++b;
        const int64_t nz = p.zend[b] - p.zbeg[b];
        const int64_t zb = v / (p.tiles * p.zc[b]);
        const int64_t rem = v - zb * p.tiles * p.zc[b];
        const int64_t blen = (nz - zb * p.zc[b]) < p.zc[b] ? (nz - zb * p.zc[b]) : p.zc[b];
        const int64_t tile = rem / blen, zin = rem % blen;
        const int64_t z = zb * p.zc[b] + zin;
        const int64_t len = (blen - zin) < (uend - u) ? (blen - zin) : (uend - u);
        const int64_t x0 = (tile % p.tiles_x) * TX;
        const int64_t y0 = (tile / p.tiles_x) * TY;
        const int64_t zs = p.zbeg[b] + z;
        if constexpr (R == 1)
            run_chunk<R, 0, 1, 2>(p, smbase, zs, zs + len, x0, y0, lx, ly);
        else if constexpr (R == 2)
            run_chunk<R, 0, 1, 2, 3, 4>(p, smbase, zs, zs + len, x0, y0, lx, ly);
        else
            run_chunk_rot<R>(p, smbase, zs, zs + len, x0, y0, lx, ly);
        u += len;
        __syncthreads();   // the next run refills the ring from slot 0
    }
}

template <int R>
cudaError_t launch_t(const StencilGeom& g, const RowBands& bands, const float* weights, int num_sms, cudaStream_t s) {
    constexpr int TY = Items<R>::TY;
    constexpr size_t smem = (size_t)NBUF * Items<R>::ROWS * SW * sizeof(float);
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
    p.tiles = tiles;
    p.top_map = g.top_map;
    p.bot_map = g.bot_map;
    p.mode = g.col_mode;
    constexpr int K = 2 * R + 1;
    for (int i = 0; i < K * K * K; ++i) p.wt[i] = weights[i];
    for (int zy = 0; zy < K * K; ++zy)
        for (int dx = 1 - R; dx <= R; ++dx)
            p.wp[zy * 2 * R + dx + R - 1] = make_float2(weights[zy * K + dx + R - 1], weights[zy * K + dx + R]);
    int64_t total = 0;
    for (int b = 0; b < bands.nbands; ++b) total += bands.end[b] - bands.begin[b];
    if (total <= 0 || tiles <= 0) return cudaSuccess;
    cudaError_t e = cudaFuncSetAttribute(conv3d_kernel<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;   // (per device; cheap, so set on every launch)
    // one wave of MINB CTAs per SM (persistent), each with an equal share of
    // the plane-tiles; a share ends in at most a few runs (2R halo planes each)
    p.nbands = bands.nbands;
    p.units = 0;
    for (int b = 0; b < bands.nbands; ++b) {
        p.zbeg[b] = bands.begin[b];
        p.zend[b] = bands.end[b] > bands.begin[b] ? bands.end[b] : bands.begin[b];
        p.units += tiles * (p.zend[b] - p.zbeg[b]);
    }
    // One run (a z-block of one tile) per CTA where the shape allows: the CTAs
    // of a z-block then march through the same planes in step, and the x/y
    // apron sectors a tile shares with its neighbours are read once from DRAM
    // (measured: a balanced split with runs starting at unrelated planes read
    // 1.7x the algorithmic bytes).  The grid is the largest multiple of the
    // tile count that fits in one wave, else one wave of balanced runs.
    const int64_t slots = (int64_t)num_sms * Cfg<R>::MINB;
    int64_t nzb = slots / tiles;
    int64_t ctas;
    if (nzb >= 1 && bands.nbands == 1) {
        ctas = tiles * nzb;
    } else {
        ctas = slots;
        nzb = (slots + tiles - 1) / tiles;
    }
    if (ctas > p.units) ctas = p.units;
    for (int b = 0; b < bands.nbands; ++b) {
        const int64_t nz = p.zend[b] - p.zbeg[b];
        p.zc[b] = nz > 0 ? (nz + nzb - 1) / nzb : 1;
    }
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_CONV3D;
        g.rec->ctas = ctas;
        g.rec->threads = NT;
        g.rec->smem = smem;
    }
    conv3d_kernel<R><<<(unsigned)ctas, NT, smem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_conv3d(const StencilGeom& g, const RowBands& b, int r, const float* weights, int num_sms,
                          cudaStream_t s) {
    switch (r) {
        case 1: return launch_t<1>(g, b, weights, num_sms, s);
        case 2: return launch_t<2>(g, b, weights, num_sms, s);
        case 3: return launch_t<3>(g, b, weights, num_sms, s);
        case 4: return launch_t<4>(g, b, weights, num_sms, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace mapsm
