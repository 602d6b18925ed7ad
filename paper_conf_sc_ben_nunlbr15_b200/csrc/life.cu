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

#include "kernels.h"

namespace mapsm {
namespace {

constexpr int kThreads = 256;
constexpr unsigned kFull = 0xffffffffu;

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

__device__ __forceinline__ int64_t map_row(const LifeParams& p, int64_t y) {
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

template <int V>
__device__ __forceinline__ void load_vec(const uint32_t* ptr, uint32_t (&x)[V]) {
    if constexpr (V == 4) {
        uint4 v = __ldg(reinterpret_cast<const uint4*>(ptr));
        x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
    } else {
        uint2 v = __ldg(reinterpret_cast<const uint2*>(ptr));
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

// Per-lane constants of the column layout.
struct LaneCols {
    int64_t vi;          // vector index of this lane within the row
    bool active;         // vi < nvec
    bool need_l, need_r; // this lane supplies its own edge word instead of a shuffle
    int64_t l_idx, r_idx;  // word index of the edge word to load, -1 = synthesise
};

template <int V>
__device__ __forceinline__ void fetch_row(const LifeParams& p, const LaneCols& c, int64_t y,
                                          Fetch<V>& f) {
    const uint32_t* row = p.in + map_row(p, y) * p.pitch_w;
    if (c.active) {
        load_vec<V>(row + c.vi * V, f.x);
    } else {
#pragma unroll
        for (int i = 0; i < V; ++i) f.x[i] = 0u;
    }
    f.le = (c.need_l && c.l_idx >= 0) ? __ldg(row + c.l_idx) : 0u;
    f.re = (c.need_r && c.r_idx >= 0) ? __ldg(row + c.r_idx) : 0u;
}

// Horizontal 3-cell sums of one row: s0 = parity, s1 = carry (L + x + R).
template <int V>
__device__ __forceinline__ void row_sums(const LifeParams& p, const LaneCols& c, const Fetch<V>& f,
                                         uint32_t (&s0)[V], uint32_t (&s1)[V]) {
    const uint32_t up = __shfl_up_sync(kFull, f.x[V - 1], 1);
    const uint32_t dn = __shfl_down_sync(kFull, f.x[0], 1);
    uint32_t lw = c.need_l ? f.le : up;
    uint32_t rw = c.need_r ? f.re : dn;
    if (c.l_idx < 0) lw = (p.col_mode == COL_CLAMP) ? (f.x[0] << 31) : 0u;
    if (c.r_idx < 0) rw = (p.col_mode == COL_CLAMP) ? (f.x[V - 1] >> 31) : 0u;
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

template <int V, int P>
__global__ void __launch_bounds__(kThreads) life_step_kernel(const __grid_constant__ LifeParams p) {
    const int lane = threadIdx.x & 31;
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

    LaneCols c;
    c.vi = strip * 32 + lane;
    c.active = c.vi < p.nvec;
    c.need_l = c.active && (lane == 0 || c.vi == 0);
    c.need_r = c.active && (lane == 31 || c.vi == p.nvec - 1);
    c.l_idx = (c.vi == 0) ? (p.col_mode == COL_WRAP ? p.nw - 1 : -1) : c.vi * V - 1;
    c.r_idx = (c.vi == p.nvec - 1) ? (p.col_mode == COL_WRAP ? 0 : -1) : (c.vi + 1) * V;
    if (!c.need_l) c.l_idx = 0;
    if (!c.need_r) c.r_idx = 0;

    // Prologue: rows ys-1 and ys, and the first P rows of the pipeline.
    Fetch<V> fa, fb;
    fetch_row<V>(p, c, ys - 1, fa);
    fetch_row<V>(p, c, ys, fb);
    Fetch<V> ring[P];
#pragma unroll
    for (int k = 0; k < P; ++k)
        if (ys + 1 + k <= ye) fetch_row<V>(p, c, ys + 1 + k, ring[k]);

    uint32_t a0[V], a1[V], b0[V], b1[V], alive[V];
    row_sums<V>(p, c, fa, a0, a1);
    row_sums<V>(p, c, fb, b0, b1);
#pragma unroll
    for (int i = 0; i < V; ++i) alive[i] = fb.x[i];

    uint32_t* out_row = p.out + ys * p.pitch_w + c.vi * V;
    for (int64_t y = ys; y < ye; y += P) {
#pragma unroll
        for (int k = 0; k < P; ++k) {
            const int64_t yy = y + k;
            if (yy < ye) {
                Fetch<V> f = ring[k];
                if (yy + 1 + P <= ye) fetch_row<V>(p, c, yy + 1 + P, ring[k]);
                uint32_t c0[V], c1[V], o[V];
                row_sums<V>(p, c, f, c0, c1);
#pragma unroll
                for (int i = 0; i < V; ++i)
                    o[i] = life_word(a0[i], a1[i], b0[i], b1[i], c0[i], c1[i], alive[i]);
                if (c.active) store_vec<V>(out_row, o);
                out_row += p.pitch_w;
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    a0[i] = b0[i]; a1[i] = b1[i];
                    b0[i] = c0[i]; b1[i] = c1[i];
                    alive[i] = f.x[i];
                }
            }
        }
    }
}

// ------------------------------------------------------------ pack / unpack
// u8 (nonzero = alive) -> bits; one thread per 32-bit word (32 bytes in).
__global__ void pack_life_kernel(const uint8_t* __restrict__ src, int64_t src_pitch,
                                 uint32_t* __restrict__ dst, int64_t dst_pitch_w, int64_t rows,
                                 int64_t nw, bool vec) {
    const int64_t wi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t y = blockIdx.y + (int64_t)blockIdx.z * gridDim.y;
    if (wi >= nw || y >= rows) return;
    const uint8_t* s = src + y * src_pitch + wi * 32;
    uint32_t word = 0;
    if (vec) {
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
        for (int j = 0; j < 32; ++j) word |= (uint32_t)(s[j] != 0) << j;
    }
    dst[y * dst_pitch_w + wi] = word;
}

// bits -> u8 0/1; one thread per 32-bit word (32 bytes out).
__global__ void unpack_life_kernel(const uint32_t* __restrict__ src, int64_t src_pitch_w,
                                   uint8_t* __restrict__ dst, int64_t dst_pitch, int64_t rows,
                                   int64_t nw, bool vec) {
    const int64_t wi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t y = blockIdx.y + (int64_t)blockIdx.z * gridDim.y;
    if (wi >= nw || y >= rows) return;
    const uint32_t word = src[y * src_pitch_w + wi];
    uint8_t* d = dst + y * dst_pitch + wi * 32;
    uint32_t v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) v[q] = (((word >> (4 * q)) & 0xFu) * 0x00204081u) & 0x01010101u;
    if (vec) {
        *reinterpret_cast<uint4*>(d) = make_uint4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<uint4*>(d + 16) = make_uint4(v[4], v[5], v[6], v[7]);
    } else {
        for (int j = 0; j < 32; ++j) d[j] = (uint8_t)((word >> j) & 1u);
    }
}

template <int V, int P>
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
                                                                      life_step_kernel<V, P>, kThreads, 0);
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
    life_step_kernel<V, P><<<grid, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_life_step(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s) {
    const int64_t nw = g.w / 32;
    if (nw % 4 == 0 && g.pitch % 16 == 0) return launch_life_t<4, 3>(g, b, num_sms, s);
    return launch_life_t<2, 3>(g, b, num_sms, s);
}

cudaError_t launch_pack_life(const uint8_t* src, int64_t src_pitch, void* dst, int64_t dst_pitch,
                             int64_t rows, int64_t w, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    const int64_t nw = w / 32;
    const bool vec = (src_pitch % 16 == 0) && ((uintptr_t)src % 16 == 0);
    const unsigned ty = (unsigned)(rows < 32768 ? rows : 32768);
    dim3 grid((unsigned)((nw + 255) / 256), ty, (unsigned)((rows + ty - 1) / ty));
    pack_life_kernel<<<grid, 256, 0, s>>>(src, src_pitch, static_cast<uint32_t*>(dst), dst_pitch / 4,
                                          rows, nw, vec);
    return cudaGetLastError();
}

cudaError_t launch_unpack_life(const void* src, int64_t src_pitch, uint8_t* dst, int64_t dst_pitch,
                               int64_t rows, int64_t w, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    const int64_t nw = w / 32;
    const bool vec = (dst_pitch % 16 == 0) && ((uintptr_t)dst % 16 == 0);
    const unsigned ty = (unsigned)(rows < 32768 ? rows : 32768);
    dim3 grid((unsigned)((nw + 255) / 256), ty, (unsigned)((rows + ty - 1) / ty));
    unpack_life_kernel<<<grid, 256, 0, s>>>(static_cast<const uint32_t*>(src), src_pitch / 4, dst,
                                            dst_pitch, rows, nw, vec);
    return cudaGetLastError();
}

}  // namespace mapsm
