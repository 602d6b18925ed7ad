// life_resident.cu — SMEM-resident, temporally blocked, persistent Game of
// Life for slabs that fit in the GPU's shared memory (sm_100a).
//
// Path rows a4/a5/a8 of SURVEY §8(a) for BASELINE configs[0]/[1] (64^2 and
// 8192^2 Life, 100 / 1000 generations, one slab, no exchanged halo): the
// Window(2D) -> Structured Injective Life step (B3/S23, §4, Fig 2b
// P:L172-262) iterated with double buffering, the WRAP boundary of
// P:L174 (or CLAMP / ZERO).
//
// Why a different kernel for these sizes.  A bit-packed 8192^2 generation is
// 8 MiB in + 8 MiB out — 2 µs at HBM speed and L2-resident anyway — so the
// per-generation kernels are bound by latency: a grid-wide barrier (or a
// launch) per generation and a pipeline fill per CTA (round 1: 5.8 µs per
// generation, 26% of the ALU ceiling).  148 SMs hold 148 x 227 KB = 33 MB of
// shared memory, enough for the whole double-buffered grid (8192^2: 56 KB of
// state per SM).  So:
//   * one cooperative launch, one CTA per SM; CTA b owns rows [y0_b, y0_b+R_b)
//     of the slab (the even split of P:L59 §2.1, applied to SMs) plus K halo
//     rows above and below, double-buffered in SHARED memory;
//   * K generations run between exchanges (temporal blocking, the deep-halo
//     schedule of SURVEY §8(f) NEXT-2 / DESIGN.md reading t1): generation j of
//     a pass computes rows [-K+j, R+K-j) (a trapezoid) from shared memory into
//     the other shared buffer, a CTA barrier between generations;
//   * after a pass each CTA publishes its first and last K rows into a global
//     (L2) slot, raises its pass counter (release), waits only for its two
//     neighbours' counters (acquire; no grid-wide barrier) and reads their rows
//     into its halo — the per-K-generation halo exchange of P:L461 between SMs;
//   * global memory is touched once at the start (generation 0 + halos) and
//     once at the end (generation n into the OTHER buffer).
// Row edges: WRAP wraps the CTA ring (CTA 0's up neighbour is CTA G-1); CLAMP
// and ZERO (global edge CTAs only) synthesise row -1 / row R at EVERY
// generation (CLAMP: a copy of row 0 / R-1; ZERO: 0), so the trapezoid never
// extends past a global edge and no mirror reading is needed.  Columns: as
// life.cu (WRAP = the row's other end, CLAMP = replicate, ZERO = 0).
//
// Per word and generation: 2 funnel shifts + 2 LOP3 (3-cell row sum, once per
// input row, reused by 3 output rows) + 8 LOP3 (bit-sliced rule) = 12 ALU-pipe
// operations for 32 cell-updates, plus the shared-memory load / store.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace mapsm {
namespace resident {

// measured on 8192^2 (profiles/r02_life8k_resident_variants.txt): 512
// threads x 2 words per lane, K = 8: 26.7 T cell-updates/s (1024 threads:
// 24.9 T; 256: 23.4 T; K = 4 / 6 / 12 / 16: 25.1 / 26.2 / 26.5 / 25.8 T)
#ifndef MAPSM_RES_THREADS
#define MAPSM_RES_THREADS 512
#endif
constexpr int kThreads = MAPSM_RES_THREADS;
constexpr int kWarps = kThreads / 32;
#ifndef MAPSM_RES_V
#define MAPSM_RES_V 2
#endif
constexpr int kV = MAPSM_RES_V;  // 32-bit words per lane per row
constexpr int kMaxSmem = 227 * 1024;
#ifndef MAPSM_RES_KMAX
#define MAPSM_RES_KMAX 8
#endif
constexpr int kMaxK = MAPSM_RES_KMAX;  // generations per exchange (largest that fits)

struct Params {
    const uint32_t* in;   // owned row 0 of generation 0 (global)
    uint32_t* out;        // owned row 0 of the buffer that receives generation n
    int64_t pitch_w;      // global row pitch in words
    int rows;             // slab rows H
    int nw;               // words per row (w / 32, a multiple of kV)
    int K;                // halo depth = generations per pass
    int64_t n;            // generations
    int col_mode;         // ColMode
    int row_wrap;         // 1: rows wrap (torus); 0: global edges (CLAMP / ZERO by col_mode)
    int row_clamp;        // global edges replicate (CLAMP) instead of zero
    int rmax;             // max rows per CTA (H / G rounded up)
    uint32_t* xbuf;       // exchange slots [G][2 parity][2 side][K][nw]
    unsigned int* flags;  // [G] passes published (zeroed before the launch)
};

__device__ __forceinline__ uint32_t maj3(uint32_t a, uint32_t b, uint32_t c) { return (a & b) | (a & c) | (b & c); }

// B3/S23 on the bit-sliced 3-row sums (see life.cu: life_word).
__device__ __forceinline__ uint32_t rule(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1, uint32_t c0, uint32_t c1,
                                         uint32_t alive) {
    const uint32_t s0 = a0 ^ b0 ^ c0;
    const uint32_t k = maj3(a0, b0, c0);
    const uint32_t t = a1 ^ b1 ^ c1;
    const uint32_t u = maj3(a1, b1, c1);
    const uint32_t C = u ^ (k | t);
    const uint32_t D = ~(s0 ^ k ^ t) & (s0 | alive);
    return C & D;
}

__device__ __forceinline__ unsigned int ld_acquire_gpu(const unsigned int* p) {
    unsigned int v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// One lane's columns: words [w0, w0+V) of a row.  The words holding its left
// and right neighbour bits are read straight from shared memory by every
// lane (no shuffles, no divergent edge handling): l_idx / r_idx are valid
// word indices; at CLAMP / ZERO row ends the word is turned into the
// replicated / zero neighbour by a shift / mask (compiled out under WRAP).
struct Lane {
    int w0;              // first word (0 for an inactive lane: reads, never stores)
    bool active;
    int l_idx, r_idx;
    int lsh, rsh;        // CLAMP row ends: 31 (the edge bit of the lane's own edge word)
    uint32_t lmask, rmask;  // ZERO row ends: 0
};

template <int CM>
__device__ __forceinline__ void row_sums(const Lane& c, const uint32_t* row, uint32_t (&x)[kV], uint32_t (&s0)[kV],
                                         uint32_t (&s1)[kV]) {
    if constexpr (kV == 4) {
        const uint4 v = *reinterpret_cast<const uint4*>(row + c.w0);
        x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
    } else if constexpr (kV == 2) {
        const uint2 v = *reinterpret_cast<const uint2*>(row + c.w0);
        x[0] = v.x; x[1] = v.y;
    } else {
        x[0] = row[c.w0];
    }
    uint32_t lw = row[c.l_idx], rw = row[c.r_idx];
    if constexpr (CM != COL_WRAP) {
        lw = (lw << c.lsh) & c.lmask;
        rw = (rw >> c.rsh) & c.rmask;
    }
#pragma unroll
    for (int i = 0; i < kV; ++i) {
        const uint32_t ls = (i == 0) ? lw : x[i - 1];
        const uint32_t rs = (i == kV - 1) ? rw : x[i + 1];
        const uint32_t L = __funnelshift_l(ls, x[i], 1);  // bit j <- column j-1
        const uint32_t R = __funnelshift_r(x[i], rs, 1);  // bit j <- column j+1
        s0[i] = L ^ x[i] ^ R;
        s1[i] = maj3(L, x[i], R);
    }
}

// One warp, one generation: output rows [ys, ye) (local; inside the trapezoid
// they may be negative or >= R) of `dst` from `src`.  Input rows ys-1 .. ye
// are all real shared-memory rows: at a global CLAMP / ZERO edge, rows -1 and
// R hold the replicated / zero row (CLAMP: every output of row 0 / R-1 is also
// stored there).  Three row slots rotate statically (unroll by 3).
template <int CM>
__device__ __forceinline__ void warp_gen(const Lane& c, const uint32_t* src, uint32_t* dst, int nw, int ys, int ye,
                                         int R, bool top_clamp, bool bot_clamp) {
    uint32_t xs[3][kV], h0[3][kV], h1[3][kV];
    row_sums<CM>(c, src + (ys - 1) * nw, xs[0], h0[0], h1[0]);
    row_sums<CM>(c, src + ys * nw, xs[1], h0[1], h1[1]);
    const uint32_t* ip = src + (ys + 1) * nw;
    uint32_t* o = dst + ys * nw + c.w0;
    auto emit = [&](int k, int y) {
        // rows y-1, y, y+1 in slots k%3, (k+1)%3, (k+2)%3 (k static)
        const int A = k % 3, B = (k + 1) % 3, C = (k + 2) % 3;
        uint32_t r[kV];
#pragma unroll
        for (int i = 0; i < kV; ++i) r[i] = rule(h0[A][i], h1[A][i], h0[B][i], h1[B][i], h0[C][i], h1[C][i], xs[B][i]);
        if (c.active) {
            if constexpr (kV == 4) *reinterpret_cast<uint4*>(o) = make_uint4(r[0], r[1], r[2], r[3]);
            else if constexpr (kV == 2) *reinterpret_cast<uint2*>(o) = make_uint2(r[0], r[1]);
            else *o = r[0];
            if constexpr (CM == COL_CLAMP) {
                // (a one-row slab is both edges: row -1 AND row 1 get the copy)
                auto put = [&](uint32_t* e) {
                    if constexpr (kV == 4) *reinterpret_cast<uint4*>(e) = make_uint4(r[0], r[1], r[2], r[3]);
                    else if constexpr (kV == 2) *reinterpret_cast<uint2*>(e) = make_uint2(r[0], r[1]);
                    else *e = r[0];
                };
                if (top_clamp && y == 0) put(o - nw);
                if (bot_clamp && y == R - 1) put(o + nw);
            }
        }
        o += nw;
    };
    int y = ys;
    for (; y + 3 <= ye; y += 3) {
        row_sums<CM>(c, ip, xs[2], h0[2], h1[2]);
        emit(0, y);
        row_sums<CM>(c, ip + nw, xs[0], h0[0], h1[0]);
        emit(1, y + 1);
        row_sums<CM>(c, ip + 2 * nw, xs[1], h0[1], h1[1]);
        emit(2, y + 2);
        ip += 3 * nw;
    }
    if (y < ye) {
        row_sums<CM>(c, ip, xs[2], h0[2], h1[2]);
        emit(0, y);
        if (y + 1 < ye) {
            row_sums<CM>(c, ip + nw, xs[0], h0[0], h1[0]);
            emit(1, y + 1);
        }
    }
}

template <int CM>
__global__ void __launch_bounds__(kThreads, 1) life_resident_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(16) uint32_t sm[];
    const int G = gridDim.x, b = blockIdx.x;
    const int base = p.rows / G, extra = p.rows % G;
    const int R = base + (b < extra ? 1 : 0);
    const int y0 = b * base + (b < extra ? b : extra);
    const int K = p.K, nw = p.nw;
    const int S = (p.rmax + 2 * K) * nw;  // words per shared buffer (row -K at index 0)
    uint32_t* bcur = sm;      // generation t (row -K at index 0)
    uint32_t* bnxt = sm + S;  // generation t+1
    const bool top_edge = !p.row_wrap && b == 0;
    const bool bot_edge = !p.row_wrap && b == G - 1;
    const int up = (b - 1 + G) % G, down = (b + 1) % G;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // lane geometry: column chunk cx of 32 * kV words, row group rg.  Rows
    // wider than kWarps chunks (w > kWarps * 32 * kV * 32 cells = 32768 at
    // 512 threads) give every warp the chunks cx, cx + kWarps, ... of all rows.
    const int nvec = nw / kV;
    const int ncx = (nvec + 31) / 32;
    const int ngr = kWarps / ncx > 0 ? kWarps / ncx : 1;
    const int cx = warp % ncx, rg = warp / ncx;
    const int cstep = ncx > kWarps ? kWarps : ncx;  // (cx < ncx: one chunk when ncx <= kWarps)
    const bool has_work = warp < ncx * ngr;
    auto lane_of = [&](int cxi) {
        Lane c;
        const int vi = cxi * 32 + lane;
        c.active = vi < nvec;
        c.w0 = c.active ? vi * kV : 0;
        const bool first = c.w0 == 0, last = c.w0 + kV == nw;
        c.l_idx = first ? (CM == COL_WRAP ? nw - 1 : 0) : c.w0 - 1;
        c.r_idx = last ? (CM == COL_WRAP ? 0 : nw - 1) : c.w0 + kV;
        c.lsh = (CM == COL_CLAMP && first) ? 31 : 0;
        c.rsh = (CM == COL_CLAMP && last) ? 31 : 0;
        c.lmask = (CM == COL_ZERO && first) ? 0u : ~0u;
        c.rmask = (CM == COL_ZERO && last) ? 0u : ~0u;
        return c;
    };

    // generation 0: rows [-K, R+K) on the torus; at a CLAMP / ZERO global edge
    // rows [-1, R+1) with row -1 / R the replicated / zero row (both buffers
    // for ZERO: the trapezoid never writes them)
    {
        const bool clamp = p.row_clamp;
        const int lo = top_edge ? -1 : -K, hi = bot_edge ? R + 1 : R + K;
        const int q = nw / 4;  // uint4 per row
        for (int i = threadIdx.x; i < (hi - lo) * q; i += kThreads) {
            const int y = lo + i / q;
            uint4 v = make_uint4(0u, 0u, 0u, 0u);
            const bool edge_row = (top_edge && y < 0) || (bot_edge && y >= R);
            if (!edge_row || clamp) {
                int gy = y0 + (edge_row ? (y < 0 ? 0 : R - 1) : y);
                gy %= p.rows;
                if (gy < 0) gy += p.rows;
                v = __ldg(reinterpret_cast<const uint4*>(p.in + (int64_t)gy * p.pitch_w) + i % q);
            }
            reinterpret_cast<uint4*>(bcur + (y + K) * nw)[i % q] = v;
            if (edge_row && !clamp) reinterpret_cast<uint4*>(bnxt + (y + K) * nw)[i % q] = v;
        }
    }
    __syncthreads();

    // Rows [a, e) of one generation split over the row groups; two bands
    // [a0, a1) and [b0, b1) split over the two halves of the row groups.
    auto rows_split = [&](int a, int e, int g0, int ng) {
        const int nr = e - a;
        const int rr = rg - g0;
        if (!has_work || nr <= 0 || rr < 0 || rr >= ng) return;
        const int ys = a + rr * nr / ng, ye = a + (rr + 1) * nr / ng;
        if (ys < ye)
            for (int cxi = cx; cxi < ncx; cxi += cstep)
                warp_gen<CM>(lane_of(cxi), bcur + K * nw, bnxt + K * nw, nw, ys, ye, R, top_edge, bot_edge);
    };
    auto two_bands = [&](int a0, int a1, int b0, int b1) {
        if (ngr >= 2) {
            rows_split(a0, a1, 0, ngr / 2);
            rows_split(b0, b1, ngr / 2, ngr - ngr / 2);
        } else {
            rows_split(a0, a1, 0, 1);
            rows_split(b0, b1, 0, 1);
        }
    };
    const size_t side = (size_t)K * nw, slot = 2 * side;
    // ---- halo exchange with the two neighbour CTAs, through L2.
    // publish(q): my first / last K rows of the current generation into my
    // slot of parity q, then my pass counter := q + 1 (release; no wait).
    auto publish = [&](unsigned int q) {
        const uint32_t* mine = bcur + K * nw;  // owned row 0
        uint32_t* my = p.xbuf + ((size_t)b * 2 + (q & 1)) * slot;
        const int nq = (int)(side / 4);
        for (int i = threadIdx.x; i < 2 * nq; i += kThreads) {
            const int sd = i / nq, k = i % nq;
            const uint4 v = reinterpret_cast<const uint4*>(mine + (sd == 0 ? 0 : (R - K) * nw))[k];
            __stcg(reinterpret_cast<uint4*>(my + sd * side) + k, v);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(p.flags + b) : "memory");
        }
    };
    // receive(q): wait for both neighbours' pass q (acquire), then read their
    // rows into my halo rows [-K, 0) and [R, R+K) of the current buffer.
    auto receive = [&](unsigned int q) {
        if (threadIdx.x == 0) {
            const unsigned int target = q + 1;
            if (!top_edge)
                while ((int)(ld_acquire_gpu(p.flags + up) - target) < 0) __nanosleep(32);
            if (!bot_edge)
                while ((int)(ld_acquire_gpu(p.flags + down) - target) < 0) __nanosleep(32);
            __threadfence();
        }
        __syncthreads();
        uint32_t* hrow = bcur;  // row -K
        const uint32_t* su = p.xbuf + ((size_t)up * 2 + (q & 1)) * slot + side;  // up's last K rows
        const uint32_t* sd = p.xbuf + ((size_t)down * 2 + (q & 1)) * slot;      // down's first K rows
        const int nq = (int)(side / 4);
        for (int i = threadIdx.x; i < 2 * nq; i += kThreads) {
            const int sdx = i / nq, k = i % nq;
            if (sdx == 0 && top_edge) continue;
            if (sdx == 1 && bot_edge) continue;
            const uint4 v = __ldcg(reinterpret_cast<const uint4*>(sdx == 0 ? su : sd) + k);
            reinterpret_cast<uint4*>(hrow + (sdx == 0 ? 0 : (R + K) * nw))[k] = v;
        }
        __syncthreads();
    };

    // A pass publishes its last generation's edge rows and goes on: the
    // next pass's first generation computes the rows that need no halo
    // ([1, R-1), from the owned rows only) while the neighbours' rows are in
    // flight, then receives them and computes the edge rows of the
    // trapezoid — the exchange overlaps a generation of compute.
    unsigned int pass = 0;
    bool pending = false;  // the current buffer's halos are still to be received (pass - 1)
    for (int64_t done = 0; done < p.n;) {
        const int kk = (p.n - done < K) ? (int)(p.n - done) : K;
        for (int j = 1; j <= kk; ++j) {
            const int lo = top_edge ? 0 : -kk + j;
            const int hi = bot_edge ? R : R + kk - j;
            if (pending && R >= 3) {
                rows_split(1, R - 1, 0, ngr);
                receive(pass - 1);
                two_bands(lo, 1, R - 1, hi);
                pending = false;
            } else {
                if (pending) {
                    receive(pass - 1);
                    pending = false;
                }
                rows_split(lo, hi, 0, ngr);
            }
            __syncthreads();
            uint32_t* t = bcur;
            bcur = bnxt;
            bnxt = t;
        }
        done += kk;
        if (done >= p.n) break;
        publish(pass);
        pending = true;
        ++pass;
    }
    // generation n -> global (owned rows)
    {
        const int q = nw / 4;
        const uint4* src = reinterpret_cast<const uint4*>(bcur + K * nw);
        for (int i = threadIdx.x; i < R * q; i += kThreads) {
            const int y = i / q;
            reinterpret_cast<uint4*>(p.out + (int64_t)(y0 + y) * p.pitch_w)[i % q] = src[i];
        }
    }
}

}  // namespace resident

// Host: can the slab run resident (and with which CTA count / K)?
bool life_resident_plan(int64_t w, int64_t rows, int num_sms, int* ctas, int* K, int* smem) {
    using namespace resident;
    if (w % 128 != 0 || rows < 1) return false;
    const int64_t nw = w / 32;
    if (nw % kV) return false;
    // one CTA per SM with enough rows per CTA for the halo to come from the
    // direct neighbours; at least ~1K words of state per CTA
    for (int k : {16, 12, 8, 6, 4, 3, 2, 1}) {
        if (k > kMaxK) continue;
        int64_t G = (rows * nw + 1023) / 1024;
        if (G > num_sms) G = num_sms;
        if (G > rows / k) G = rows / k;
        if (G < 1) continue;
        const int64_t rmax = (rows + G - 1) / G;
        const int64_t bytes = 2 * (rmax + 2 * k) * nw * 4;
        if (bytes > kMaxSmem) continue;
        *ctas = (int)G;
        *K = k;
        *smem = (int)bytes;
        return true;
    }
    return false;
}

int64_t life_resident_xbuf_bytes(int64_t w, int ctas, int K) { return (int64_t)ctas * 4 * K * (w / 32) * 4; }

cudaError_t launch_life_resident(const StencilGeom& g, int64_t n, int ctas, int K, int smem, uint32_t* xbuf,
                                 unsigned int* flags, cudaStream_t s) {
    using namespace resident;
    if (n <= 0) return cudaSuccess;
    Params p;
    p.in = static_cast<const uint32_t*>(g.in);
    p.out = static_cast<uint32_t*>(g.out);
    p.pitch_w = g.pitch / 4;
    p.rows = (int)g.rows;
    p.nw = (int)(g.w / 32);
    p.K = K;
    p.n = n;
    p.col_mode = g.col_mode;
    p.row_wrap = g.top_map == ROWMAP_WRAP;
    p.row_clamp = g.top_map == ROWMAP_CLAMP;
    p.rmax = (int)((g.rows + ctas - 1) / ctas);
    p.xbuf = xbuf;
    p.flags = flags;
    const void* fn;
    switch (g.col_mode) {
        case COL_WRAP: fn = (const void*)life_resident_kernel<COL_WRAP>; break;
        case COL_CLAMP: fn = (const void*)life_resident_kernel<COL_CLAMP>; break;
        default: fn = (const void*)life_resident_kernel<COL_ZERO>; break;
    }
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmem);
    if (e != cudaSuccess) return e;
    e = cudaMemsetAsync(flags, 0, sizeof(unsigned int) * ctas, s);
    if (e != cudaSuccess) return e;
    if (g.rec) {
        *g.rec = LaunchRec();
        g.rec->kernel = LK_LIFE_TB_PERSIST;
        g.rec->ctas = ctas;
        g.rec->threads = kThreads;
        g.rec->smem = smem;
        g.rec->gens = (int)(n < (1 << 30) ? n : (1 << 30));
        g.rec->rows_per_stage = K;  // generations per exchange
    }
    void* args[] = {(void*)&p};
    return cudaLaunchCooperativeKernel(fn, dim3((unsigned)ctas), dim3(kThreads), args, (size_t)smem, s);
}

}  // namespace mapsm
