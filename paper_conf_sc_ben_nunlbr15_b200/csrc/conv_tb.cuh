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
// Layout.  A CTA (1024 threads) = NW level-1 warps + NW level-2 warps + 1
// ghost warp + 1 producer warp.  The producer streams the input rows
// [ys-2r, ye+2r) of the CTA's (strip, rows) segments through an NS-stage TMA
// ring whose stages carry 8-float margins.  Level-1 lane t owns the vector
// (4 columns) t of the strip; the ghost warp's lanes 0 / 1 compute the
// level-1 vectors just left / right of the strip (columns [-4, 0) / [S, S+4)).
// Per input row, level 1 advances 2r+1 accumulator rows (register-renamed by
// the row phase: no accumulator moves) with one FFMA2 per tap and pair of
// outputs, and writes its completed generation-t+1 row into a D-row shared
// ring.  The level-2 warps consume that ring the same way (lane t: vector t)
// and store generation t+2.  The two levels synchronise per ring row with
// mbarriers only (full: written by every level-1 warp; empty: released by
// every level-2 warp), so neither waits for the other in lock-step, each warp
// holds ONE set of accumulators, and the 32 warps spread the FFMA2 work evenly
// over the 4 SM sub-partitions (the ghost warp sits on the one with a level-1
// warp less).
//
// Boundaries.  Columns: level 1 synthesises inputs outside the grid (CLAMP:
// the edge column, ZERO: 0; WRAP: the producer copies the row's other end
// into the margin); level 2 synthesises generation t+1 values outside the
// grid the same way (CLAMP: the edge column of generation t+1, ZERO: 0),
// while under WRAP the ghost / neighbour lanes computed them from wrapped
// inputs.  Rows: exchanged halos and one-slab WRAP give real generation t+1
// rows outside the slab; at a global CLAMP edge level 2 consumes the
// generation t+1 edge row in place of the r rows outside (r+1 times), at a
// ZERO edge it consumes r zero rows (the oracle's fmaf(w, 0, acc) terms).
#include <utility>

#include "conv_impl.cuh"

namespace mapsm {
namespace conv_detail {

// Weight loads of the two-generation kernel: plain (not volatile) constant
// loads at uniform addresses, so ptxas keeps the 5x5 pairs in uniform
// registers across input rows instead of re-issuing an LDCU per tap and row
// (static LDCU 3746 -> 1171; 934 -> 1008 G cell-updates/s on 16384^2,
// profiles/r02_conv5_tb2_variants.txt).
__device__ __forceinline__ unsigned long long ldc_pair_u(unsigned long long a) {
    unsigned long long r;
    asm("ld.const.b64 %0, [%1];" : "=l"(r) : "l"(a));
    return r;
}
__device__ __forceinline__ float ldc_one_u(unsigned long long a) {
    float r;
    asm("ld.const.f32 %0, [%1];" : "=f"(r) : "l"(a));
    return r;
}

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

// Weight pairs of the two-generation kernel: c_tb_wq[slot][d*2R + s-1] =
// (lo: W[d][s], hi: W[d][s-1]), s = 1..2R.  A lane's 4 outputs form two pairs
// (out c, out c+1) in one 64-bit accumulator, LOW half = the even column c,
// so a completed row is stored with one 16-byte store.  Input value x of
// column c-R+s (s = 0..2R+1) feeds out c with tap s (s <= 2R) and out c+1
// with tap s-1 (s >= 1): one fma.rn.f32x2 with x broadcast and the pair from
// a uniform register for s = 1..2R, one scalar fma on a half for s = 0 /
// 2R+1 (the conv_impl.cuh scheme with the halves swapped).  Each half is an
// IEEE fma (RN-even) and each output takes its taps in increasing (d, s) —
// the oracle's fmaf chain (reading c11).
constexpr int kTbMaxPairs = 5 * 4;
static __constant__ float2 c_tb_wq[kConvWeightSlots][kTbMaxPairs];

template <int R>
cudaError_t tb2_upload_weights(int slot, const float* weights) {
    constexpr int K = 2 * R + 1;
    static_assert(K * (K - 1) <= kTbMaxPairs, "weight slot too small");
    if (slot < 0 || slot >= kConvWeightSlots) return cudaErrorInvalidValue;
    float2 wq[K * (K - 1)];
    for (int d = 0; d < K; ++d)
        for (int s = 1; s < K; ++s) wq[d * (K - 1) + s - 1] = make_float2(weights[d * K + s], weights[d * K + s - 1]);
    return cudaMemcpyToSymbol(c_tb_wq, wq, sizeof wq, sizeof(float2) * kTbMaxPairs * slot);
}

// The 2R+4 floats of columns [c0-R, c0+4+R) of a row (`base` = the row's
// strip column 0): the inputs of the 4-column vector at strip column c0.
template <int R>
__device__ __forceinline__ void window(const float* base, int c0, float (&b)[2 * R + 4]) {
    static_assert(R == 1 || R == 2, "two-generation kernel: R = 1, 2");
    const float4 q = *reinterpret_cast<const float4*>(base + c0);
    b[R] = q.x; b[R + 1] = q.y; b[R + 2] = q.z; b[R + 3] = q.w;
    if (R == 2) {
        const float2 l = *reinterpret_cast<const float2*>(base + c0 - 2);
        const float2 h = *reinterpret_cast<const float2*>(base + c0 + 4);
        b[0] = l.x; b[1] = l.y; b[R + 4] = h.x; b[R + 5] = h.y;
    } else {
        b[0] = base[c0 - 1];
        b[R + 4] = base[c0 + 4];
    }
}

__device__ __forceinline__ void vfma_pair(Acc2& acc, float v, unsigned long long wv) {
    asm volatile("{\n\t.reg .b64 x;\n\tmov.b64 x, {%1, %1};\n\tfma.rn.f32x2 %0, x, %2, %0;\n\t}" : "+l"(acc) : "f"(v), "l"(wv));
}
__device__ __forceinline__ void vfma_lo(Acc2& acc, float w, float v) {
    asm volatile("{\n\t.reg .f32 l, h;\n\tmov.b64 {l, h}, %0;\n\tfma.rn.f32 l, %1, %2, l;\n\tmov.b64 %0, {l, h};\n\t}" : "+l"(acc) : "f"(w), "f"(v));
}
__device__ __forceinline__ void vfma_hi(Acc2& acc, float w, float v) {
    asm volatile("{\n\t.reg .f32 l, h;\n\tmov.b64 {l, h}, %0;\n\tfma.rn.f32 h, %1, %2, h;\n\tmov.b64 %0, {l, h};\n\t}" : "+l"(acc) : "f"(w), "f"(v));
}

// One input row's taps into the 2R+1 accumulator rows of a lane's 4 outputs,
// register-renamed by the row phase PH (no accumulator moves): the
// accumulator of output row o is acc[o mod K]; input row Y feeds output row
// Y+R-d with tap row d, so acc[(PH+R) mod K] starts (d = 0) and
// acc[(PH-R) mod K] completes (d = 2R) with this row.
template <int R, int PH>
__device__ __forceinline__ void taps_ph(Acc2 (&acc)[2 * R + 1][2], const float (&b)[2 * R + 4],
                                        unsigned long long cwq, unsigned long long cw) {
    constexpr int K = 2 * R + 1;
    constexpr int NEW = (PH + R) % K;
    acc[NEW][0] = acc[NEW][1] = 0ull;  // (+0.0f, +0.0f): the oracle's acc = 0
#pragma unroll
    for (int d = 0; d < K; ++d) {
        const int ph = (PH + R - d + K) % K;
#pragma unroll
        for (int s = 0; s <= K; ++s) {
            if (s == 0 || s == K) {
                const float wv = ldc_one_u(cw + 4 * (d * K + (s == 0 ? 0 : K - 1)));
#pragma unroll
                for (int jp = 0; jp < 2; ++jp) {
                    if (s == 0) vfma_lo(acc[ph][jp], wv, b[2 * jp + s]);
                    else vfma_hi(acc[ph][jp], wv, b[2 * jp + s]);
                }
            } else {
                const unsigned long long wq = ldc_pair_u(cwq + 8 * (d * (K - 1) + s - 1));
#pragma unroll
                for (int jp = 0; jp < 2; ++jp) vfma_pair(acc[ph][jp], b[2 * jp + s], wq);
            }
        }
    }
}

template <int I>
using ic = std::integral_constant<int, I>;

template <typename F, int... Is>
__device__ __forceinline__ void unroll_seq(F& f, int j0, std::integer_sequence<int, Is...>) {
    (f(ic<Is>(), j0 + Is), ...);
}

__device__ __forceinline__ void st_shared_pairs(float* dst, Acc2 a, Acc2 b) {
    asm volatile("st.shared.v2.b64 [%0], {%1, %2};" ::"r"(tma::smem_u32(dst)), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void st_shared_f4(float* dst, float v) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %1, %1, %1};" ::"r"(tma::smem_u32(dst)), "f"(v) : "memory");
}
__device__ __forceinline__ void st_global_pairs(float* dst, Acc2 a, Acc2 b) {
    asm volatile("st.global.v2.b64 [%0], {%1, %2};" ::"l"(dst), "l"(a), "l"(b) : "memory");
}

// ---- shared-memory access by 32-bit shared addresses (the whole layout is
// compile-time offsets from one base, so per-step addresses are immediates)
__device__ __forceinline__ void mbar_wait_s(uint32_t bar, uint32_t parity) {
    // suspends the warp in hardware (up to the hint, ns) instead of re-polling:
    // the waits of a pipeline stage that runs ahead would otherwise spend
    // issue slots of their SM sub-partition
    uint32_t done = 0;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(bar), "r"(parity), "r"(0x989680)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void mbar_arrive_s(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ bool elect_one() {
    uint32_t pred;
    asm volatile("{\n\t.reg .pred p;\n\telect.sync _|p, 0xffffffff;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(pred));
    return pred != 0;
}
// every lane's shared stores / loads of this step are done, then one lane arrives
__device__ __forceinline__ void warp_arrive(uint32_t bar) {
    __syncwarp();
    if (elect_one()) mbar_arrive_s(bar);
}

// The 2R+4 floats of columns [c0-R, c0+4+R) of a row at shared address `a`
// (= the row's column c0): the inputs of the 4-column vector at c0.
template <int R>
__device__ __forceinline__ void window_s(uint32_t a, float (&b)[2 * R + 4]) {
    static_assert(R == 1 || R == 2, "two-generation kernel: R = 1, 2");
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                 : "=f"(b[R]), "=f"(b[R + 1]), "=f"(b[R + 2]), "=f"(b[R + 3])
                 : "r"(a)
                 : "memory");
    if (R == 2) {
        asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(b[0]), "=f"(b[1]) : "r"(a - 8) : "memory");
        asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(b[R + 4]), "=f"(b[R + 5]) : "r"(a + 16) : "memory");
    } else {
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(b[0]) : "r"(a - 4) : "memory");
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(b[R + 4]) : "r"(a + 16) : "memory");
    }
}
__device__ __forceinline__ void st_shared_pairs_s(uint32_t a, Acc2 x, Acc2 y) {
    asm volatile("st.shared.v2.b64 [%0], {%1, %2};" ::"r"(a), "l"(x), "l"(y) : "memory");
}
__device__ __forceinline__ void st_shared_f4_s(uint32_t a, float v) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %1, %1, %1};" ::"r"(a), "f"(v) : "memory");
}

// level-1 (= level-2) warps: 2 * 13 + ghost + producer = 28 warps.  Not a
// free knob: builds with 10, 12 or 14 hung on the 16384^2 bench grid
// (round 2), so any change needs the ring's arrival counts re-derived.
constexpr int kTbWarps = 13;
constexpr int kTbL1Margin = 8;

// Ring bookkeeping.  Both rings (the TMA input ring and the generation-t+1
// ring) have 2K slots, K = 2R+1, and are indexed by the segment's input-row
// step j: step j uses slot j mod 2K of both.  Every segment is padded to a
// multiple of 2K steps (the padding steps move no data but keep every slot's
// mbarrier phases in step), so a group of K steps j0 .. j0+K-1 uses slots
// h*K + J (h = the group's half, J = 0..K-1 a compile-time offset) and
// accumulator phase J: nothing is recomputed per step.  Step j:
//   level 1: input row ys - 2R + j (j < n_in) into the accumulators; for
//     2R <= j < n_in the completed generation-t+1 row ys - 3R + j goes to the
//     ring slot (after its previous occupant was released).
//   level 2: for 2R <= j < n_in, feed k = j - 2R: that same row (or, past a
//     global CLAMP edge, the edge row; past a ZERO edge, a zero row); for
//     j >= 4R the output row ys - 4R + j completes.  Level 2 waits for every
//     slot occupant (data or padding) before releasing it, so a slot's full
//     and empty phases alternate strictly.  The bottom CLAMP edge row, which
//     the last R feeds read again, is released after the last feed.
// Deadlock-free: a level-1 write waits only for the release of the occupant
// 2K steps earlier, and level 2 never waits for a row more than R steps
// ahead of its own.
template <int R, int NW>
struct TbLayout {
    static constexpr int K = 2 * R + 1, NS = 2 * K, S = NW * 128;
    static constexpr int SB = (S + 2 * kTbMargin) * 4;  // TMA stage bytes: [8 | S | 8] floats
    static constexpr int L1B = (S + 2 * kTbL1Margin) * 4;  // generation-t+1 row bytes: [8 | S | 8]
    static constexpr int OFF_L1 = NS * SB;
    static constexpr int OFF_ZERO = OFF_L1 + NS * L1B;
    static constexpr int OFF_FULL = OFF_ZERO + L1B;
    static constexpr int OFF_EMPTY = OFF_FULL + 8 * NS;
    static constexpr int OFF_L1FULL = OFF_EMPTY + 8 * NS;
    static constexpr int OFF_L1EMPTY = OFF_L1FULL + 8 * NS;
    static constexpr int BYTES = OFF_L1EMPTY + 8 * NS;
};

// Producer: the segment's n_in input rows, then empty rounds up to P steps.
template <int NS>
__device__ __forceinline__ void tb2_produce_seg(const tma::RowStream& p, const tma::Seg& t, uint8_t* smem,
                                                int stage_bytes, uint64_t* full, uint64_t* empty, int64_t y_first,
                                                int n_in, int P, tma::RingPos& r, bool wrap_cols) {
    tb2_produce<NS>(p, t, smem, stage_bytes, full, empty, y_first, n_in, r, wrap_cols);
    for (int j = n_in; j < P; ++j) {
        if (r.count >= NS) mbar_wait_s(tma::smem_u32(&empty[r.stage]), r.phase ^ 1u);
        tma::mbar_arrive(&full[r.stage]);
        r.advance(NS);
    }
}

template <int K, typename F>
__device__ __forceinline__ void group_steps(F&& f) {
    unroll_seq(f, 0, std::make_integer_sequence<int, K>());
}

template <int R, int NW, int NS_, int CM>
__global__ void __launch_bounds__((2 * NW + 2) * 32, 1) conv_tb2_kernel(const __grid_constant__ ConvTb2Params pp) {
    using Ly = TbLayout<R, NW>;
    constexpr int K = Ly::K, NS = Ly::NS, S = Ly::S;
    static_assert(NS_ == NS, "ring size");
    const tma::RowStream& p = pp.s;
    extern __shared__ __align__(128) uint8_t smem[];
    const uint32_t sb = tma::smem_u32(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + Ly::OFF_FULL);
    uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Ly::OFF_EMPTY);
    for (int i = threadIdx.x; i < Ly::L1B / 4; i += blockDim.x)
        reinterpret_cast<float*>(smem + Ly::OFF_ZERO)[i] = 0.f;
    if (threadIdx.x == 0)
        for (int s = 0; s < NS; ++s) {
            tma::mbar_init(reinterpret_cast<uint64_t*>(smem + Ly::OFF_L1FULL) + s, NW + 1);
            tma::mbar_init(reinterpret_cast<uint64_t*>(smem + Ly::OFF_L1EMPTY) + s, NW);
        }
    tma::init_barriers<NS>(full, empty, NW + 1);
    tma::pdl_wait_and_release();
    const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
    tma::SegIter it = tma::seg_iter(p);
    tma::Seg sg;

    if (warp == 2 * NW + 1) {  // producer
        if (lane == 0) {
            tma::RingPos ring;
            while (tma::seg_next<NW, 4>(p, it, sg)) {
                const int n_in = (int)(sg.ye - sg.ys) + 4 * R;
                const int P = (n_in + NS - 1) / NS * NS;
                tb2_produce_seg<NS>(p, sg, smem, Ly::SB, full, empty, sg.ys - 2 * R, n_in, P, ring,
                                    CM == COL_WRAP);
            }
        }
        return;
    }
    const unsigned long long cwq = to_const(&c_tb_wq[pp.slot][0]);
    const unsigned long long cw = to_const(&c_conv_w[pp.slot][0]);
    Acc2 a[K][2];
#pragma unroll
    for (int d = 0; d < K; ++d) a[d][0] = a[d][1] = 0ull;
    uint32_t h = 0, ph = 0;  // the group's half and the round's phase parity
    auto next_group = [&]() {
        h ^= 1u;
        ph ^= (h ^ 1u);
    };

    if (warp < NW || warp == 2 * NW) {
        // ---- level 1; the ghost warp's lanes 0 / 1: the vectors left / right of the strip
        const bool ghost = warp == 2 * NW;
        const int v = ghost ? (lane == 0 ? -1 : NW * 32) : warp * 32 + lane;
        const bool on = !ghost || lane < 2;
        const uint32_t lo4 = (uint32_t)(16 * v);  // the lane's byte offset in a row (column 4v)
        while (tma::seg_next<NW, 4>(p, it, sg)) {
            const int seg = (int)sg.seg;
            const int n_in = (int)(sg.ye - sg.ys) + 4 * R;
            const int P = (n_in + NS - 1) / NS * NS;
            const bool lf = CM != COL_WRAP && on && sg.first_strip && v == 0;
            const bool rf = CM != COL_WRAP && on && sg.last_strip && 4 * v + 4 == seg;
            // vectors outside the grid under CLAMP / ZERO are not stored (lf / rf write those margins)
            const bool store = on && !(CM != COL_WRAP && ((sg.first_strip && v < 0) || (sg.last_strip && 4 * v >= seg)));
            const bool wedge = __any_sync(0xffffffffu, lf || rf);
            auto step = [&](auto JC, int j, auto fullc) {
                constexpr int J = decltype(JC)::value;
                constexpr bool FULL = decltype(fullc)::value;
                const uint32_t hs = h * K;  // slot of J = 0
                const uint32_t st = sb + hs * Ly::SB + J * Ly::SB + kTbMargin * 4;  // stage column 0
                const uint32_t rw = sb + Ly::OFF_L1 + hs * Ly::L1B + J * Ly::L1B + kTbL1Margin * 4;  // ring row column 0
                // every lane runs the taps of every step, padding included: an
                // accumulator is zeroed when its row starts and completes 2R
                // steps later, so stale stage data never reaches a stored row
                // (and no lane-dependent control flow doubles the accumulators)
                mbar_wait_s(sb + Ly::OFF_FULL + (hs + J) * 8, ph);
                float b[2 * R + 4];
                window_s<R>(st + lo4, b);
                warp_arrive(sb + Ly::OFF_EMPTY + (hs + J) * 8);
                if (wedge) {
#pragma unroll
                    for (int t = 0; t < R; ++t) b[t] = lf ? (CM == COL_CLAMP ? b[R] : 0.f) : b[t];
#pragma unroll
                    for (int t = R + 4; t < 2 * R + 4; ++t) b[t] = rf ? (CM == COL_CLAMP ? b[R + 3] : 0.f) : b[t];
                }
                taps_ph<R, J % K>(a, b, cwq, cw);
                // the slot's previous occupant released (first round: parity 1 of a fresh barrier passes)
                mbar_wait_s(sb + Ly::OFF_L1EMPTY + (hs + J) * 8, ph ^ 1u);
                if (FULL || (j >= 2 * R && j < n_in)) {
                    constexpr int DONE = (J - R + K) % K;
                    if (store) st_shared_pairs_s(rw + lo4, a[DONE][0], a[DONE][1]);
                    if (wedge) {
                        if (lf) st_shared_f4_s(rw - 16, CM == COL_CLAMP ? __uint_as_float((unsigned)a[DONE][0]) : 0.f);
                        if (rf)
                            st_shared_f4_s(rw + lo4 + 16,
                                           CM == COL_CLAMP ? __uint_as_float((unsigned)(a[DONE][1] >> 32)) : 0.f);
                    }
                }
                warp_arrive(sb + Ly::OFF_L1FULL + (hs + J) * 8);
            };
#pragma unroll 1
            for (int j0 = 0; j0 < P; j0 += K) {
                if (j0 >= 2 * R && j0 + K <= n_in)
                    group_steps<K>([&](auto JC, int) { step(JC, j0 + decltype(JC)::value, std::true_type()); });
                else
                    group_steps<K>([&](auto JC, int) { step(JC, j0 + decltype(JC)::value, std::false_type()); });
                next_group();
            }
        }
    } else {
        // ---- level 2
        const int v = (warp - NW) * 32 + lane;
        const uint32_t lo4 = (uint32_t)(16 * v);
        const bool clamp_top = p.top_map == ROWMAP_CLAMP, clamp_bot = p.bot_map == ROWMAP_CLAMP;
        const bool edge_top = clamp_top || pp.zero_top, edge_bot = clamp_bot || pp.zero_bot;
        while (tma::seg_next<NW, 4>(p, it, sg)) {
            const int n_in = (int)(sg.ye - sg.ys) + 4 * R;
            const int P = (n_in + NS - 1) / NS * NS;
            const int64_t ys = sg.ys;
            const bool active = 4 * v < (int)sg.seg;
            // steps whose fed row needs the row map: top j < jt, bottom j >= jb
            const int jt = edge_top ? (int)(3 * R - ys) : 0;
            const int jb = edge_bot ? (int)(p.rows - ys + 3 * R) : n_in;
            const int jhold = (clamp_bot && jb < n_in) ? jb - 1 : -1;  // the bottom CLAMP edge row's step
            float* outp = reinterpret_cast<float*>(p.out) + sg.e0 + 4 * v + (ys - 4 * R) * p.pitch;
            const int64_t pitch = p.pitch;
            const int lo = jt > 4 * R ? jt : 4 * R, hi = jb < n_in ? jb : n_in;
            auto step = [&](auto JC, int j, auto fullc) {
                constexpr int J = decltype(JC)::value;
                constexpr bool FULL = decltype(fullc)::value;
                const uint32_t hs = h * K;
                const uint32_t slot = hs + J;
                mbar_wait_s(sb + Ly::OFF_L1FULL + slot * 8, ph);
                if (FULL || (j >= 2 * R && j < n_in)) {
                    uint32_t src = sb + Ly::OFF_L1 + slot * Ly::L1B + kTbL1Margin * 4;
                    int relh = -1;
                    if (!FULL) {
                        const int64_t y = ys - 3 * R + j;  // generation-t+1 row fed by step j
                        int jm = j;
                        if (y < 0 && edge_top) jm = clamp_top ? j - (int)y : -1;                       // row 0
                        else if (y >= p.rows && edge_bot) jm = clamp_bot ? j - (int)(y - (p.rows - 1)) : -1;  // row rows-1
                        if (jm < 0) {
                            src = sb + Ly::OFF_ZERO + kTbL1Margin * 4;
                        } else if (jm != j) {
                            // the mapped row's slot / phase (within R steps: same or adjacent round)
                            int ms = (int)slot + (jm - j);
                            uint32_t mph = ph;
                            if (ms >= NS) {
                                ms -= NS;
                                mph ^= 1u;
                            } else if (ms < 0) {
                                ms += NS;
                                mph ^= 1u;
                            }
                            mbar_wait_s(sb + Ly::OFF_L1FULL + ms * 8, mph);
                            src = sb + Ly::OFF_L1 + ms * Ly::L1B + kTbL1Margin * 4;
                            if (jm == jhold && j == n_in - 1) relh = ms;
                        }
                    }
                    float b[2 * R + 4];
                    window_s<R>(src + lo4, b);
                    if (FULL || j != jhold) warp_arrive(sb + Ly::OFF_L1EMPTY + slot * 8);
                    if (!FULL && relh >= 0) warp_arrive(sb + Ly::OFF_L1EMPTY + relh * 8);  // after its last read
                    constexpr int PH = ((J - 2 * R) % K + K) % K;
                    taps_ph<R, PH>(a, b, cwq, cw);
                    if ((FULL || j >= 4 * R) && active) {
                        constexpr int DONE = (PH - R + K) % K;
                        st_global_pairs(outp, a[DONE][0], a[DONE][1]);
                    }
                } else {
                    warp_arrive(sb + Ly::OFF_L1EMPTY + slot * 8);
                }
                outp += pitch;
            };
#pragma unroll 1
            for (int j0 = 0; j0 < P; j0 += K) {
                if (j0 >= lo && j0 + K <= hi)
                    group_steps<K>([&](auto JC, int) { step(JC, j0 + decltype(JC)::value, std::true_type()); });
                else
                    group_steps<K>([&](auto JC, int) { step(JC, j0 + decltype(JC)::value, std::false_type()); });
                next_group();
            }
        }
    }
    (void)S;
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
    const int smem = TbLayout<R, NC>::BYTES;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(conv_tb2_kernel<R, NC, NS, CM>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    const int64_t ctas = tma_plan_grid(p, b, num_sms, 1, S);
    tma_record(g.rec, LK_CONV_TB2, p, ctas, (2 * NC + 2) * 32, smem, NS, 1, NC, 2);
    if (ctas == 0) return cudaSuccess;
    return tma_launch(conv_tb2_kernel<R, NC, NS, CM>, (unsigned)ctas, (2 * NC + 2) * 32, smem, s, pp, g.pdl);
}

template <int R>
cudaError_t launch_conv_tb2_r(const StencilGeom& g, const RowBands& b, int zero_top, int zero_bot, int num_sms,
                              cudaStream_t s) {
    constexpr int NS = 2 * (2 * R + 1);  // both rings: 2K slots (conv_tb2_kernel)
    const int64_t nvec = g.w / 4;
    auto go = [&](auto nc_tag) -> cudaError_t {
        constexpr int NC = decltype(nc_tag)::value;
        switch (g.col_mode) {
            case COL_WRAP: return launch_conv_tb2_t<R, NC, NS, COL_WRAP>(g, b, zero_top, zero_bot, num_sms, s);
            case COL_CLAMP: return launch_conv_tb2_t<R, NC, NS, COL_CLAMP>(g, b, zero_top, zero_bot, num_sms, s);
            default: return launch_conv_tb2_t<R, NC, NS, COL_ZERO>(g, b, zero_top, zero_bot, num_sms, s);
        }
    };
    if (nvec > 4 * 32) return go(std::integral_constant<int, kTbWarps>());
    return go(std::integral_constant<int, 4>());
}

}  // namespace conv_detail
}  // namespace mapsm
