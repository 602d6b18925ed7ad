// plan.cpp — row-slab partition and static halo plan (pure host arithmetic).
//
// The Segmenter / Memory Analyzer / Segment Location Monitor of the paper
// (§4, §4.2, Alg 2 P:L335-339 §4.4) reduced to what the
// Window(2D) -> Structured Injective path needs:
//   * thread blocks (here: output rows) are split evenly over the g devices
//     (§2.1), the first h mod g slabs taking one extra row (reading c8);
//   * every buffer gets r halo rows above and below, for BOTH buffers of the
//     double-buffered pair (Fig 3 after the second AnalyzeCall);
//   * the N-D intersection of a slab's required segment with the other
//     devices' lastOutput (Alg 2 line 10) is, for rows_j >= r, exactly the
//     r rows of the up neighbour (top halo) and of the down neighbour (bottom
//     halo), taken mod h under WRAP — the "naive O(g)" search collapses
//     to two neighbours, so it is computed in O(1).
#include <cstdint>

#include "mapsm.h"

namespace mapsm {

mapsm_status compute_plan(int64_t h, int g, int r, mapsm_boundary b, int rank, mapsm_slab_plan* out) {
    if (!out || g < 1 || h < 1 || r < 0 || rank < 0 || rank >= g) return MAPSM_EINVAL;
    if (b != MAPSM_WRAP && b != MAPSM_CLAMP && b != MAPSM_ZERO && b != MAPSM_NO_CHECKS) return MAPSM_EINVAL;
    if (b == MAPSM_NO_CHECKS && r != 0) return MAPSM_EINVAL;  // NO_CHECKS = no neighbours (radius 0)
    const int64_t base = h / g, extra = h % g;
    if (g > 1 && base < r) return MAPSM_EINVAL;  // a halo row would not belong to a neighbour
    mapsm_slab_plan p;
    p.rows = base + (rank < extra ? 1 : 0);
    p.y0 = (int64_t)rank * base + (rank < extra ? rank : extra);
    p.alloc_rows = p.rows + 2 * (int64_t)r;
    if (g == 1) {
        p.up = p.down = -1;
        const int k = (b == MAPSM_WRAP) ? MAPSM_HALO_WRAP_LOCAL : (b == MAPSM_CLAMP) ? MAPSM_HALO_CLAMP : MAPSM_HALO_ZERO;
        p.top_kind = p.bottom_kind = k;
    } else if (b == MAPSM_WRAP) {
        p.up = (rank - 1 + g) % g;
        p.down = (rank + 1) % g;
        p.top_kind = p.bottom_kind = MAPSM_HALO_EXCHANGE;
    } else {
        const int edge = (b == MAPSM_CLAMP) ? MAPSM_HALO_CLAMP : MAPSM_HALO_ZERO;
        p.up = rank > 0 ? rank - 1 : -1;
        p.down = rank < g - 1 ? rank + 1 : -1;
        p.top_kind = p.up >= 0 ? MAPSM_HALO_EXCHANGE : edge;
        p.bottom_kind = p.down >= 0 ? MAPSM_HALO_EXCHANGE : edge;
    }
    if (r == 0) {
        p.top_kind = p.bottom_kind = MAPSM_HALO_ZERO;  // nothing to exchange
        p.up = p.down = -1;
    }
    auto modh = [h](int64_t v) { int64_t m = v % h; return m < 0 ? m + h : m; };
    p.top_src_row = p.top_kind == MAPSM_HALO_EXCHANGE ? modh(p.y0 - r) : -1;
    p.bottom_src_row = p.bottom_kind == MAPSM_HALO_EXCHANGE ? modh(p.y0 + p.rows) : -1;
    p.n_send = (p.top_kind == MAPSM_HALO_EXCHANGE) + (p.bottom_kind == MAPSM_HALO_EXCHANGE);
    p.n_recv = p.n_send;
    *out = p;
    return MAPSM_OK;
}

}  // namespace mapsm

extern "C" mapsm_status mapsm_plan_query(int64_t h, int g, int radius, mapsm_boundary boundary, int rank,
                                         mapsm_slab_plan* out) {
    return mapsm::compute_plan(h, g, radius, boundary, rank, out);
}
