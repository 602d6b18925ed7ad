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

// The halo exchange of one pass (Alg 1's P2P copies, "two-line
// boundary exchanges per iteration") as an ordered message list, for one
// slab buffer laid out as [halo rows | rows owned rows | halo rows] at
// `pitch` bytes per row.  The ISSUE ORDER is part of the contract: send-up
// (my first `depth` rows to up), send-down (my last `depth` rows to down),
// recv-bottom (from down into my bottom halo), recv-top (from up into my top
// halo).  Point-to-point messages between one pair of ranks match in issue
// order, so with g == 2 under WRAP (up == down) the peer's first receive (its
// bottom halo) takes my first send (my top rows) — which is exactly the row
// that follows its last row on the torus.
int exchange_messages(const mapsm_slab_plan& p, int64_t h, int64_t depth, int64_t halo, int64_t pitch,
                      mapsm_msg* out) {
    int n = 0;
    auto modh = [h](int64_t v) { int64_t m = v % h; return m < 0 ? m + h : m; };
    auto put = [&](int kind, int peer, int64_t row) {
        mapsm_msg m;
        m.kind = kind;
        m.peer = peer;
        m.row = row;
        m.rows = depth;
        m.offset = (row + halo) * pitch;
        m.bytes = depth * pitch;
        m.global_row = modh(p.y0 + row);
        out[n++] = m;
    };
    const bool top = p.top_kind == MAPSM_HALO_EXCHANGE, bot = p.bottom_kind == MAPSM_HALO_EXCHANGE;
    if (depth <= 0) return 0;
    if (top) put(MAPSM_MSG_SEND, p.up, 0);
    if (bot) put(MAPSM_MSG_SEND, p.down, p.rows - depth);
    if (bot) put(MAPSM_MSG_RECV, p.down, p.rows);
    if (top) put(MAPSM_MSG_RECV, p.up, -depth);
    return n;
}

}  // namespace mapsm

extern "C" mapsm_status mapsm_exchange_plan(int64_t h, int g, int radius, mapsm_boundary boundary, int rank,
                                            int64_t depth, int64_t halo, int64_t pitch, mapsm_msg* out,
                                            int max_msgs, int* n_msgs) {
    if (!out || !n_msgs || pitch < 1 || depth < 0 || halo < depth) return MAPSM_EINVAL;
    mapsm_slab_plan p;
    mapsm_status st = mapsm::compute_plan(h, g, radius, boundary, rank, &p);
    if (st != MAPSM_OK) return st;
    if (g > 1 && depth > h / g) return MAPSM_EINVAL;  // every halo row must belong to the neighbour
    mapsm_msg tmp[4];
    const int n = mapsm::exchange_messages(p, h, depth, halo, pitch, tmp);
    *n_msgs = n;
    if (n > max_msgs) return MAPSM_ENOMEM;
    for (int i = 0; i < n; ++i) out[i] = tmp[i];
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_gather_plan(int64_t h, int g, int radius, mapsm_boundary boundary, int rank, int root,
                                          int64_t halo, int64_t pitch, mapsm_msg* out, int max_msgs, int* n_msgs) {
    if (!out || !n_msgs || pitch < 1 || halo < 0 || root < 0 || root >= g) return MAPSM_EINVAL;
    mapsm_slab_plan p;
    mapsm_status st = mapsm::compute_plan(h, g, radius, boundary, rank, &p);
    if (st != MAPSM_OK) return st;
    int n = 0;
    const int need = rank == root ? g - 1 : 1;
    *n_msgs = need;
    if (need > max_msgs) return MAPSM_ENOMEM;
    if (rank != root) {
        // my owned rows [0, rows) to the root
        out[n++] = mapsm_msg{MAPSM_MSG_SEND, root, 0, p.rows, halo * pitch, p.rows * pitch, p.y0};
    } else {
        // the root receives every other slab, in slab order, into a staging
        // buffer (offset 0) and places it at global row y0_k
        for (int k = 0; k < g; ++k) {
            if (k == root) continue;
            mapsm_slab_plan q;
            mapsm::compute_plan(h, g, radius, boundary, k, &q);
            out[n++] = mapsm_msg{MAPSM_MSG_RECV, k, 0, q.rows, 0, q.rows * pitch, q.y0};
        }
    }
    return MAPSM_OK;
}

extern "C" mapsm_status mapsm_plan_query(int64_t h, int g, int radius, mapsm_boundary boundary, int rank,
                                         mapsm_slab_plan* out) {
    return mapsm::compute_plan(h, g, radius, boundary, rank, out);
}
