"""GPU brute-force pins of SURVEY §8(c) (the WRAP rule of P:L174 §4, B3/S23
on the 8-neighbour Moore window of P:L133).

1. Every one of the 2^16 states of a 4x4 torus.  A 4x4 WRAP torus tiled
   periodically is a fixed point of "tile, then step": under WRAP the tiling's
   evolution is the tiling of the torus's evolution.  (a) Literally: sampled
   states tiled 16x16 into a 64x64 WRAP grid, compared with the tiling of the
   oracle's 4x4 result.  (b) All 2^16 states at once: each state tiled into a
   16x16 block, 65536 blocks in one 4096x4096 grid; after n generations a
   cell depends only on cells within distance n (light cone), so the inner
   [n, 16-n)^2 of every block equals the tiling of its torus's generation n,
   whatever the neighbouring blocks hold.  Run on both Life paths the bench
   uses (persistent kernel and the TMA ring kernel).
2. All 512 3x3 neighbourhoods centred on the FIRST and on the LAST row of
   every slab of a g-slab partition (g = 2, 4, 8; copy and fused peer-memory
   exchange), so each one reads a halo row the exchange delivered, at word
   edges and inside words."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def _tori(states):
    """(len(states), 4, 4) uint8: bit i of the state = cell (i // 4, i % 4)."""
    s = np.asarray(states, dtype=np.int64)[:, None]
    bits = (s >> np.arange(16)) & 1
    return bits.reshape(-1, 4, 4).astype(np.uint8)


def _run(ctx, g0, n, b="wrap", persistent=True):
    h, w = g0.shape
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        if not persistent:
            g.set_option(M.OPT_PERSISTENT, 0)
        g.bind(g0)
        g.iterate(n)
        return g.gather(), g.launch()


def test_tiny_tori_tiled_64x64_wrap_sampled(ctx):
    """(a) SURVEY §8(c) literally: state tiled 16x16 -> 64x64 WRAP grid."""
    states = list(range(0, 1 << 16, 257)) + [0xFFFF, 0x0001, 0x8421, 0x0660]
    tori = _tori(states)
    for t, st in zip(tori, states):
        g0 = np.tile(t, (16, 16))
        for n in (1, 4):
            got, _ = _run(ctx, g0, n)
            exp = np.tile(oracle.life(t, n, "wrap"), (16, 16))
            assert np.array_equal(got, exp), (hex(st), n)


@pytest.mark.parametrize("persistent", [True, False])
def test_all_65536_tiny_tori_batched(ctx, persistent):
    """(b) every 4x4 torus state, light-cone batched into one 4096^2 grid."""
    tori = _tori(range(1 << 16))                       # (65536, 4, 4)
    blocks = np.tile(tori, (1, 4, 4))                  # (65536, 16, 16): each torus tiled 4x4
    g0 = blocks.reshape(256, 256, 16, 16).transpose(0, 2, 1, 3).reshape(4096, 4096)
    g0 = np.ascontiguousarray(g0)
    # the oracle, per torus (the plain definition on a 4x4 WRAP grid)
    exp_t = {n: np.empty_like(tori) for n in (1, 2, 3)}
    for n in (1, 2, 3):
        for i in range(1 << 16):
            exp_t[n][i] = oracle.life(tori[i], n, "wrap")
    for n in (1, 2, 3):
        got, li = _run(ctx, g0, n, persistent=persistent)
        if not persistent:
            assert li.kernel == 1  # life_tma_kernel
        gb = got.reshape(256, 16, 256, 16).transpose(0, 2, 1, 3).reshape(1 << 16, 16, 16)
        inner = gb[:, n:16 - n, n:16 - n]
        exp = np.tile(exp_t[n], (1, 4, 4))[:, n:16 - n, n:16 - n]
        bad = np.nonzero((inner != exp).reshape(1 << 16, -1).any(axis=1))[0]
        assert bad.size == 0, (n, [hex(x) for x in bad[:8]])


def _edge_grid(w, h, g, which, shift):
    """All 512 neighbourhoods centred on the first (which=0) or last (1) row of
    every slab of the even g-way row split, centres at columns 4m + shift."""
    g0 = np.zeros((h, w), np.uint8)
    for k in range(g):
        p = M.mapsm_plan_query(h, g, 1, M.WRAP, k)
        yc = p.y0 if which == 0 else p.y0 + p.rows - 1
        for m in range(512):
            bits = np.array([(m >> i) & 1 for i in range(9)], np.uint8).reshape(3, 3)
            xc = (4 * m + shift) % w
            for dy in range(3):
                for dx in range(3):
                    g0[(yc + dy - 1) % h, (xc + dx - 1) % w] = bits[dy, dx]
    return g0


@pytest.mark.parametrize("g", [2, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("mode", ["copy", "p2p"])
def test_512_neighbourhoods_on_slab_edge_rows(local_ctx, g, b, mode):
    w = 2048
    h = 7 * g + 3  # ragged: the first h mod g slabs get one more row
    for which in (0, 1):
        for shift in (0, 31):
            g0 = _edge_grid(w, h, g, which, shift)
            with M.Grid(local_ctx(g), w, h, "life", 1, b) as gr:
                if mode == "p2p":
                    gr.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
                gr.bind(g0)
                gr.iterate(1)
                got = gr.gather()
            assert np.array_equal(got, oracle.life(g0, 1, b)), (which, shift)
