"""The fused compute + peer-memory halo exchange (MAPSM_OPT_EXCHANGE = P2P):
one kernel per iteration whose boundary CTAs write their rows into the
neighbours' halos and signal a device mailbox.  Exercised here with g slabs
in one process on one GPU (same kernels and protocol; the pointers are local
instead of CUDA-IPC peer mappings) — bit-exact against the oracle."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def run_life(ctx, g0, n, b, steps=None):
    h, w = g0.shape
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        g.bind(g0)
        for k in (steps or [n]):
            g.iterate(k)
        return g.gather(), g.info()


@pytest.mark.parametrize("g", [2, 3, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
def test_life_fused_exchange(local_ctx, g, b):
    h, w, n = 8 * 11 + 3, 512, 17
    g0 = mi.life_u8(900 + g, w, h)
    out, info = run_life(local_ctx(g), g0, n, b, steps=[5, 1, 11])
    assert np.array_equal(out, oracle.life(g0, n, b))
    assert info.launches == g * n  # one fused launch per slab and iteration


@pytest.mark.parametrize("g", [2, 4])
def test_life_fused_wide_rows_many_strips(local_ctx, g):
    """Rows wider than one CTA strip (several strips deliver per generation)."""
    h, w, n = 40, 65536 + 128, 6
    g0 = mi.life_u8(31, w, h)
    out, _ = run_life(local_ctx(g), g0, n, "wrap")
    assert np.array_equal(out, oracle.life(g0, n, "wrap"))


@pytest.mark.parametrize("g", [2, 3, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_conv_fused_exchange(local_ctx, g, b, r):
    h, w, n = 8 * (2 * r + 2) + 5, 2048 + 16, 7
    f0 = mi.field_f32(700 + g + r, w, h)
    W = mi.weights_f32(710 + r, r)
    with M.Grid(local_ctx(g), w, h, "conv", r, b, W) as gr:
        gr.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        gr.bind(f0)
        gr.iterate(3)
        gr.iterate(n - 3)
        out = gr.gather()
    exp = oracle.conv(f0, W, n, b)
    assert np.array_equal(out.view(np.uint32), exp.view(np.uint32))


def test_rebind_resets_protocol(local_ctx):
    g0 = mi.life_u8(5, 256, 64)
    g1 = mi.life_u8(6, 256, 64)
    with M.Grid(local_ctx(4), 256, 64, "life", 1, "wrap") as g:
        g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        g.bind(g0)
        g.iterate(9)
        assert np.array_equal(g.gather(), oracle.life(g0, 9, "wrap"))
        g.bind(g1)
        g.iterate(4)
        assert np.array_equal(g.gather(), oracle.life(g1, 4, "wrap"))


def test_ineligible_grid_is_rejected(local_ctx):
    with M.Grid(local_ctx(2), 192, 64, "life", 1, "wrap") as g:  # 192 % 128 != 0: register kernel only
        g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        with pytest.raises(M.MapsmError) as e:
            g.bind(np.zeros((64, 192), np.uint8))
        assert e.value.status == M.EUNSUPPORTED
