"""The light-cone sampler used by the full-size GPU parity tests agrees with
the whole-grid oracle (CPU)."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("blk", [(0, 4, 0, 8), (60, 64, 100, 128), (30, 35, 61, 67), (0, 64, 0, 3)])
def test_life_cone_matches_full(b, blk):
    h, w, n = 64, 128, 9
    gen = lambda y0, k: mi.life_u8(77, w, k, y0=y0)
    full = oracle.life(gen(0, h), n, b)
    ys, ye, xs, xe = blk
    assert np.array_equal(cone_eval("life", gen, h, w, 1, n, b, ys, ye, xs, xe), full[ys:ye, xs:xe])


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("blk", [(0, 3, 0, 5), (40, 44, 50, 56), (20, 23, 0, 56)])
def test_conv_cone_matches_full(b, blk):
    h, w, n, r = 44, 56, 4, 2
    W = mi.weights_f32(3, r)
    gen = lambda y0, k: mi.field_f32(78, w, k, y0=y0)
    full = oracle.conv(gen(0, h), W, n, b)
    ys, ye, xs, xe = blk
    got = cone_eval("conv", gen, h, w, r, n, b, ys, ye, xs, xe, W)
    assert np.array_equal(got.view(np.uint32), full[ys:ye, xs:xe].view(np.uint32))
