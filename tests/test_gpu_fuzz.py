"""Seeded random shapes through every single-GPU kernel path, bit-exact
against the oracle (oracle/oracle.c): the SMEM-resident and grid-barrier
persistent Life kernels, the per-generation TMA / register / any-width Life
kernels, deep-halo Life and conv passes (incl. the two-generation conv
kernel), and the conv TMA / register / wide kernels — small heights
(down to one row), ragged widths, odd and even generation counts, all three
boundaries.  Two resident-kernel bugs (rows wider than 32768 cells, a one-row
CLAMP slab) were found by shape coverage of this kind; this sweep widens it."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu
BOUNDS = ["wrap", "clamp", "zero"]


def life_cases(n_cases, seed):
    rng = np.random.default_rng(seed)
    out = []
    for i in range(n_cases):
        w = int(rng.choice([128, 256, 384, 1024, 2048, 4096, 8192, 12288, 34816, 40960]))
        h = int(rng.choice([1, 2, 3, 5, 8, 17, 64, 100, 149, 300, 777]))
        n = int(rng.integers(1, 24))
        out.append((w, h, n, BOUNDS[i % 3], int(rng.integers(0, 3))))
    return out


@pytest.mark.parametrize("w,h,n,b,mode", life_cases(60, 20261018))
def test_life_fuzz(ctx, w, h, n, b, mode):
    """mode 0: resident / persistent default, 1: grid-barrier persistent, 2: per-generation launches."""
    x0 = mi.life_u8(11000 + w + 7 * h + n, w, h)
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.set_option(M.OPT_PERSISTENT, {0: 1, 1: 2, 2: 0}[mode])
        g.bind(x0)
        g.iterate(n)
        out = g.gather()
    assert np.array_equal(out, oracle.life(x0, n, b))


@pytest.mark.parametrize("w,h,n,b,K", [(w, h, n, b, K) for (w, h, n, b, _), K in
                                       zip(life_cases(24, 77), [2, 3, 4, 6, 8] * 5) if h >= K])
def test_life_deep_fuzz(ctx, w, h, n, b, K):
    x0 = mi.life_u8(12000 + w + h, w, h)
    with M.Grid(ctx, w, h, "life", 1, b, deep_halo=K) as g:
        g.bind(x0)
        g.iterate(n)
        out = g.gather()
    assert np.array_equal(out, oracle.life(x0, n, b))


def conv_cases(n_cases, seed):
    rng = np.random.default_rng(seed)
    out = []
    for i in range(n_cases):
        r = int(rng.choice([1, 2, 3, 4, 5]))
        w = int(rng.choice([4, 8, 12, 36, 100, 516, 1028, 4096, 6004])) + (0 if i % 4 else int(rng.integers(1, 4)))
        h = int(rng.choice([1, 2, 3, 5, 9, 20, 63, 130]))
        n = int(rng.integers(1, 7))
        K = int(rng.choice([1, 1, 2, 3]))
        out.append((r, w, h, n, BOUNDS[i % 3], K))
    return out


@pytest.mark.parametrize("r,w,h,n,b,K", conv_cases(60, 4242))
def test_conv_fuzz(ctx, r, w, h, n, b, K):
    f0 = mi.field_f32(13000 + w + h + r, w, h)
    W = mi.weights_f32(13100 + r, r)
    with M.Grid(ctx, w, h, "conv", r, b, W, deep_halo=K) as g:
        g.bind(f0)
        g.iterate(n)
        out = g.gather()
    assert np.array_equal(out.view(np.uint32), oracle.conv(f0, W, n, b).view(np.uint32))
