"""GPU parity on the launch configurations the bench times, element by element.

The TMA ring kernels (life_tma_kernel, conv_tma_kernel) split the flattened
(strip, output row) space of a slab evenly over one wave of CTAs and stream
each CTA's rows through an NS-stage shared-memory ring with a loop unrolled by
NS (tma_rows.cuh).  Small grids give every CTA 1-2 rows, so only the
partial-trip tail runs; the bench workloads give each CTA hundreds of rows,
i.e. the first trip, many steady trips, the phase flip every NS rows and the
re-alignment between segments.  These tests drive every bench instantiation
(Life NC = 16/8/4/2 consumer warps, conv r = 1..4) through >= 2 full ring
trips per CTA — asserted from the library's own launch record
(mapsm_launch_query), so a test cannot silently shrink below that — and
compare the whole grid cell for cell with the oracle (north_star: "bit-exact
... on the same seeded random grids"; §4 double-buffered generations;
P:L469 §5.2 the 8K GoL experiment)."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu

KERNEL_LIFE_TMA = 1
KERNEL_LIFE_PERSIST = 4
KERNEL_CONV_TMA = 6


def _assert_full_trips(li, n_in_extra, kernel, nc=None, steady_on_out=False):
    """Every CTA's longest segment runs the unrolled first trip and at least
    one steady trip: Life needs n_in = rows + 2 >= 2 NS, conv n_out >= 2 NS."""
    assert li.kernel == kernel, (li.kernel, M.KERNEL_NAMES.get(li.kernel))
    if nc is not None:
        assert li.consumer_warps == nc, li.consumer_warps
    ns = li.ring_stages
    assert ns > 0
    need = 2 * ns - (0 if steady_on_out else n_in_extra)
    assert li.min_cta_seg_rows >= need, (li.min_cta_seg_rows, ns, li.ctas)
    return ns


# (w, h, consumer warps): every Life TMA instantiation the row width selects
# (w = 65536 is the bench's NC = 16); heights are ragged (not a multiple of
# the CTA count) so CTAs get unequal row runs.
LIFE_SHAPES = [(65536, 8192 + 37, 16), (32768, 16384 + 5, 8), (16384, 32768 + 11, 4), (4096, 131072 + 77, 2)]


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", LIFE_SHAPES, ids=lambda s: f"{s[0]}x{s[1]}_nc{s[2]}")
def test_life_full_ring_trips_vs_oracle(ctx, shape, b):
    w, h, nc = shape
    g0 = mi.life_u8(0x5EED0100 + nc, w, h)
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.bind(g0)
        g.iterate(1)
        li = g.launch()
        _assert_full_trips(li, 2, KERNEL_LIFE_TMA, nc)
        got1 = g.gather()
        exp1 = oracle.life(g0, 1, b)
        assert np.array_equal(got1, exp1), "generation 1"
        del got1
        g.iterate(2)
        got3 = g.gather()
    exp3 = oracle.life(exp1, 2, b)
    assert np.array_equal(got3, exp3), "generation 3"


def test_life_bench_kernel_graph_replay_vs_oracle(ctx):
    """The bench's exact launch path for the 65536-wide rows: CUDA graphs of
    16 generations (two replays + a direct tail), WRAP."""
    w, h = 65536, 8192 + 37
    n = 35
    g0 = mi.life_u8(0x5EED0003, w, h)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(n)
        info = g.info()
        li = g.launch()
        got = g.gather()
    assert info.used_graphs == 1 and info.launches == n
    _assert_full_trips(li, 2, KERNEL_LIFE_TMA, 16)
    assert np.array_equal(got, oracle.life(g0, n, "wrap"))


def test_config1_8192_full_grid_1000_generations(ctx):
    """BASELINE configs[1] in full: 8192^2 random (seed 0x5EED0002), 1000
    generations, WRAP, the bench's launch path — compared on every cell."""
    w = h = 8192
    n = 1000
    g0 = mi.life_u8(mi.SEED_LIFE_8K, w, h)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(n)
        li = g.launch()
        got = g.gather()
    assert li.kernel in (KERNEL_LIFE_PERSIST, M.KERNEL_LIFE_TB_PERSIST), M.KERNEL_NAMES.get(li.kernel)
    assert np.array_equal(got, oracle.life(g0, n, "wrap"))


# conv: (r, w, h).  r = 2 at the 5x5 bench's row width (16 consumer warps, 8
# strips of 2048 floats, 1 CTA/SM); r = 4 at the 9x9 bench's width (16
# consumer warps, 16 strips of 2048 floats, weights in a constant slot); r =
# 1, 3 at widths that select the same instantiations.
CONV_SHAPES = [(2, 16384, 2048 + 3), (4, 32768, 1024 + 5), (1, 16384, 2048 + 1), (3, 32768, 512 + 7)]


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", CONV_SHAPES, ids=lambda s: f"r{s[0]}_{s[1]}x{s[2]}")
def test_conv_full_ring_trips_vs_oracle(ctx, shape, b):
    r, w, h = shape
    f0 = mi.field_f32(0x5EED0200 + r, w, h)
    W = mi.weights_f32(0x5EED0300 + r, r)
    with M.Grid(ctx, w, h, "conv", r, b, W) as g:
        g.bind(f0)
        g.iterate(1)
        li = g.launch()
        _assert_full_trips(li, 2 * r, KERNEL_CONV_TMA, steady_on_out=True)
        got1 = g.gather()
        g.iterate(1)
        got2 = g.gather()
    exp1 = oracle.conv(f0, W, 1, b)
    assert np.array_equal(got1.view(np.uint32), exp1.view(np.uint32)), "iteration 1"
    exp2 = oracle.conv(exp1, W, 1, b)
    tol = 1e-5 * max(1.0, float(np.abs(exp2).max()))
    assert float(np.abs(got2.astype(np.float64) - exp2).max()) <= tol
    assert np.array_equal(got2.view(np.uint32), exp2.view(np.uint32)), "iteration 2"


# ---------------------------------------------------------------------------
# BASELINE full sizes, the bench's exact launch configuration, EVERY cell
# (the oracle runs a few iterations of the full grid in seconds; the long
# runs of the bench are covered by the light-cone tests of test_gpu_life.py /
# test_gpu_conv.py / test_gpu_conv3d.py)

def test_config2_65536_full_grid_two_generations(ctx):
    """BASELINE configs[2] at N = 1: 65536^2 WRAP (seed 0x5EED0003), 148 CTAs
    x ~443 rows through the 24-stage ring — generations 1 and 2, every cell."""
    import torch

    w = h = 65536
    g0 = np.empty((h, w), np.uint8)
    mi.life_u8(mi.SEED_LIFE_64K, w, h, out=g0)
    dev = torch.empty((h, w), dtype=torch.uint8, device="cuda")
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(1)
        li = g.launch()
        _assert_full_trips(li, 2, KERNEL_LIFE_TMA, 16)
        assert li.ctas == 148 and li.min_cta_seg_rows >= 400
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
        exp = oracle.life(g0, 1, "wrap")
        del g0
        assert torch.equal(dev, torch.from_numpy(exp).cuda()), "generation 1"
        g.iterate(1)
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
    exp = oracle.life(exp, 1, "wrap")
    assert torch.equal(dev, torch.from_numpy(exp).cuda()), "generation 2"


def test_config3_5x5_16384_full_grid(ctx):
    """BASELINE configs[3]: 16384^2 CLAMP 5x5 (seeds 0x5EED0004 / 0x5EED0044),
    the bench's kernel and grid — iterations 1 and 2, every cell."""
    w = h = 16384
    f0 = mi.field_f32(mi.SEED_CONV5_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV5_W, 2)
    with M.Grid(ctx, w, h, "conv", 2, "clamp", W) as g:
        g.bind(f0)
        g.iterate(1)
        _assert_full_trips(g.launch(), 4, KERNEL_CONV_TMA, steady_on_out=True)
        got1 = g.gather()
        g.iterate(1)
        got2 = g.gather()
    exp1 = oracle.conv(f0, W, 1, "clamp")
    assert np.array_equal(got1.view(np.uint32), exp1.view(np.uint32))
    exp2 = oracle.conv(exp1, W, 1, "clamp")
    assert np.array_equal(got2.view(np.uint32), exp2.view(np.uint32))


def test_config4_9x9_slab_full_grid(ctx):
    """BASELINE configs[4] per-GPU slab: 32768 x 4096 ZERO 9x9 (seeds
    0x5EED0005 / 0x5EED0055), the bench's kernel (16 consumer warps, weights
    in a constant slot) — iteration 1 and 2, every cell."""
    w, h = 32768, 4096
    f0 = mi.field_f32(mi.SEED_CONV9_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV9_W, 4)
    with M.Grid(ctx, w, h, "conv", 4, "zero", W) as g:
        g.bind(f0)
        g.iterate(2)
        li = g.launch()
        assert li.kernel == KERNEL_CONV_TMA and li.consumer_warps == 16
        got = g.gather()
    exp = oracle.conv(f0, W, 2, "zero")
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))


@pytest.mark.parametrize("r,b,n", [(1, "zero", 2), (2, "clamp", 1)])
def test_window3d_bench_volume_full_grid(ctx, r, b, n):
    """The Window(3D) bench volume 512^3 (r = 1) and a 256^3 r = 2 volume,
    every cell after n iterations."""
    d = h = w = 512 if r == 1 else 256
    v0 = mi.volume_f32(mi.SEED_CONV3D_FIELD, w, h, d)
    W = mi.weights3d_f32(mi.SEED_CONV3D_W + r - 1, r)
    with M.Grid(ctx, w, h, "conv", r, b, W, d=d) as g:
        g.bind(v0)
        g.iterate(n)
        got = g.gather()
    exp = oracle.conv3d(v0, W, n, b)
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))
