"""GPU parity of deep halos for the fp32 convolution (SURVEY §8(f) NEXT-2,
DESIGN.md reading t1) through the C ABI vs the fixed-order fp32 oracle,
bit-exact.

MAPSM_OPT_DEEP_HALO = K keeps K*r halo rows per slab and exchanges them once
per pass of K generations (instead of r rows every generation);
inside a pass every slab recomputes the neighbours' rows it needs on a
trapezoid.  The oracle is the one-iteration-at-a-time definition
(oracle/oracle.c); the schedule must be invisible in the result: several
slabs (g = 1, 2, 4, 8, ragged splits, slabs of exactly K*r rows), all three
boundaries, radii from the TMA kernels (1, 2, 4) to the tiled one (5),
remainders n mod K, odd and even K (buffer parity), CUDA graphs and direct
launches, Window(3D)."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def run(ctx, f0, W, K, b, steps, graphs=True, d=0):
    if d:
        dd, h, w = f0.shape
    else:
        h, w = f0.shape
    r = (W.shape[0] - 1) // 2
    with M.Grid(ctx, w, h, "conv", r, b, W, deep_halo=K, d=d if d else 0) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        g.bind(f0)
        for k in steps:
            g.iterate(k)
        out = g.gather()
        info = g.info()
    return out, info


def same_bits(a, b):
    return np.array_equal(a.view(np.uint32), b.view(np.uint32))


@pytest.mark.parametrize("g", [1, 2, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r,K", [(1, 2), (2, 2), (1, 5), (2, 3), (2, 4), (4, 2), (5, 2)])
def test_local_slabs_vs_oracle(local_ctx, ctx, g, b, r, K):
    w = 512 + 4
    h = g * K * r + 2 * g + 1  # ragged: slabs of K*r + 2 or + 3 rows
    f0 = mi.field_f32(3000 + 31 * r + K + g, w, h)
    W = mi.weights_f32(3100 + r, r)
    n = 2 * K + 1  # two passes and a one-generation remainder
    c = ctx if g == 1 else local_ctx(g)
    out, info = run(c, f0, W, K, b, [n])
    assert info.gens_per_pass == K and info.halo_rows == K * r
    assert same_bits(out, oracle.conv(f0, W, n, b))


@pytest.mark.parametrize("K", [2, 3, 4])
def test_minimum_slabs_of_kr_rows(local_ctx, K):
    """Every slab exactly K*r rows: the whole slab is halo for its neighbours."""
    r, g = 2, 4
    h, w = g * K * r, 256
    f0 = mi.field_f32(77 + K, w, h)
    W = mi.weights_f32(78, r)
    out, _ = run(local_ctx(g), f0, W, K, "wrap", [3 * K])
    assert same_bits(out, oracle.conv(f0, W, 3 * K, "wrap"))


@pytest.mark.parametrize("K", [2, 3])
@pytest.mark.parametrize("graphs", [True, False])
def test_split_calls_graphs_single_slab(ctx, K, graphs):
    """One slab (the bench's process), graphs of several passes, split calls."""
    r = 2
    f0 = mi.field_f32(5, 1024, 300)
    W = mi.weights_f32(6, r)
    steps = [5, 1, 2 * K, 17, K]
    out, info = run(ctx, f0, W, K, "clamp", steps, graphs=graphs)
    n = sum(steps)
    assert info.generation == n
    assert same_bits(out, oracle.conv(f0, W, n, "clamp"))


@pytest.mark.parametrize("g", [1, 2, 3])
@pytest.mark.parametrize("b", ["wrap", "zero"])
def test_window3d_deep_halo(local_ctx, ctx, g, b):
    r, K = 1, 2
    d, h, w = g * K * r + 3, 20, 36
    v0 = mi.volume_f32(900 + g, w, h, d)
    W = mi.weights3d_f32(901, r)
    c = ctx if g == 1 else local_ctx(g)
    out, info = run(c, v0, W, K, b, [2 * K + 1], d=d)
    assert info.halo_rows == K * r
    assert same_bits(out, oracle.conv3d(v0, W, 2 * K + 1, b))


# ---- the fused two-generation kernel (conv_tb.cuh): K = 2, r = 1..2

@pytest.mark.parametrize("r", [1, 2])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("w", [4, 12, 516, 2048, 2052, 8192 + 4])
def test_two_generation_kernel_widths(ctx, r, b, w):
    """Strip edges, partial last strips, whole-row strips, rows narrower than
    the window: one slab, 2 passes + a single generation."""
    h = 37
    f0 = mi.field_f32(4000 + w + r, w, h)
    W = mi.weights_f32(4100 + r, r)
    with M.Grid(ctx, w, h, "conv", r, b, W, deep_halo=2) as g:
        g.bind(f0)
        g.iterate(4)
        li = g.launch()
        mid = g.gather()
        g.iterate(1)  # the remainder runs a single generation
        out = g.gather()
    assert li.kernel == M.KERNEL_CONV_TB2, M.KERNEL_NAMES.get(li.kernel)
    exp4 = oracle.conv(f0, W, 4, b)
    assert same_bits(mid, exp4)
    assert same_bits(out, oracle.conv(exp4, W, 1, b))


def test_two_generation_kernel_config3_full_grid(ctx):
    """BASELINE configs[3] (16384^2 CLAMP 5x5) through the two-generation
    kernel: 2 passes = 4 iterations, every cell."""
    w = h = 16384
    f0 = mi.field_f32(mi.SEED_CONV5_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV5_W, 2)
    with M.Grid(ctx, w, h, "conv", 2, "clamp", W, deep_halo=2) as g:
        g.bind(f0)
        g.iterate(4)
        li = g.launch()
        out = g.gather()
    assert li.kernel == M.KERNEL_CONV_TB2 and li.gens_per_launch == 2
    assert same_bits(out, oracle.conv(f0, W, 4, "clamp"))


def test_two_generation_kernel_negative_weights(ctx):
    """Signed weights and signed zeros: the ZERO-row feeds at the global
    edges are the oracle's fmaf(w, 0, acc) terms, sign of zero included."""
    rng = np.random.default_rng(9)
    f0 = (rng.standard_normal((40, 256))).astype(np.float32)
    f0[0, :8] = -0.0
    W = (rng.standard_normal((5, 5))).astype(np.float32)
    W[2, 2] = -0.0
    with M.Grid(ctx, 256, 40, "conv", 2, "zero", W, deep_halo=2) as g:
        g.bind(f0)
        g.iterate(4)
        out = g.gather()
    assert same_bits(out, oracle.conv(f0, W, 4, "zero"))
