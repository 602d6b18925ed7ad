"""GPU parity: fp32 window convolution through the C ABI vs the fixed-order
fp32 oracle.  The north_star gate is max|d| <= 1e-5 * max(1, max|o|); because
both sides evaluate the same fmaf chain (reading c11) the kernels are in fact
bit-exact, and the tests assert that stronger property too."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def gate(got, exp):
    tol = 1e-5 * max(1.0, float(np.abs(exp).max()))
    assert float(np.abs(got.astype(np.float64) - exp).max()) <= tol
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), "not bit-exact"


def run(ctx, f0, W, n, b, steps=None, graphs=True):
    h, w = f0.shape
    r = W.shape[0] // 2
    with M.Grid(ctx, w, h, "conv", r, b, W) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        g.bind(f0)
        for k in (steps or [n]):
            g.iterate(k)
        out = g.gather()
        info = g.info()
    return out, info


@pytest.mark.parametrize("r", [1, 2, 3, 4])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(4, 9), (8, 8), (16, 5), (132, 70), (260, 33), (1024, 100), (4096 + 4, 40),
                                   (3, 7), (21, 13), (130, 17)])
def test_random_vs_oracle(ctx, r, b, shape):
    w, h = shape
    f0 = mi.field_f32(200 + w, w, h)
    W = mi.weights_f32(300 + r, r)
    for n in (1, 3):
        out, _ = run(ctx, f0, W, n, b)
        gate(out, oracle.conv(f0, W, n, b))


def test_n0_and_split_calls(ctx):
    f0 = mi.field_f32(1, 256, 64)
    W = mi.weights_f32(2, 2)
    out, _ = run(ctx, f0, W, 0, "wrap")
    assert np.array_equal(out, f0)
    a, _ = run(ctx, f0, W, 0, "clamp", steps=[3, 1, 16, 1])
    gate(a, oracle.conv(f0, W, 21, "clamp"))


def test_negative_and_signed_zero_weights(ctx):
    rng = np.random.default_rng(3)
    f0 = (rng.standard_normal((40, 64))).astype(np.float32)
    W = rng.standard_normal((5, 5)).astype(np.float32)
    W[0, 0] = -0.0
    out, _ = run(ctx, f0, W, 2, "zero")
    gate(out, oracle.conv(f0, W, 2, "zero"))


@pytest.mark.parametrize("g", [2, 3, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_local_multislab_partition_invariance(local_ctx, g, b, r):
    h, w, n = 8 * 4 + 3, 96, 5
    f0 = mi.field_f32(40 + g, w, h)
    W = mi.weights_f32(50 + r, r)
    out, info = run(local_ctx(g), f0, W, n, b)
    gate(out, oracle.conv(f0, W, n, b))


def test_config4_5x5_16384_clamp_500_sampled(ctx):
    """BASELINE configs[3] at N=1: 16384^2, 5x5, CLAMP, 500 iterations — the
    bench's conv workload — sampled light cones at corners, edges, interior."""
    import torch

    w = h = 16384
    n, r = 500, 2
    f0 = mi.field_f32(mi.SEED_CONV5_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV5_W, r)
    with M.Grid(ctx, w, h, "conv", r, "clamp", W) as g:
        g.bind(f0)
        g.iterate(n)
        dev = torch.empty((h, w), dtype=torch.float32, device="cuda")
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
    gen = lambda y0, k: mi.field_f32(mi.SEED_CONV5_FIELD, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (16380, 16376), (8000, 9000), (0, 12000)]:
        exp = cone_eval("conv", gen, h, w, r, n, "clamp", ys, ys + 4, xs, xs + 8, W)
        got = dev[ys:ys + 4, xs:xs + 8].cpu().numpy()
        gate(got, exp)


def test_config5_9x9_zero_single_gpu_slab_sampled(ctx):
    """BASELINE configs[4] per-GPU share (reading: 4096 rows x 32768 per GPU):
    9x9 (r=4), ZERO, 100 iterations; sampled light cones."""
    import torch

    w, h = 32768, 4096
    n, r = 100, 4
    f0 = mi.field_f32(mi.SEED_CONV9_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV9_W, r)
    with M.Grid(ctx, w, h, "conv", r, "zero", W) as g:
        g.bind(f0)
        g.iterate(n)
        dev = torch.empty((h, w), dtype=torch.float32, device="cuda")
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
    gen = lambda y0, k: mi.field_f32(mi.SEED_CONV9_FIELD, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (4092, 32760), (2000, 16000)]:
        exp = cone_eval("conv", gen, h, w, r, n, "zero", ys, ys + 4, xs, xs + 8, W)
        got = dev[ys:ys + 4, xs:xs + 8].cpu().numpy()
        gate(got, exp)


# ------------------------------------------- radii 5..8

@pytest.mark.parametrize("r", [5, 6, 7, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(128, 40), (300, 70), (5, 17), (17, 9), (257, 33)])
def test_wide_radius_vs_oracle(ctx, r, b, shape):
    """The shared-memory tile kernel: tiles of 32 x 128 outputs, ragged in
    both directions, windows wider than the grid under WRAP (multiplicity)."""
    w, h = shape
    f0 = mi.field_f32(500 + w + r, w, h)
    W = mi.weights_f32(600 + r, r)
    for n in (1, 2):
        out, _ = run(ctx, f0, W, n, b)
        gate(out, oracle.conv(f0, W, n, b))


@pytest.mark.parametrize("g", [2, 3])
@pytest.mark.parametrize("b", ["wrap", "zero"])
def test_wide_radius_local_multislab(local_ctx, g, b):
    """r = 8 halos of 8 rows exchanged between slabs every iteration."""
    r = 8
    h, w = g * 20 + 3, 160
    f0 = mi.field_f32(77 + g, w, h)
    W = mi.weights_f32(78, r)
    out, info = run(local_ctx(g), f0, W, 3, b)
    gate(out, oracle.conv(f0, W, 3, b))
    assert info.radius == r


def test_wide_radius_limits(ctx, local_ctx):
    gh = M.mapsm_grid_create(ctx, 64, 64, M.F32)
    try:
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_window_set(gh, 9, M.WRAP)
        assert e.value.status == M.EUNSUPPORTED
    finally:
        M.mapsm_grid_destroy(gh)
    # the fused peer-memory exchange needs the TMA kernels (r <= 4)
    with M.Grid(local_ctx(2), 128, 64, "conv", 5, "wrap", mi.weights_f32(1, 5)) as g:
        g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        with pytest.raises(M.MapsmError) as e:
            g.bind(mi.field_f32(1, 128, 64))
        assert e.value.status == M.EUNSUPPORTED
