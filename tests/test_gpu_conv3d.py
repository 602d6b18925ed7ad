"""GPU parity: the Window(3D) fp32 convolution (P:L526,
Table 1) through the C ABI vs the CPU oracle (oracle.conv3d).

Bit-exact (both sides evaluate the same (dz, dy, dx) fmaf chain, reading v1),
which implies the north_star gate max|d| <= 1e-5 * max(1, max|o|) that is also
asserted.  Shapes span several 64 x 16 tiles with ragged x / y / z tails, one-
plane and one-row volumes, radii 1-4, all boundaries, plane-slab partitions
g = 2..4 (halo planes exchanged every iteration), and the bench volume on
light-cone samples."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval3d
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def check(got, exp):
    tol = 1e-5 * max(1.0, float(np.abs(exp).max()))
    assert float(np.abs(got.astype(np.float64) - exp).max()) <= tol
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))


def run(ctx, vol, W, n, boundary):
    d, h, w = vol.shape
    r = W.shape[0] // 2
    with M.Grid(ctx, w, h, "conv", r, boundary, W, d=d) as g:
        g.bind(vol)
        g.iterate(n)
        out = g.gather()
        info = g.info()
    return out, info


SHAPES = [(1, 1, 1), (1, 16, 64), (5, 7, 9), (8, 16, 64), (3, 17, 65), (12, 33, 130), (9, 40, 257), (20, 5, 3)]


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("r", [1, 2, 3, 4])
@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_vs_oracle(ctx, shape, r, boundary):
    d, h, w = shape
    vol = mi.volume_f32(1000 + w + h + d, w, h, d)
    W = mi.weights3d_f32(2000 + r, r)
    for n in (1, 3):
        got, info = run(ctx, vol, W, n, boundary)
        check(got, oracle.conv3d(vol, W, n, boundary))
        assert info.d == d and info.generation == n


@pytest.mark.parametrize("g", [2, 3, 4])
@pytest.mark.parametrize("r", [1, 2, 3, 4])
@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_plane_slabs_exchange(local_ctx, g, r, boundary):
    d, h, w = max(4, r) * g + 1, 19, 70
    vol = mi.volume_f32(3000 + g, w, h, d)
    W = mi.weights3d_f32(3100 + r, r)
    got, info = run(local_ctx(g), vol, W, 5, boundary)
    check(got, oracle.conv3d(vol, W, 5, boundary))
    assert info.world == g and info.exchanges > 0


def test_negative_weights_and_planar_equals_2d(ctx):
    """Signed weights; and weights only on dz = 0 evolve each plane like the
    2-D path (cross-check of the plane indexing)."""
    d, h, w = 6, 24, 96
    vol = mi.volume_f32(41, w, h, d) - 0.5
    W = mi.weights3d_f32(42, 1) - np.float32(1.0 / 27)
    got, _ = run(ctx, vol.astype(np.float32), W.astype(np.float32), 2, "clamp")
    check(got, oracle.conv3d(vol, W, 2, "clamp"))
    Wp = np.zeros((3, 3, 3), np.float32)
    Wp[1] = mi.weights_f32(43, 1)
    vol = mi.volume_f32(44, w, h, d)
    got, _ = run(ctx, vol, Wp, 3, "wrap")
    for z in range(d):
        assert np.array_equal(got[z].view(np.uint32), oracle.conv(vol[z], Wp[1], 3, "wrap").view(np.uint32))


def test_validation(ctx):
    with pytest.raises(M.MapsmError) as e:
        M.mapsm_grid_create_3d(ctx, 8, 8, 8, M.U8)
    assert e.value.status == M.EUNSUPPORTED
    g = M.mapsm_grid_create_3d(ctx, 8, 8, 8, M.F32)
    try:
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_window_set(g, 5, M.WRAP)   # Window(3D) radii 1..4
        assert e.value.status == M.EUNSUPPORTED
        M.mapsm_window_set(g, 1, M.WRAP)
        assert M.mapsm_grid_slab(g, 0) == (0, 8)
        M.mapsm_op_set(g, M.OP_CONV, mi.weights3d_f32(1, 1))
        with pytest.raises(M.MapsmError) as e:   # the fused P2P exchange is 2-D only
            M.mapsm_set_option(g, M.OPT_EXCHANGE, M.EXCHANGE_P2P)
            M.mapsm_bind(g, mi.volume_f32(1, 8, 8, 8), 32)
        assert e.value.status == M.EUNSUPPORTED
    finally:
        M.mapsm_grid_destroy(g)


def test_chained_histogram_of_a_volume(local_ctx):
    d, h, w = 13, 21, 50
    vol = mi.volume_f32(51, w, h, d)
    W = mi.weights3d_f32(52, 2)
    with M.Grid(local_ctx(3), w, h, "conv", 2, "zero", W, d=d) as g:
        g.bind(vol)
        g.iterate(2)
        exp = oracle.histogram_f32(oracle.conv3d(vol, W, 2, "zero").reshape(d * h, w))
        for T in (0, 2, 1):
            bins, _ = g.task_histogram(T)
            assert np.array_equal(bins, exp)


@pytest.mark.parametrize("boundary", ["zero", "wrap"])
def test_bench_volume_on_cones(ctx, boundary):
    """512^3 r = 1 (the bench workload) after 6 iterations, on light-cone
    samples at corners, edges and the interior."""
    import torch

    d = h = w = 512
    r, n = 1, 6
    seed = mi.SEED_CONV3D_FIELD
    W = mi.weights3d_f32(mi.SEED_CONV3D_W, r)
    vol = torch.from_numpy(mi.volume_f32(seed, w, h, d)).pin_memory()
    with M.Grid(ctx, w, h, "conv", r, boundary, W, d=d) as g:
        g.bind(vol)
        g.iterate(n)
        out = torch.empty((d, h, w), dtype=torch.float32, device="cuda")
        M.mapsm_read(g.handle, out, w * 4)
        torch.cuda.synchronize()

    def vol_rows(z, y0, nr):
        return mi.field_f32(seed, w, nr, y0=z * h + y0)

    for zr, yr, xr in [((0, 4), (0, 4), (0, 8)), ((508, 512), (508, 512), (504, 512)), ((250, 254), (0, 3), (300, 309)),
                       ((100, 103), (200, 205), (509, 512)), ((0, 2), (511, 512), (0, 512))]:
        exp = cone_eval3d(vol_rows, d, h, w, r, n, boundary, zr, yr, xr, W)
        got = out[zr[0]:zr[1], yr[0]:yr[1], xr[0]:xr[1]].cpu().numpy()
        check(got, exp)
