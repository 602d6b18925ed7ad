"""GPU parity of the deep-halo (temporally blocked) Life path — SURVEY §8(f)
NEXT-2 — through the C ABI vs the CPU oracle, bit-exact.

MAPSM_OPT_DEEP_HALO = K keeps K halo rows per slab, exchanges them once per
pass and runs K generations per launch of ``life_tb_kernel``.  The oracle is
the same one-generation-at-a-time definition (oracle/oracle.c); every
difference in how the GPU gets there (ghost words at warp and strip edges,
mirror rows for CLAMP, per-generation zero forcing for ZERO, trapezoids of
rows, remainders n mod K) must be invisible in the result."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu

KS = [2, 3, 4, 6, 8]


def run(ctx, g0, K, b, steps, graphs=True, graph_iters=None):
    h, w = g0.shape
    with M.Grid(ctx, w, h, "life", 1, b, deep_halo=K) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        if graph_iters:
            g.set_option(M.OPT_GRAPH_ITERS, graph_iters)
        g.bind(g0)
        for k in steps:
            g.iterate(k)
        out = g.gather()
        info = g.info()
    return out, info


@pytest.mark.parametrize("K", KS)
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(128, 8), (128, 61), (256, 100), (1024, 9), (4096, 130), (16384, 40),
                                   (15488, 33)])
def test_random_vs_oracle(ctx, K, b, shape):
    w, h = shape
    if h < K:
        pytest.skip("slab shorter than K: per-generation path")
    g0 = mi.life_u8(2000 + w + 7 * h + K, w, h)
    n = 3 * K + 1  # three passes and a one-generation remainder
    out, info = run(ctx, g0, K, b, [n])
    assert info.gens_per_pass == K and info.halo_rows == K
    assert np.array_equal(out, oracle.life(g0, n, b))


@pytest.mark.parametrize("K", [2, 8])
@pytest.mark.parametrize("n", [0, 1, 7, 8, 16, 33])
def test_generation_counts(ctx, K, n):
    g0 = mi.life_u8(44 + n, 512, 96)
    out, info = run(ctx, g0, K, "wrap", [n])
    assert np.array_equal(out, oracle.life(g0, n, "wrap"))
    assert info.generation == n


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("K", [4, 8])
def test_all_512_neighbourhoods_at_warp_and_strip_edges(ctx, b, K):
    """Every 3x3 neighbourhood centred on the columns where a warp's stored
    words end (ghost lanes: words 29|30|31 of a warp = columns 959/960), where
    CTA strips meet (w = 16384 -> 2 strips of 256 words: column 8191/8192),
    and at the grid's first / last column; K generations later the pattern
    has spread over K cells, so each row-block is K+2 rows apart."""
    w = 16384
    cols = [0, 1, 31, 32, 959, 960, 991, 8191, 8192, 8192 + 960, w - 33, w - 32, w - 1]
    sp = 2 * K + 4
    h = 512 * sp
    g0 = np.zeros((h, w), np.uint8)
    for m in range(512):
        bits = np.array([(m >> i) & 1 for i in range(9)], np.uint8).reshape(3, 3)
        for c in cols:
            for dy in range(3):
                for dx in range(3):
                    g0[sp * m + dy, (c + dx - 1) % w] = bits[dy, dx]
    out, _ = run(ctx, g0, K, b, [K])
    assert np.array_equal(out, oracle.life(g0, K, b))


def test_split_calls_graphs_and_direct_agree(ctx):
    """Per-generation remainders break the deep halo (only r rows are
    exchanged then); the next pass must refresh it.  Graphs and direct
    launches, and every split of n, give the same generation."""
    g0 = mi.life_u8(9, 1024, 200)
    exp = oracle.life(g0, 45, "clamp")
    a, ia = run(ctx, g0, 4, "clamp", [45])
    b, ib = run(ctx, g0, 4, "clamp", [45], graphs=False)
    c, _ = run(ctx, g0, 4, "clamp", [5, 3, 1, 8, 20, 8], graph_iters=8)
    for x in (a, b, c):
        assert np.array_equal(x, exp)
    assert ia.launches == ib.launches == 45 // 4 + 1
    assert ia.used_graphs == 1 and ib.used_graphs == 0


@pytest.mark.parametrize("g", [2, 3, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("K", [2, 4, 8])
def test_local_multislab_deep_exchange(local_ctx, g, b, K):
    """g slabs on one GPU with K-row halos exchanged once per pass (device
    copies); split iterate calls force halo refreshes."""
    h, w = g * (2 * K + 3) + 5, 512
    g0 = mi.life_u8(300 + g + K, w, h)
    out, info = run(local_ctx(g), g0, K, b, [2 * K + 3, K, 1, 2 * K])
    n = 5 * K + 4
    assert np.array_equal(out, oracle.life(g0, n, b))
    assert info.halo_rows == K


def test_local_multislab_min_rows(local_ctx):
    """Every slab exactly K rows: the whole slab is boundary band."""
    K, g = 4, 4
    g0 = mi.life_u8(12, 256, K * g)
    out, _ = run(local_ctx(g), g0, K, "wrap", [3 * K])
    assert np.array_equal(out, oracle.life(g0, 3 * K, "wrap"))


def test_errors(ctx, local_ctx):
    gh = M.mapsm_grid_create(ctx, 128, 16, M.U8)
    try:
        M.mapsm_window_set(gh, 1, M.WRAP)
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 5)
        assert e.value.status == M.EUNSUPPORTED
        M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 4)
        assert M.mapsm_get_info(gh).halo_rows == 4
        M.mapsm_bind(gh, np.zeros((16, 128), np.uint8))
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 8)
        assert e.value.status == M.ESTATE
        M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 4)  # unchanged value: fine
    finally:
        M.mapsm_grid_destroy(gh)
    # conv grids: K in 2..16 (tests/test_gpu_conv_deep_halo.py); K = 17 is refused
    gh = M.mapsm_grid_create(ctx, 128, 16, M.F32)
    try:
        M.mapsm_window_set(gh, 1, M.WRAP)
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 17)
        assert e.value.status == M.EUNSUPPORTED
        M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 4)
        assert M.mapsm_get_info(gh).halo_rows == 4
    finally:
        M.mapsm_grid_destroy(gh)
    # g = 4 slabs of 5 rows cannot hold 8-row halos
    gh = M.mapsm_grid_create(local_ctx(4), 128, 20, M.U8)
    try:
        M.mapsm_window_set(gh, 1, M.WRAP)
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 8)
        assert e.value.status == M.EINVAL
        M.mapsm_set_option(gh, M.OPT_DEEP_HALO, 4)  # still usable after the failure
        M.mapsm_bind(gh, mi.life_u8(1, 128, 20))
        M.mapsm_iterate(gh, 8)
        out = np.empty((20, 128), np.uint8)
        M.mapsm_gather(gh, out)
        assert np.array_equal(out, oracle.life(mi.life_u8(1, 128, 20), 8, "wrap"))
    finally:
        M.mapsm_grid_destroy(gh)


def test_fallback_widths_and_short_slabs(ctx):
    """w % 128 != 0 or h < K: the per-generation kernels run (same result)."""
    g0 = mi.life_u8(3, 192, 50)
    out, info = run(ctx, g0, 4, "zero", [9])
    assert np.array_equal(out, oracle.life(g0, 9, "zero")) and info.gens_per_pass == 1
    g0 = mi.life_u8(4, 128, 3)
    out, info = run(ctx, g0, 4, "wrap", [9])
    assert np.array_equal(out, oracle.life(g0, 9, "wrap")) and info.gens_per_pass == 1


@pytest.mark.parametrize("K", [4, 8])
def test_config2_8192_deep_halo_sampled(ctx, K):
    """BASELINE configs[1] (8192^2, 1000 generations, WRAP) on the deep-halo
    path, sampled light cones."""
    w = h = 8192
    n = 1000
    g0 = mi.life_u8(mi.SEED_LIFE_8K, w, h)
    out, info = run(ctx, g0, K, "wrap", [n])
    assert info.gens_per_pass == K
    gen = lambda y0, k: mi.life_u8(mi.SEED_LIFE_8K, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (4000, 6000), (8190, 8160)]:
        exp = cone_eval("life", gen, h, w, 1, n, "wrap", ys, ys + 2, xs, xs + 32)
        got = out[np.arange(ys, ys + 2) % h][:, np.arange(xs, xs + 32) % w]
        assert np.array_equal(got, exp), (ys, xs)


def test_config3_65536_deep_halo_sampled(ctx):
    """BASELINE configs[2] (65536^2, 200 generations, WRAP) with K = 8, the
    bench's deep-halo configuration; sampled light cones incl. both wrap edges
    and a CTA strip boundary."""
    import torch

    w = h = 65536
    n = 200
    g0 = np.empty((h, w), np.uint8)
    mi.life_u8(mi.SEED_LIFE_64K, w, h, out=g0)
    with M.Grid(ctx, w, h, "life", 1, "wrap", deep_halo=8) as g:
        g.bind(g0)
        del g0
        g.iterate(n)
        dev = torch.empty((h, w), dtype=torch.uint8, device="cuda")
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
        assert g.info().gens_per_pass == 8
    gen = lambda y0, k: mi.life_u8(mi.SEED_LIFE_64K, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (65530, 65500), (12345, 13150), (32767, 65535)]:
        yy = torch.as_tensor(np.arange(ys, ys + 8) % h, device="cuda")
        xx = torch.as_tensor(np.arange(xs, xs + 64) % w, device="cuda")
        got = dev[yy][:, xx].cpu().numpy()
        exp = cone_eval("life", gen, h, w, 1, n, "wrap", ys, ys + 8, xs, xs + 64)
        assert np.array_equal(got, exp), (ys, xs)
