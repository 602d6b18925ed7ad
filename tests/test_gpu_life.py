"""GPU parity: Life through the C ABI vs the CPU oracle, bit-exact
(BASELINE.json north_star: "bit-exact for Life")."""
import os

import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def run(ctx, g0, n, b, steps=None, graphs=True, graph_iters=None, persistent=True):
    h, w = g0.shape
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        if persistent is not True:
            g.set_option(M.OPT_PERSISTENT, int(persistent))
        if graph_iters:
            g.set_option(M.OPT_GRAPH_ITERS, graph_iters)
        g.bind(g0)
        for k in (steps or [n]):
            g.iterate(k)
        out = g.gather()
        info = g.info()
    return out, info


def test_config0_closed_form(ctx):
    exp = np.zeros((64, 64), np.uint8)
    for line in open(os.path.join(GOLDEN, "life_config0_gen100.txt")):
        if line.strip() and not line.startswith("#"):
            y, x = map(int, line.split())
            exp[y, x] = 1
    out, info = run(ctx, mi.config0_grid(), 100, "wrap")
    assert np.array_equal(out, exp)
    assert info.generation == 100 and info.launches == 1  # persistent kernel: one launch
    out, info = run(ctx, mi.config0_grid(), 100, "wrap", persistent=False)
    assert np.array_equal(out, exp)
    assert info.generation == 100 and info.launches == 100


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(64, 1), (64, 2), (64, 3), (128, 130), (192, 77), (320, 64), (1024, 333),
                                   (4096, 257), (8192 + 64, 100)])
@pytest.mark.parametrize("n", [0, 1, 2, 7])
@pytest.mark.parametrize("persistent", [True, 2, False])
def test_random_vs_oracle(ctx, b, shape, n, persistent):
    w, h = shape
    g0 = mi.life_u8(1000 + w + h, w, h)
    out, _ = run(ctx, g0, n, b, persistent=persistent)
    assert np.array_equal(out, oracle.life(g0, n, b))


def test_nonbinary_input_bytes(ctx):
    rng = np.random.default_rng(1)
    g0 = (rng.integers(0, 4, (50, 128)) * 85).astype(np.uint8)  # 0, 85, 170, 255
    out, _ = run(ctx, g0, 3, "wrap")
    assert np.array_equal(out, oracle.life(g0, 3, "wrap"))
    out0, _ = run(ctx, g0, 0, "wrap")
    assert np.array_equal(out0, (g0 != 0).astype(np.uint8))


@pytest.mark.parametrize("center", [0, 1, 31, 32, 33, 63, 64, 95, 96, 127])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
def test_all_512_neighbourhoods_at_word_edges(ctx, center, b):
    """Every 3x3 neighbourhood centred on a word-edge bit / grid-edge column."""
    w = 128
    h = 512 * 4
    g0 = np.zeros((h, w), np.uint8)
    for m in range(512):
        bits = np.array([(m >> i) & 1 for i in range(9)], np.uint8).reshape(3, 3)
        for dy in range(3):
            for dx in range(3):
                g0[4 * m + dy, (center + dx - 1) % w] = bits[dy, dx]
    out, _ = run(ctx, g0, 1, b)
    assert np.array_equal(out, oracle.life(g0, 1, b))


def test_graphs_direct_and_split_calls_agree(ctx):
    g0 = mi.life_u8(5, 512, 300)
    exp = oracle.life(g0, 37, "wrap")
    a, ia = run(ctx, g0, 37, "wrap", persistent=False)
    b, ib = run(ctx, g0, 37, "wrap", graphs=False, persistent=False)
    c, _ = run(ctx, g0, 37, "wrap", steps=[5, 6, 1, 20, 5], graph_iters=4, persistent=False)
    d, idd = run(ctx, g0, 37, "wrap", steps=[5, 6, 1, 20, 5])
    assert np.array_equal(a, exp) and np.array_equal(b, exp) and np.array_equal(c, exp) and np.array_equal(d, exp)
    assert ia.used_graphs == 1 and ib.used_graphs == 0
    assert ia.launches == ib.launches == 37
    assert idd.launches == 5 and idd.used_graphs == 0  # persistent: one launch per iterate call


@pytest.mark.parametrize("g", [2, 3, 4, 8])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
def test_local_multislab_partition_invariance(local_ctx, g, b):
    h, w, n = 8 * 9 + 5, 256, 11
    g0 = mi.life_u8(31 + g, w, h)
    out, info = run(local_ctx(g), g0, n, b)
    assert np.array_equal(out, oracle.life(g0, n, b))
    assert info.world == g and info.local_slabs == g
    exp_recv = sum(M.mapsm_plan_query(h, g, 1, M.BOUNDARY[b], k).n_recv for k in range(g))
    assert info.exchanges == exp_recv * n


def test_persistent_long_run_many_chunks(ctx):
    """> 1024 generations on the grid-barrier persistent kernel (mode 2):
    several launches, odd total."""
    g0 = mi.life_u8(77, 256, 96)
    out, info = run(ctx, g0, 2051, "wrap", persistent=2)
    assert np.array_equal(out, oracle.life(g0, 2051, "wrap"))
    assert info.launches == 3


# ------------------------------------- SMEM-resident kernel (life_resident.cu)

@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(128, 16), (256, 96), (1024, 333), (4096, 1000), (8192, 1200), (2048, 4096),
                                   (128, 9), (2048, 1), (128, 1), (4096, 2)])
@pytest.mark.parametrize("n", [1, 7, 8, 9, 33])
def test_resident_vs_oracle(ctx, b, shape, n):
    """One cooperative launch, all generations in shared memory, K generations
    between neighbour exchanges: shapes from one CTA to all SMs with R == K
    rows per CTA (4096x1000), ragged splits, n below / at / above K."""
    w, h = shape
    g0 = mi.life_u8(4000 + w + h, w, h)
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.bind(g0)
        g.iterate(n)
        info, li = g.info(), g.launch()
        out = g.gather()
    assert li.kernel == M.KERNEL_LIFE_TB_PERSIST and info.launches == 1 and info.generation == n
    assert np.array_equal(out, oracle.life(g0, n, b))


@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(65536, 256), (65536, 1024), (32768 + 4096, 300), (131072, 64), (32768, 500)])
@pytest.mark.parametrize("persistent", [True, 2])
def test_persistent_wide_rows_vs_oracle(ctx, b, shape, persistent):
    """Rows wider than the resident kernel's warps cover in one chunk
    (w > 512 threads x 64 cells = 32768): every warp then takes several
    column chunks of each row.  Found by the one-rank NCCL ring test (its
    65536 x 1024 grid disagreed with the plain context, whose resident kernel
    left columns >= 32768 uncomputed).  Also the grid-barrier kernel (2)."""
    w, h = shape
    n = 5
    g0 = mi.life_u8(4100 + w + h, w, h)
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.set_option(M.OPT_PERSISTENT, persistent)
        g.bind(g0)
        g.iterate(n)
        li = g.launch()
        out = g.gather()
    assert li.kernel == (M.KERNEL_LIFE_TB_PERSIST if persistent is True else M.KERNEL_LIFE_PERSIST)
    assert np.array_equal(out, oracle.life(g0, n, b))


def test_resident_split_calls_and_parity(ctx):
    """Several iterate calls (odd and even n) keep the buffer parity right."""
    g0 = mi.life_u8(17, 8192, 1024)
    with M.Grid(ctx, 8192, 1024, "life", 1, "wrap") as g:
        g.bind(g0)
        for k in (3, 8, 1, 16, 5):
            g.iterate(k)
        out = g.gather()
    assert np.array_equal(out, oracle.life(g0, 33, "wrap"))


def test_local_multislab_min_height(local_ctx):
    g0 = mi.life_u8(4, 64, 8)
    out, _ = run(local_ctx(8), g0, 13, "wrap")  # rows = r = 1 per slab
    assert np.array_equal(out, oracle.life(g0, 13, "wrap"))


def test_bind_and_read_device_pointers(ctx):
    import torch

    g0 = mi.life_u8(8, 256, 100)
    t = torch.from_numpy(g0).cuda()
    with M.Grid(ctx, 256, 100, "life", 1, "zero") as g:
        g.bind(t)
        g.iterate(6)
        o = torch.empty_like(t)
        M.mapsm_read(g.handle, o)
        torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy(), oracle.life(g0, 6, "zero"))


def test_state_machine_and_errors(ctx):
    gh = M.mapsm_grid_create(ctx, 128, 10, M.U8)
    try:
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_iterate(gh, 1)
        assert e.value.status == M.ESTATE
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_window_set(gh, 2, M.WRAP)
        assert e.value.status == M.EUNSUPPORTED
        M.mapsm_window_set(gh, 1, M.WRAP)
        M.mapsm_bind(gh, np.zeros((10, 128), np.uint8))
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_window_set(gh, 1, M.CLAMP)
        assert e.value.status == M.ESTATE
    finally:
        M.mapsm_grid_destroy(gh)
    gh = M.mapsm_grid_create(ctx, 100, 10, M.U8)  # any width is accepted (NEXT-2)
    try:
        M.mapsm_window_set(gh, 1, M.WRAP)
        assert M.mapsm_get_info(gh).pitch_bytes == 16
    finally:
        M.mapsm_grid_destroy(gh)


def test_config2_8192_full_run_sampled(ctx):
    """BASELINE configs[1]: 8192^2 random (seed 0x5EED0002), 1000 generations,
    WRAP, the bench's launch configuration (graphs); sampled light cones."""
    w = h = 8192
    n = 1000
    g0 = mi.life_u8(mi.SEED_LIFE_8K, w, h)
    out, info = run(ctx, g0, n, "wrap")
    assert info.launches == 1  # the bench's path for this L2-resident grid: one persistent launch
    gen = lambda y0, k: mi.life_u8(mi.SEED_LIFE_8K, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (4000, 6000), (8190, 8160)]:
        exp = cone_eval("life", gen, h, w, 1, n, "wrap", ys, ys + 2, xs, xs + 32)
        got = out[np.arange(ys, ys + 2) % h][:, np.arange(xs, xs + 32) % w]
        assert np.array_equal(got, exp), (ys, xs)


def test_config3_65536_bench_size_sampled(ctx):
    """BASELINE configs[2] at N=1: 65536^2 random (seed 0x5EED0003), 200
    generations, WRAP — exactly the bench's workload — sampled light cones,
    including blocks straddling both wrap edges."""
    import torch

    w = h = 65536
    n = 200
    g0 = np.empty((h, w), np.uint8)
    mi.life_u8(mi.SEED_LIFE_64K, w, h, out=g0)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        del g0
        g.iterate(n)
        dev = torch.empty((h, w), dtype=torch.uint8, device="cuda")
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
        assert g.info().used_graphs == 1
    gen = lambda y0, k: mi.life_u8(mi.SEED_LIFE_64K, w, k, y0=y0)
    for (ys, xs) in [(0, 0), (65530, 65500), (12345, 40000), (32767, 65535)]:
        yy = torch.as_tensor(np.arange(ys, ys + 8) % h, device="cuda")
        xx = torch.as_tensor(np.arange(xs, xs + 64) % w, device="cuda")
        got = dev[yy][:, xx].cpu().numpy()
        exp = cone_eval("life", gen, h, w, 1, n, "wrap", ys, ys + 8, xs, xs + 64)
        assert np.array_equal(got, exp), (ys, xs)
    # population sanity at any size: 0/1 only
    assert int(dev.max()) <= 1


# ------------------------------------------- any width

@pytest.mark.parametrize("w", [1, 2, 3, 31, 32, 33, 63, 65, 96, 100, 161, 1000])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
def test_any_width_vs_oracle(ctx, w, b):
    """Rows of ceil(w/32) words with a partial last word: WRAP pairs column
    w-1 (bit (w-1) % 32 of the last word) with column 0; unused bits stay 0."""
    h = 37
    g0 = mi.life_u8(900 + w, w, h)
    for n in (1, 5):
        out, info = run(ctx, g0, n, b)
        assert np.array_equal(out, oracle.life(g0, n, b)), n


@pytest.mark.parametrize("g", [2, 3])
def test_any_width_local_multislab(local_ctx, g):
    g0 = mi.life_u8(55, 77, 40)
    out, _ = run(local_ctx(g), g0, 9, "wrap")
    assert np.array_equal(out, oracle.life(g0, 9, "wrap"))


def test_any_width_device_pointers(ctx):
    import torch

    g0 = mi.life_u8(8, 45, 30)
    t = torch.from_numpy(g0).cuda()
    with M.Grid(ctx, 45, 30, "life", 1, "clamp") as g:
        g.bind(t)
        g.iterate(4)
        o = torch.full_like(t, 7)
        M.mapsm_read(g.handle, o)
        torch.cuda.synchronize()
    assert np.array_equal(o.cpu().numpy(), oracle.life(g0, 4, "clamp"))
