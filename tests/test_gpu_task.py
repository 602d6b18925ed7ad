"""GPU parity: chained tasks and GatherAsync.

mapsm_task_histogram runs a Reductive-Static histogram task (Fig 4,
P:L359-403) over a stencil grid's current generation with its own row
partition; the Segment Location Monitor (Alg 2) infers the rows
each target slab must receive.  Checked against the CPU oracle: bins
bit-exact (oracle.histogram of oracle.life / oracle.histogram_f32 of
oracle.conv), and the bytes moved equal to what the cell-level Alg 2 oracle
(oracle/locmon.py) says must move — zero when the partition is unchanged or
the rows are already up to date (upToDate).
"""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from oracle.locmon import CellMonitor
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def even_rows(h, g):
    base, extra = divmod(h, g)
    out, y = [], 0
    for k in range(g):
        n = base + (1 if k < extra else 0)
        out.append((y, y + n))
        y += n
    return out


def expected_moved_rows(h, G, T, ref=None):
    """Rows the targets of a T-slab re-partition must receive from a G-slab
    datum, by the cell-level Alg 2 oracle on a 1-D row model."""
    if ref is None:
        ref = CellMonitor()
        ref.output(0, [(k, (r,)) for k, r in enumerate(even_rows(h, G))])
    n = 0
    for j, r in enumerate(even_rows(h, T)):
        loc = j if T == G else 1000 + j
        pairs, _ = ref.query(0, (r,), loc)
        ref.copied(0, loc, pairs)
        n += len(pairs)
    return n, ref


@pytest.mark.parametrize("shape", [(256, 192), (1000, 77), (4096, 513), (96, 3)])
@pytest.mark.parametrize("n", [0, 5])
def test_life_population_task(ctx, shape, n):
    w, h = shape
    g0 = mi.life_u8(mi.SEED_LIFE_8K + w, w, h)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(n)
        bins, moved = g.task_histogram(0)
    exp = oracle.histogram(oracle.life(g0, n, "wrap"))
    assert np.array_equal(bins, exp) and moved == 0
    assert bins[0] + bins[1] == w * h and bins[2:].sum() == 0


@pytest.mark.parametrize("boundary", ["clamp", "zero", "wrap"])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_conv_field_histogram_task(ctx, boundary, r):
    w, h = 333, 129
    f0 = mi.field_f32(mi.SEED_CONV5_FIELD + r, w, h)
    W = mi.weights_f32(mi.SEED_CONV5_W + r, r)
    with M.Grid(ctx, w, h, "conv", r, boundary, W) as g:
        g.bind(f0)
        g.iterate(3)
        bins, moved = g.task_histogram(0)
    exp = oracle.histogram_f32(oracle.conv(f0, W, 3, boundary))
    assert np.array_equal(bins, exp) and moved == 0


def test_f32_binning_edges(ctx):
    """Values at and around every bin edge, negatives, >= 1, -0.0, NaN, inf
    (reading h4); r = 1 conv with a centre tap of 1 leaves the field as is."""
    edges = np.arange(257, dtype=np.float32) / 256
    vals = np.concatenate([edges, np.nextafter(edges, np.float32(-1)), np.nextafter(edges, np.float32(2)),
                           np.array([-1, -0.0, 1.5, 1e30, -1e30, np.inf, -np.inf, np.nan], np.float32)])
    vals = np.resize(vals, 16 * 64).reshape(16, 64).astype(np.float32)
    W = np.zeros(9, np.float32)
    W[4] = 1
    with M.Grid(ctx, 64, 16, "conv", 1, "clamp", W) as g:
        g.bind(vals)
        bins, _ = g.task_histogram(0)
    assert np.array_equal(bins, oracle.histogram_f32(vals))


@pytest.mark.parametrize("G,T", [(4, 1), (4, 2), (4, 3), (4, 4), (3, 2), (2, 1), (8, 5)])
@pytest.mark.parametrize("kind", ["life", "conv", "histogram"])
def test_repartitioned_task_moves_what_alg2_infers(local_ctx, G, T, kind):
    w, h = (320, 203) if kind != "life" else (1000, 203)
    c = local_ctx(G)
    if kind == "life":
        data = mi.life_u8(77, w, h)
        grid = M.Grid(c, w, h, "life", 1, "wrap")
    elif kind == "conv":
        data = mi.field_f32(78, w, h)
        W = mi.weights_f32(79, 2)
        grid = M.Grid(c, w, h, "conv", 2, "zero", W)
    else:
        data = mi.image_u8(80, w, h, kind="skewed")
        grid = M.Grid(c, w, h, "histogram")
    with grid as g:
        g.bind(data)
        if kind != "histogram":
            g.iterate(2)
        pitch = g.info().pitch_bytes
        if kind == "life":
            exp = oracle.histogram(oracle.life(data, 2, "wrap"))
        elif kind == "conv":
            exp = oracle.histogram_f32(oracle.conv(data, W, 2, "zero"))
        else:
            exp = oracle.histogram(data)
        rows, ref = expected_moved_rows(h, G, T)
        bins, moved = g.task_histogram(T)
        assert np.array_equal(bins, exp)
        assert moved == rows * pitch
        bins2, moved2 = g.task_histogram(T)              # datum unmodified: all rows up to date
        assert np.array_equal(bins2, exp) and moved2 == 0
        if kind != "histogram":
            g.iterate(1)                                 # new version: the copies are stale
            if kind == "life":
                exp3 = oracle.histogram(oracle.life(data, 3, "wrap"))
            else:
                exp3 = oracle.histogram_f32(oracle.conv(data, W, 3, "zero"))
            bins3, moved3 = g.task_histogram(T)
            assert np.array_equal(bins3, exp3) and moved3 == rows * pitch
        same, moved4 = g.task_histogram(0)               # own partition never moves data
        assert moved4 == 0


def test_task_errors(ctx):
    with M.Grid(ctx, 128, 64, "life", 1, "wrap") as g:
        with pytest.raises(M.MapsmError) as e:
            g.task_histogram(0)
        assert e.value.status == M.ESTATE
        g.bind(mi.life_u8(1, 128, 64))
        with pytest.raises(M.MapsmError) as e:
            g.task_histogram(2)                          # more target slabs than slabs
        assert e.value.status == M.EINVAL
        out = np.zeros(255, np.uint64)
        assert M.lib().mapsm_task_histogram(g.handle, 0, out.ctypes.data, 255, None) == M.EINVAL


def test_life_task_at_scale(ctx):
    """32768^2 Life after 2 generations: the population task equals the count
    of the gathered grid (which the cone tests tie to the oracle)."""
    import torch

    w = h = 32768
    g0 = mi.life_u8(mi.SEED_LIFE_64K, w, h)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(2)
        bins, moved = g.task_histogram(0)
        out = torch.empty((h, w), dtype=torch.uint8, device="cuda")
        M.mapsm_read(g.handle, out)
        alive = int(out.sum(dtype=torch.int64).item())
    assert bins[1] == alive and bins[0] == w * h - alive and moved == 0


# ------------------------------------------------------------- GatherAsync

@pytest.mark.parametrize("G", [1, 3])
@pytest.mark.parametrize("kind", ["life", "conv"])
def test_gather_async(local_ctx, G, kind):
    import torch

    w, h = 640, 150
    c = local_ctx(G)
    if kind == "life":
        data = mi.life_u8(5, w, h)
        exp = oracle.life(data, 7, "clamp")
        grid = M.Grid(c, w, h, "life", 1, "clamp")
        host = torch.empty((h, w), dtype=torch.uint8).pin_memory()
    else:
        W = mi.weights_f32(6, 1)
        data = mi.field_f32(7, w, h)
        exp = oracle.conv(data, W, 7, "clamp")
        grid = M.Grid(c, w, h, "conv", 1, "clamp", W)
        host = torch.empty((h, w), dtype=torch.float32).pin_memory()
    with grid as g:
        g.bind(data)
        g.iterate(7)
        host.fill_(0)
        g.gather_async(host)
        g.sync()
        got = host.numpy()
        if kind == "life":
            assert np.array_equal(got, exp)
        else:
            assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))
        dev = torch.zeros((h, w), dtype=host.dtype, device="cuda")
        g.gather_async(dev)
        g.sync()
        assert np.array_equal(dev.cpu().numpy(), got)
