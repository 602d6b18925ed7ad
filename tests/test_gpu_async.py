"""Asynchronous Bind / read and per-grid streams (mapsm_bind_async,
mapsm_read_async, MAPSM_OPT_OWN_STREAM): several grids of one ctx pipelined
(one grid's upload, another's generations and a third's download in flight
together — the bench's e2e mode), every result bit-exact vs the oracle."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("op,b", [("life", "wrap"), ("life", "zero"), ("conv", "clamp")])
def test_pipelined_grids_own_streams(ctx, op, b):
    import torch

    w, h, n, G, steps = 1024, 300, 9, 3, 7
    r = 1 if op == "life" else 4
    W = mi.weights_f32(31, r) if op == "conv" else None
    dt = torch.uint8 if op == "life" else torch.float32
    inputs = []
    for k in range(steps):
        a = mi.life_u8(100 + k, w, h) if op == "life" else mi.field_f32(100 + k, w, h)
        inputs.append(torch.from_numpy(a).pin_memory())
    outs = [torch.empty((h, w), dtype=dt).pin_memory() for _ in range(steps)]
    grids = [M.Grid(ctx, w, h, op, r, b, W) for _ in range(G)]
    try:
        for g in grids:
            g.set_option(M.OPT_OWN_STREAM, 1)
        streams = {M.mapsm_grid_stream(g.handle) for g in grids}
        assert len(streams) == G  # private streams
        for k in range(steps):
            g = grids[k % G]  # stream order: after this grid's previous step (no host wait)
            M.mapsm_bind_async(g.handle, inputs[k])
            g.iterate(n)
            M.mapsm_read_async(g.handle, outs[k])
        for g in grids:
            g.sync()
    finally:
        for g in grids:
            g.close()
    for k in range(steps):
        exp = oracle.life(inputs[k].numpy(), n, b) if op == "life" else oracle.conv(inputs[k].numpy(), W, n, b)
        assert np.array_equal(outs[k].numpy().view(np.uint8), exp.view(np.uint8)), k


@pytest.mark.parametrize("g", [2, 4])
def test_async_bind_local_slabs_exchange(local_ctx, g):
    """The first halo exchange after an asynchronous Bind is stream-ordered."""
    import torch

    w, h, n = 512, 8 * g + 3, 6
    g0 = torch.from_numpy(mi.life_u8(7 + g, w, h)).pin_memory()
    out = torch.empty_like(g0).pin_memory()
    with M.Grid(local_ctx(g), w, h, "life", 1, "wrap") as gr:
        M.mapsm_bind_async(gr.handle, g0)
        gr.iterate(n)
        M.mapsm_read_async(gr.handle, out)
        gr.sync()
    assert np.array_equal(out.numpy(), oracle.life(g0.numpy(), n, "wrap"))


def test_own_stream_after_allocation_and_rebind(ctx):
    """Switching an allocated grid to a private stream, rebinding (weights of a
    slot-based radius uploaded once), results unchanged."""
    f0 = mi.field_f32(3, 256, 64)
    W = mi.weights_f32(4, 3)
    with M.Grid(ctx, 256, 64, "conv", 3, "zero", W) as g:
        g.bind(f0)
        g.set_option(M.OPT_OWN_STREAM, 1)
        g.iterate(2)
        a = g.gather()
        g.bind(f0)
        g.iterate(2)
        b2 = g.gather()
    exp = oracle.conv(f0, W, 2, "zero")
    assert np.array_equal(a.view(np.uint32), exp.view(np.uint32))
    assert np.array_equal(b2.view(np.uint32), exp.view(np.uint32))
