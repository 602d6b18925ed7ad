"""MAPSM_OPT_HOST_PACKED (include/mapsm.h): Life host rows in the device's
bit-packed format — w / 32 little-endian uint32 words per row, bit j of word
k = column 32k + j — through mapsm_bind / mapsm_read / mapsm_gather, against
the oracle on the u8 grid (np.packbits(..., bitorder="little") writes exactly
that layout)."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def pack(x):
    return np.ascontiguousarray(np.packbits(x != 0, axis=1, bitorder="little"))


def unpack(p, w):
    return np.unpackbits(p, axis=1, bitorder="little")[:, :w]


@pytest.mark.parametrize("w,h,n", [(4096, 300, 9), (65536, 128, 4), (96, 50, 7), (2048, 1, 3)])
@pytest.mark.parametrize("b", ["wrap", "clamp", "zero"])
def test_packed_bind_read_vs_oracle(ctx, w, h, n, b):
    x0 = mi.life_u8(9100 + w + h, w, h)
    with M.Grid(ctx, w, h, "life", 1, b) as g:
        g.set_option(M.OPT_HOST_PACKED, 1)
        g.bind(pack(x0))
        g.iterate(n)
        out = np.zeros((h, w // 8), dtype=np.uint8)
        g.read(out)
        gat = np.zeros((h, w // 8), dtype=np.uint8)
        g.gather(gat)
    exp = oracle.life(x0, n, b)
    assert np.array_equal(unpack(out, w), exp)
    assert np.array_equal(unpack(gat, w), exp)


def test_packed_pitched_rows_and_u8_equivalence(ctx):
    """A row pitch wider than w / 8 bytes, and the same grid through u8 rows."""
    w, h, n = 1024, 200, 6
    x0 = mi.life_u8(9200, w, h)
    wide = np.zeros((h, w // 8 + 40), dtype=np.uint8)
    wide[:, : w // 8] = pack(x0)
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.set_option(M.OPT_HOST_PACKED, 1)
        g.bind(wide)
        g.iterate(n)
        out = np.full((h, w // 8 + 24), 0xAB, dtype=np.uint8)
        g.read(out)
    assert np.all(out[:, w // 8:] == 0xAB)  # bytes past the row untouched
    with M.Grid(ctx, w, h, "life", 1, "wrap") as g:
        g.bind(x0)
        g.iterate(n)
        ref = g.gather()
    assert np.array_equal(unpack(out[:, : w // 8], w), ref)


@pytest.mark.parametrize("g_", [2, 3])
def test_packed_local_multislab(local_ctx, g_):
    w, h, n = 2048, 301, 5
    x0 = mi.life_u8(9300 + g_, w, h)
    with M.Grid(local_ctx(g_), w, h, "life", 1, "wrap") as g:
        g.set_option(M.OPT_HOST_PACKED, 1)
        g.bind(pack(x0))
        g.iterate(n)
        out = np.zeros((h, w // 8), dtype=np.uint8)
        g.gather(out)
    assert np.array_equal(unpack(out, w), oracle.life(x0, n, "wrap"))


def test_packed_device_buffers(ctx):
    import torch

    w, h, n = 4096, 256, 5
    x0 = mi.life_u8(9400, w, h)
    d_in = torch.from_numpy(pack(x0)).cuda()
    d_out = torch.zeros_like(d_in)
    with M.Grid(ctx, w, h, "life", 1, "zero") as g:
        g.set_option(M.OPT_HOST_PACKED, 1)
        g.bind(d_in)
        g.iterate(n)
        g.read(d_out)
        g.sync()
    assert np.array_equal(unpack(d_out.cpu().numpy(), w), oracle.life(x0, n, "zero"))


def test_packed_unsupported(ctx):
    with M.Grid(ctx, 100, 20, "life", 1, "wrap") as g:  # w % 32 != 0
        with pytest.raises(M.MapsmError):
            g.set_option(M.OPT_HOST_PACKED, 1)
    W = mi.weights_f32(1, 1)
    with M.Grid(ctx, 128, 20, "conv", 1, "wrap", W) as g:
        with pytest.raises(M.MapsmError):
            g.set_option(M.OPT_HOST_PACKED, 1)
