"""GPU parity: the Reductive-Static 256-bin histogram (SURVEY §8(f) NEXT-1,
Fig 4) through the C ABI vs the CPU oracle — bit-exact counts."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def run(ctx, img):
    h, w = img.shape
    with M.Grid(ctx, w, h, "histogram") as g:
        g.bind(img)
        out = g.histogram()
        info = g.info()
    return out, info


@pytest.mark.parametrize("shape", [(1, 1), (1, 15), (3, 16), (7, 17), (64, 64), (100, 1000), (513, 4099),
                                   (2048, 2048)])
@pytest.mark.parametrize("kind", ["uniform", "skewed"])
def test_vs_oracle(ctx, shape, kind):
    h, w = shape
    img = mi.image_u8(101 + w, w, h, kind=kind)
    out, info = run(ctx, img)
    assert np.array_equal(out, oracle.histogram(img))
    assert int(out.sum()) == w * h


def test_constant_image_all_one_bin(ctx):
    img = np.full((333, 1024), 77, np.uint8)
    out, _ = run(ctx, img)
    assert out[77] == 333 * 1024 and out.sum() == 333 * 1024


@pytest.mark.parametrize("g", [2, 3, 8])
def test_local_multislab_aggregation(local_ctx, g):
    img = mi.image_u8(55, 1000, 123, kind="skewed")
    out, info = run(local_ctx(g), img)
    assert np.array_equal(out, oracle.histogram(img))
    assert info.world == g


def test_device_output_and_rebind(ctx):
    import torch

    a = mi.image_u8(1, 512, 256)
    b = mi.image_u8(2, 512, 256, kind="skewed")
    with M.Grid(ctx, 512, 256, "histogram") as g:
        g.bind(a)
        d = torch.zeros(256, dtype=torch.int64, device="cuda")
        M.mapsm_histogram(g.handle, d)
        torch.cuda.synchronize()
        assert np.array_equal(d.cpu().numpy().astype(np.uint64), oracle.histogram(a))
        g.bind(torch.from_numpy(b).cuda())
        assert np.array_equal(g.histogram(), oracle.histogram(b))


def test_state_errors(ctx):
    with M.Grid(ctx, 256, 16, "histogram") as g:
        with pytest.raises(M.MapsmError) as e:
            g.histogram()
        assert e.value.status == M.ESTATE
        g.bind(np.zeros((16, 256), np.uint8))
        with pytest.raises(M.MapsmError) as e:
            g.iterate(1)
        assert e.value.status == M.EUNSUPPORTED
    with M.Grid(ctx, 256, 16, "life") as g:
        g.bind(np.zeros((16, 256), np.uint8))
        with pytest.raises(M.MapsmError) as e:
            g.histogram()
        assert e.value.status == M.ESTATE


def test_paper_size_8k_uniform(ctx):
    """The paper's workload: 256 bins on an 8K square image."""
    img = mi.image_u8(mi.SEED_HIST_UNIFORM, 8192, 8192)
    out, _ = run(ctx, img)
    assert np.array_equal(out, oracle.histogram(img))


@pytest.mark.parametrize("nslabs", [1, 3])
def test_device_bins_stream_ordered(local_ctx, nslabs):
    """Device-memory bins: the call is stream-ordered (include/mapsm.h); after
    mapsm_sync the counts are exact, and back-to-back calls on a rebound image
    each see their own image (the per-slab bins are re-zeroed in stream order)."""
    import torch

    imgs = [mi.image_u8(900 + k, 4096, 777, kind="uniform" if k % 2 else "skewed") for k in range(3)]
    with M.Grid(local_ctx(nslabs), 4096, 777, "histogram") as g:
        outs = []
        for img in imgs:
            g.bind(img)
            d = torch.full((256,), -1, dtype=torch.int64, device="cuda")
            torch.cuda.synchronize()  # the grid runs on its own stream
            M.mapsm_histogram(g.handle, d)
            g.sync()
            outs.append(d.cpu().numpy().astype(np.uint64))
        for img, out in zip(imgs, outs):
            assert np.array_equal(out, oracle.histogram(img))
        # repeated calls without a host sync in between: the last one must be exact
        d = torch.zeros(256, dtype=torch.int64, device="cuda")
        torch.cuda.synchronize()
        for _ in range(5):
            M.mapsm_histogram(g.handle, d)
        g.sync()
        assert np.array_equal(d.cpu().numpy().astype(np.uint64), oracle.histogram(imgs[-1]))
