"""Pins for the histogram oracle (Reductive-Static output pattern, P:L104,
Fig 4): numpy.bincount (library routine), closed forms and
invariants.  CPU only."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle


@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (64, 64), (100, 257), (513, 31)])
@pytest.mark.parametrize("kind", ["uniform", "skewed"])
def test_vs_bincount(shape, kind):
    h, w = shape
    img = mi.image_u8(17 + h, w, h, kind=kind)
    exp = np.bincount(img.ravel(), minlength=256).astype(np.uint64)
    assert np.array_equal(oracle.histogram(img), exp)


def test_constant_and_ramp_closed_forms():
    for v in (0, 1, 127, 255):
        img = np.full((37, 41), v, np.uint8)
        hst = oracle.histogram(img)
        assert hst[v] == 37 * 41 and hst.sum() == 37 * 41
    ramp = (np.arange(512)[None, :] % 256).astype(np.uint8).repeat(9, axis=0)
    assert np.all(oracle.histogram(ramp) == 9 * 2)


def test_pitch_padding_not_counted():
    big = np.full((10, 64), 200, np.uint8)
    big[:, :50] = 7
    view = big[:, :50]
    hst = oracle.histogram(view)
    assert hst[7] == 500 and hst[200] == 0


def test_invariants():
    img = mi.image_u8(5, 300, 200)
    hst = oracle.histogram(img)
    assert int(hst.sum()) == 300 * 200
    rng = np.random.default_rng(0)
    perm = rng.permutation(img.ravel()).reshape(img.shape)
    assert np.array_equal(oracle.histogram(perm), hst)
    # additivity over row slabs (the multi-GPU duplicate-and-aggregate)
    parts = [oracle.histogram(np.ascontiguousarray(img[a:b])) for a, b in [(0, 13), (13, 100), (100, 200)]]
    assert np.array_equal(sum(parts), hst)


def test_generators():
    u = mi.image_u8(mi.SEED_HIST_UNIFORM, 512, 512)
    s = mi.image_u8(mi.SEED_HIST_SKEWED, 512, 512, kind="skewed")
    hu, hs = oracle.histogram(u), oracle.histogram(s)
    assert hu.min() > 0 and hu.max() < 3 * hu.mean()
    assert hs.argmax() in range(100, 156) and hs[:30].sum() < 0.01 * hs.sum() and hs.max() > 2 * hu.max()


# ---- fp32-field histogram task (reading h4) ----

def test_f32_histogram_closed_forms():
    """bin = floor(v * 256) on [0, 1): every bin edge k/256 lands in bin k,
    the float just below it in bin k-1; < 0, -0.0 and NaN -> 0; >= 1 -> 255."""
    k = np.arange(256)
    edges = (k / 256).astype(np.float32)[None, :]
    out = oracle.histogram_f32(edges)
    assert np.array_equal(out, np.ones(256, np.uint64))
    below = np.nextafter(edges[:, 1:], np.float32(-1))
    out = oracle.histogram_f32(below)
    assert np.array_equal(out[:255], np.ones(255, np.uint64)) and out[255] == 0
    special = np.array([[-1.0, -0.0, np.nan, -np.inf, 1.0, 7.5, np.inf, 0.99999994]], np.float32)
    out = oracle.histogram_f32(special)
    assert out[0] == 4 and out[255] == 4 and out.sum() == 8


def test_f32_histogram_vs_numpy_binning():
    """Against numpy's floor/clip on a random field in [-0.1, 1.1)."""
    rng = np.random.default_rng(5)
    f = (rng.random((37, 101)) * 1.2 - 0.1).astype(np.float32)
    b = np.clip(np.floor(f.astype(np.float64) * 256), 0, 255).astype(np.int64)
    assert np.array_equal(oracle.histogram_f32(f), np.bincount(b.ravel(), minlength=256).astype(np.uint64))
