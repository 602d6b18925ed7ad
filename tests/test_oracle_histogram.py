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
