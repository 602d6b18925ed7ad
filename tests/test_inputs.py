"""The shared seeded-input module (no method arithmetic): recipe checks."""
import numpy as np

import mapsm_inputs as mi


def test_splitmix64_published_vector():
    # splitmix64 seeded with 0: first output 0xE220A8397B1DCDAF (Vigna's reference generator).
    assert mi.splitmix64(0) == 0xE220A8397B1DCDAF


def test_life_rows_are_global_and_sliceable():
    full = mi.life_u8(0x5EED0002, 256, 64)
    part = mi.life_u8(0x5EED0002, 256, 10, y0=20)
    assert np.array_equal(full[20:30], part)
    assert set(np.unique(full)) <= {0, 1}
    assert 0.45 < full.mean() < 0.55
    assert full[3, 7] == mi.splitmix64(0x5EED0002 + 3 * 256 + 7) >> 63


def test_field_recipe_exact():
    f = mi.field_f32(0x5EED0004, 33, 5, y0=2)
    v = mi.splitmix64(0x5EED0004 + (2 + 1) * 33 + 4)
    assert f[1, 4] == np.float32((v >> 40) * 2.0 ** -24)
    assert f.min() >= 0 and f.max() < 1


def test_config0_population():
    assert mi.config0_grid().sum() == 12
