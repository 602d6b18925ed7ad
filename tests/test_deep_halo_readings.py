"""CPU checks of the two facts the deep-halo Life kernel (life_tb.cu) rests on,
evaluated with the pinned oracle only (no GPU):

* CLAMP is the MIRROR extension: evolving a grid padded by its own mirror
  image (row -1-i := row i, column -1-i := column i) for K generations gives,
  on the original region, exactly K CLAMP generations — so the kernel may read
  mirrored input rows and bit-reversed edge words instead of applying CLAMP
  at every generation.
* WRAP is the periodic extension (the kernel reads rows mod h).
Both: the K-cell pad is the trapezoid of a K-generation pass."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle


@pytest.mark.parametrize("K", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("shape", [(8, 64), (17, 40), (33, 9)])
def test_clamp_equals_mirror_extension(K, shape):
    h, w = shape
    g0 = mi.life_u8(77 + K + h, w, h)
    ext = np.pad(g0, K, mode="symmetric")  # mirror, edge cell repeated: col -1 = col 0
    out = oracle.life(ext, K, "zero")[K:K + h, K:K + w]
    assert np.array_equal(out, oracle.life(g0, K, "clamp"))


@pytest.mark.parametrize("K", [1, 4, 8])
def test_wrap_equals_periodic_extension(K):
    g0 = mi.life_u8(5 + K, 48, 20)
    ext = np.pad(g0, K, mode="wrap")
    out = oracle.life(ext, K, "zero")[K:K + 20, K:K + 48]
    assert np.array_equal(out, oracle.life(g0, K, "wrap"))


def test_zero_is_not_an_extension():
    """ZERO has no such extension (zero cells next to live ones give births),
    which is why the kernel forces rows/columns outside the grid back to 0 at
    every generation: a zero pad evolved freely differs from K ZERO steps."""
    g0 = np.zeros((12, 12), np.uint8)
    g0[0, 4:7] = 1  # a blinker on the top edge: it would grow upwards
    K = 2
    ext = np.pad(g0, K)
    free = oracle.life(ext, K, "zero")[K:K + 12, K:K + 12]
    assert not np.array_equal(free, oracle.life(g0, K, "zero"))
