"""The 3-D light-cone helper (tests/cones.py) against the full-volume oracle:
cut-out evaluation must reproduce every sampled block exactly.  CPU only."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from cones import cone_eval3d


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r,n", [(1, 3), (2, 2)])
def test_cone3d_matches_full_oracle(boundary, r, n):
    d, h, w = 14, 13, 17
    seed = 91
    vol = mi.volume_f32(seed, w, h, d)
    W = mi.weights3d_f32(92, r)
    full = oracle.conv3d(vol, W, n, boundary)

    def vol_rows(z, y0, nr):
        return mi.field_f32(seed, w, nr, y0=z * h + y0)

    for zr, yr, xr in [((0, 2), (0, 3), (0, 4)), ((6, 8), (5, 7), (7, 10)), ((12, 14), (11, 13), (14, 17)),
                       ((0, 14), (4, 6), (3, 5))]:
        got = cone_eval3d(vol_rows, d, h, w, r, n, boundary, zr, yr, xr, W)
        exp = full[zr[0]:zr[1], yr[0]:yr[1], xr[0]:xr[1]]
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), (zr, yr, xr)
