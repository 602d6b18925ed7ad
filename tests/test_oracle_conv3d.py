"""Pins for the Window(3D) fp32 convolution oracle (oracle.conv3d; P:L526,
Table 1; reading v1).

- exact-rational simulation of the fixed (dz, dy, dx) fmaf chain with explicit
  round-to-nearest-even to binary32: bit-exact on small volumes;
- scipy.ndimage.correlate in 3-D (library routine, float64; modes wrap /
  nearest / constant = WRAP / CLAMP / ZERO) within the fp32 rounding bound;
- closed forms: single tap == np.roll (orientation, no flip); weights only on
  the dz = 0 plane == the (separately pinned) 2-D oracle on every plane,
  bit for bit; centre tap identity;
- invariant: mass conservation under WRAP.
CPU only."""
from fractions import Fraction

import numpy as np
import pytest
from scipy import ndimage

import mapsm_inputs as mi
import oracle
from test_oracle_conv import fmaf_exact

_SCIPY_MODE = {"wrap": "wrap", "clamp": "nearest", "zero": "constant"}


def _cell3(v, z, y, x, b):
    d, h, w = v.shape
    if b == "wrap":
        return v[z % d, y % h, x % w]
    if b == "clamp":
        return v[min(max(z, 0), d - 1), min(max(y, 0), h - 1), min(max(x, 0), w - 1)]
    return v[z, y, x] if (0 <= z < d and 0 <= y < h and 0 <= x < w) else np.float32(0)


def conv3_exact(v, W, n, b):
    r = W.shape[0] // 2
    d, h, w = v.shape
    cur = v.astype(np.float32)
    for _ in range(n):
        nxt = np.empty_like(cur)
        for z in range(d):
            for y in range(h):
                for x in range(w):
                    acc = Fraction(0)
                    for dz in range(-r, r + 1):
                        for dy in range(-r, r + 1):
                            for dx in range(-r, r + 1):
                                acc = fmaf_exact(float(W[dz + r, dy + r, dx + r]),
                                                 float(_cell3(cur, z + dz, y + dy, x + dx, b)), acc)
                    nxt[z, y, x] = np.float32(float(acc))
        cur = nxt
    return cur


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r,shape,n", [(1, (3, 4, 5), 2), (1, (2, 3, 7), 1), (2, (3, 5, 4), 1)])
def test_fixed_order_chain_bit_exact(boundary, r, shape, n):
    d, h, w = shape
    v = mi.volume_f32(11 + r, w, h, d)
    W = mi.weights3d_f32(12 + r, r)
    got = oracle.conv3d(v, W, n, boundary)
    exp = conv3_exact(v, W, n, boundary)
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))


def test_dz_order_matters_case_is_detected():
    """Reversing the dz order changes the fp32 result on this input, so the
    chain test above really pins the (dz, dy, dx) order."""
    v = mi.volume_f32(21, 5, 4, 3)
    W = mi.weights3d_f32(22, 1)
    fwd = conv3_exact(v, W, 1, "wrap")
    rev = conv3_exact(v[::-1].copy(), W[::-1].copy(), 1, "wrap")[::-1]
    assert not np.array_equal(fwd.view(np.uint32), rev.view(np.uint32))
    assert np.array_equal(oracle.conv3d(v, W, 1, "wrap").view(np.uint32), fwd.view(np.uint32))


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r", [1, 2])
def test_vs_scipy_within_rounding_bound(boundary, r):
    n = 4
    v = mi.volume_f32(31, 13, 9, 7)
    W = mi.weights3d_f32(32, r)
    cur = v.astype(np.float64)
    for _ in range(n):
        cur = ndimage.correlate(cur, W.astype(np.float64), mode=_SCIPY_MODE[boundary], cval=0.0)
    got = oracle.conv3d(v, W, n, boundary)
    bound = n * (2 * r + 1) ** 3 * 2.0 ** -24 * max(1.0, np.abs(cur).max())
    err = np.max(np.abs(got.astype(np.float64) - cur))
    assert 0 < err <= bound


@pytest.mark.parametrize("dz,dy,dx", [(1, 0, 0), (-1, 1, 0), (0, -1, 1), (1, 1, -1), (-2, 2, 1)])
def test_single_tap_is_roll(dz, dy, dx):
    r = 2
    v = mi.volume_f32(41, 7, 6, 5)
    W = np.zeros((5, 5, 5), np.float32)
    W[dz + r, dy + r, dx + r] = 1
    got = oracle.conv3d(v, W, 1, "wrap")
    assert np.array_equal(got, np.roll(v, (-dz, -dy, -dx), axis=(0, 1, 2)))


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_planar_weights_equal_2d_oracle(boundary):
    """Weights only on the dz = 0 plane: every plane evolves by the 2-D
    oracle with those weights, bit for bit (the zero taps add +0 to a
    non-negative accumulator)."""
    r = 2
    v = mi.volume_f32(51, 19, 11, 4)
    W2 = mi.weights_f32(52, r)
    W = np.zeros((5, 5, 5), np.float32)
    W[r] = W2
    got = oracle.conv3d(v, W, 3, boundary)
    for z in range(v.shape[0]):
        exp = oracle.conv(v[z], W2, 3, boundary)
        assert np.array_equal(got[z].view(np.uint32), exp.view(np.uint32))


def test_zero_and_clamp_edges_single_tap():
    v = mi.volume_f32(61, 4, 3, 3)
    W = np.zeros((3, 3, 3), np.float32)
    W[2, 1, 1] = 1          # reads plane z + 1
    z = oracle.conv3d(v, W, 1, "zero")
    assert np.array_equal(z[:-1], v[1:]) and not z[-1].any()
    c = oracle.conv3d(v, W, 1, "clamp")
    assert np.array_equal(c[:-1], v[1:]) and np.array_equal(c[-1], v[-1])


def test_mass_conservation_wrap():
    v = mi.volume_f32(71, 8, 6, 5)
    W = mi.weights3d_f32(72, 1)
    got = oracle.conv3d(v, W, 10, "wrap").astype(np.float64)
    s = float(W.astype(np.float64).sum())
    assert abs(got.sum() - v.astype(np.float64).sum() * s ** 10) <= 1e-4 * v.size
