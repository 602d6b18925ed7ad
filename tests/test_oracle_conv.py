"""Pins for the fp32 / fp64 window-convolution oracle (oracle/oracle.c).

- exact-rational simulation of the fixed-order fmaf chain (reading c11) with
  explicit round-to-nearest-even to binary32: bit-exact on small grids;
- scipy.ndimage.correlate in float64 (library routine, modes wrap / nearest /
  constant = WRAP / CLAMP / ZERO, reading c4) against the fp64 oracle;
- closed forms: centre-tap identity, single-tap shift == np.roll (fixes the
  no-flip orientation, reading c9);
- invariant: mass conservation under WRAP (sum-1 weights), fp32 within the
  rounding bound of the fp64 result.
CPU only."""
from fractions import Fraction

import numpy as np
import pytest
from scipy import ndimage

import mapsm_inputs as mi
import oracle

_SCIPY_MODE = {"wrap": "wrap", "clamp": "nearest", "zero": "constant"}


def round_f32(q: Fraction) -> Fraction:
    """Round an exact rational to the nearest binary32 (ties to even)."""
    if q == 0:
        return Fraction(0)
    s = -1 if q < 0 else 1
    a = abs(q)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    while Fraction(2) ** (e + 1) <= a:
        e += 1
    e = max(e, -126)  # subnormals share the minimum exponent
    ulp = Fraction(2) ** (e - 23)
    m = round(a / ulp)  # Fraction.__round__ is round-half-even
    return s * m * ulp


def fmaf_exact(a, b, c) -> Fraction:
    return round_f32(Fraction(a) * Fraction(b) + Fraction(c))


def _cell(g, y, x, b):
    h, w = g.shape
    if b == "wrap":
        return g[y % h, x % w]
    if b == "clamp":
        return g[min(max(y, 0), h - 1), min(max(x, 0), w - 1)]
    return g[y, x] if (0 <= y < h and 0 <= x < w) else np.float32(0)


def conv_exact_fixed_order(g, W, n, b):
    r = W.shape[0] // 2
    h, w = g.shape
    cur = g.astype(np.float32)
    for _ in range(n):
        nxt = np.empty_like(cur)
        for y in range(h):
            for x in range(w):
                acc = Fraction(0)
                for dy in range(-r, r + 1):
                    for dx in range(-r, r + 1):
                        acc = fmaf_exact(float(W[dy + r, dx + r]), float(_cell(cur, y + dy, x + dx, b)), acc)
                nxt[y, x] = np.float32(float(acc))
        cur = nxt
    return cur


def test_round_f32_matches_numpy_on_doubles():
    rng = np.random.default_rng(0)
    for v in rng.standard_normal(2000) * 10.0 ** rng.integers(-30, 30, 2000):
        assert float(round_f32(Fraction(float(v)))) == float(np.float32(v))


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r,shape,n", [(1, (4, 5), 2), (2, (5, 6), 1), (1, (1, 3), 2), (3, (3, 4), 1)])
def test_fixed_order_fma_chain_bit_exact(boundary, r, shape, n):
    h, w = shape
    g = mi.field_f32(11 + r, w, h)
    W = mi.weights_f32(21 + r, r)
    exp = conv_exact_fixed_order(g, W, n, boundary)
    got = oracle.conv(g, W, n, boundary)
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))


def test_order_matters_case_is_detected():
    """A case where summation order changes the fp32 result, so the pin above
    really fixes the order: reversing the taps gives a different answer."""
    rng = np.random.default_rng(3)
    g = rng.random((6, 6)).astype(np.float32) * np.float32(1e3)
    W = (rng.random((3, 3)) * np.array([[1e-3, 1, 1e3]] * 3)).astype(np.float32)
    fwd = conv_exact_fixed_order(g, W, 1, "wrap")
    rev = conv_exact_fixed_order(g[::-1, ::-1].copy(), W[::-1, ::-1].copy(), 1, "wrap")[::-1, ::-1]
    assert not np.array_equal(fwd, rev)
    assert np.array_equal(oracle.conv(g, W, 1, "wrap"), fwd)


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_f64_vs_scipy_correlate(boundary, r):
    h, w = 37, 53
    g = mi.field_f32(5, w, h)
    W = mi.weights_f32(6, r)
    cur = g.astype(np.float64)
    for _ in range(3):
        cur = ndimage.correlate(cur, W.astype(np.float64), mode=_SCIPY_MODE[boundary], cval=0.0)
    got = oracle.conv_f64(g, W, 3, boundary)
    assert np.max(np.abs(got - cur)) <= 1e-13


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_f32_vs_scipy_within_rounding_bound(boundary):
    r, n = 2, 20
    g = mi.field_f32(7, 40, 30)
    W = mi.weights_f32(8, r)
    cur = g.astype(np.float64)
    for _ in range(n):
        cur = ndimage.correlate(cur, W.astype(np.float64), mode=_SCIPY_MODE[boundary], cval=0.0)
    got = oracle.conv(g, W, n, boundary)
    bound = n * (2 * r + 1) ** 2 * 2.0 ** -24 * max(1.0, np.abs(cur).max())
    err = np.max(np.abs(got - cur))
    assert err <= bound
    assert err > 0  # fp32 really is fp32


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_centre_tap_identity(boundary):
    g = mi.field_f32(9, 17, 13)
    W = np.zeros((5, 5), np.float32)
    W[2, 2] = 1.0
    assert np.array_equal(oracle.conv(g, W, 4, boundary), g)


@pytest.mark.parametrize("dy,dx", [(-2, 0), (0, 2), (1, -1), (2, 2), (-1, 2)])
def test_single_tap_is_roll_under_wrap(dy, dx):
    """out[y][x] = in[y+dy][x+dx]  <=>  np.roll(in, (-dy,-dx)) — fixes orientation."""
    g = mi.field_f32(10, 19, 11)
    W = np.zeros((5, 5), np.float32)
    W[dy + 2, dx + 2] = 1.0
    assert np.array_equal(oracle.conv(g, W, 1, "wrap"), np.roll(g, (-dy, -dx), axis=(0, 1)))
    assert np.array_equal(oracle.conv(g, W, 3, "wrap"), np.roll(g, (-3 * dy, -3 * dx), axis=(0, 1)))


def test_single_tap_zero_and_clamp_edges():
    g = mi.field_f32(12, 8, 6)
    W = np.zeros((3, 3), np.float32)
    W[0, 2] = 1.0  # out[y][x] = in[y-1][x+1]
    z = oracle.conv(g, W, 1, "zero")
    assert np.all(z[0, :] == 0) and np.all(z[:, -1] == 0)
    assert np.array_equal(z[1:, :-1], g[:-1, 1:])
    c = oracle.conv(g, W, 1, "clamp")
    assert np.array_equal(c[0, :-1], g[0, 1:]) and np.array_equal(c[1:, -1], g[:-1, -1])


def test_mass_conservation_wrap_f64():
    r, n = 4, 10
    g = mi.field_f32(13, 48, 40)
    W = mi.weights_f32(14, r)
    s_w = float(W.astype(np.float64).sum())
    got = oracle.conv_f64(g, W, n, "wrap")
    assert abs(got.sum() - g.astype(np.float64).sum() * s_w ** n) <= 1e-9 * got.sum()


def test_dyadic_inputs_are_exact():
    """Dyadic weights and coarse fields: every fp32 op is exact, so fp32 == fp64."""
    rng = np.random.default_rng(15)
    W = (rng.integers(0, 8, (5, 5)) / 64.0).astype(np.float32)
    g = (rng.integers(0, 16, (12, 14)) / 16.0).astype(np.float32)
    assert np.array_equal(oracle.conv(g, W, 2, "clamp").astype(np.float64), oracle.conv_f64(g, W, 2, "clamp"))


def test_weights_generator_recipe():
    for r in (1, 2, 3, 4):
        W = mi.weights_f32(0x5EED0044, r)
        assert W.shape == (2 * r + 1, 2 * r + 1) and W.min() > 0
        assert abs(W.astype(np.float64).sum() - 1.0) < (2 * r + 1) ** 2 * 2.0 ** -24
        assert not np.array_equal(W, W.T) and not np.array_equal(W, W[::-1, ::-1])
