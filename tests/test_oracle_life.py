"""Pins for the Life oracle (oracle/oracle.c) against facts fixed outside it:
closed-form pattern behaviour (tests/golden), the scipy neighbour count, the
B3/S23 truth table, WRAP <-> tiled-ZERO brute force on tiny tori, and
symmetry invariants.  CPU only."""
import os

import numpy as np
import pytest
from scipy import ndimage

import mapsm_inputs as mi
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _load_patterns():
    pats, cur = [], None
    for line in open(os.path.join(GOLDEN, "life_patterns.txt")):
        line = line.rstrip("\n")
        if not line or line.startswith("#"):
            continue
        if line.startswith("pattern "):
            parts = line.split()
            cur = {"name": parts[1], "prop": parts[2], "args": [int(a) for a in parts[3:]], "rows": []}
            pats.append(cur)
        else:
            cur["rows"].append([1 if c == "O" else 0 for c in line])
    for p in pats:
        wmax = max(len(r) for r in p["rows"])
        p["cells"] = np.array([r + [0] * (wmax - len(r)) for r in p["rows"]], dtype=np.uint8)
    return pats


PATTERNS = _load_patterns()


def _embed(cells, h, w, y, x):
    g = np.zeros((h, w), dtype=np.uint8)
    ph, pw = cells.shape
    g[y:y + ph, x:x + pw] = cells
    return g


@pytest.mark.parametrize("pat", PATTERNS, ids=[p["name"] for p in PATTERNS])
@pytest.mark.parametrize("boundary", ["wrap", "zero", "clamp"])
def test_classic_patterns(pat, boundary):
    # Place the pattern away from the edges so the three boundary modes agree
    # with the unbounded plane for the generations checked.
    h, w = 96, 80
    g = _embed(pat["cells"], h, w, 40, 30)
    prop, args = pat["prop"], pat["args"]
    if prop == "still":
        assert np.array_equal(oracle.life(g, 1, boundary), g)
        assert np.array_equal(oracle.life(g, 7, boundary), g)
    elif prop == "period":
        P = args[0]
        assert np.array_equal(oracle.life(g, P, boundary), g)
        assert np.array_equal(oracle.life(g, 2 * P, boundary), g)
        for k in range(1, P):
            assert not np.array_equal(oracle.life(g, k, boundary), g), f"period divides {k}"
    elif prop == "translate":
        P, dy, dx = args
        out = oracle.life(g, P, boundary)
        assert np.array_equal(out, np.roll(g, (dy, dx), axis=(0, 1)))
        out3 = oracle.life(g, 3 * P, boundary)
        assert np.array_equal(out3, np.roll(g, (3 * dy, 3 * dx), axis=(0, 1)))
    elif prop == "vanish":
        N = args[0]
        assert oracle.life(g, N - 1, boundary).sum() > 0
        assert oracle.life(g, N, boundary).sum() == 0
    else:
        raise AssertionError(prop)


def test_config0_golden():
    """BASELINE.json configs[0]: 64x64 WRAP, 100 generations (closed form)."""
    exp = np.zeros((64, 64), dtype=np.uint8)
    for line in open(os.path.join(GOLDEN, "life_config0_gen100.txt")):
        if line.strip() and not line.startswith("#"):
            y, x = map(int, line.split())
            exp[y, x] = 1
    out = oracle.life(mi.config0_grid(), 100, "wrap")
    assert out.sum() == 12
    assert np.array_equal(out, exp)


def test_glider_crosses_both_wrap_edges():
    g = _embed(np.array([[0, 1, 0], [0, 0, 1], [1, 1, 1]], np.uint8), 16, 24, 13, 21)  # straddles nothing yet
    for k in range(1, 20):
        out = oracle.life(g, 4 * k, "wrap")
        assert np.array_equal(out, np.roll(g, (k, k), axis=(0, 1)))


def test_truth_table_all_512_neighbourhoods():
    """B3/S23 on every 3x3 neighbourhood (reading c1): centre of a 3x3 ZERO grid."""
    for m in range(512):
        bits = np.array([(m >> i) & 1 for i in range(9)], dtype=np.uint8).reshape(3, 3)
        alive = bits[1, 1]
        nb = int(bits.sum()) - int(alive)
        expect = 1 if (nb == 3 or (alive and nb == 2)) else 0
        assert oracle.life(bits, 1, "zero")[1, 1] == expect, m


_SCIPY_MODE = {"wrap": "wrap", "clamp": "nearest", "zero": "constant"}


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
@pytest.mark.parametrize("shape", [(1, 1), (2, 3), (5, 7), (31, 17), (64, 64), (3, 100)])
def test_one_step_vs_scipy_neighbour_count(boundary, shape):
    """Neighbour sum from scipy.ndimage.correlate (library routine), modes
    wrap/nearest/constant = WRAP/CLAMP/ZERO (reading c4)."""
    h, w = shape
    rng = np.random.default_rng(h * 1000 + w)
    g = (rng.random((h, w)) < 0.4).astype(np.uint8)
    k = np.ones((3, 3), dtype=np.int64)
    k[1, 1] = 0
    n = ndimage.correlate(g.astype(np.int64), k, mode=_SCIPY_MODE[boundary], cval=0)
    expect = ((n == 3) | ((g == 1) & (n == 2))).astype(np.uint8)
    assert np.array_equal(oracle.life(g, 1, boundary), expect)


def test_tiny_tori_vs_tiled_zero_grid():
    """Brute force: a 4x4 WRAP torus step equals the centre tile of the state
    tiled 3x3 on a ZERO-bounded 12x12 grid (mod vs in-range lookups)."""
    rng = np.random.default_rng(4)
    states = list(range(0, 1 << 16, 37)) + [0, 0xFFFF, 0x0F0F, 0x8421]
    for s in states:
        t = np.array([(s >> i) & 1 for i in range(16)], np.uint8).reshape(4, 4)
        tor = oracle.life(t, 1, "wrap")
        big = oracle.life(np.tile(t, (3, 3)), 1, "zero")
        assert np.array_equal(tor, big[4:8, 4:8]), s
    del rng


def test_degenerate_tiny_wrap_multiplicity():
    """Reading c5: with w or h < 3 under WRAP neighbours repeat with multiplicity."""
    g = np.array([[1]], np.uint8)  # the cell is its own 8 neighbours: N=8 -> dies
    assert oracle.life(g, 1, "wrap")[0, 0] == 0
    # 1x2 torus [1,0]: (0,0) sees (0,0) twice (dy=+-1) and (0,1) 6 times -> N=2 -> survives;
    # (0,1) sees (0,0) 6 times and itself twice -> N=6 -> stays dead.
    g = np.array([[1, 0]], np.uint8)
    assert np.array_equal(oracle.life(g, 1, "wrap"), np.array([[1, 0]], np.uint8))


@pytest.mark.parametrize("boundary", ["wrap", "clamp", "zero"])
def test_d4_equivariance(boundary):
    rng = np.random.default_rng(7)
    g = (rng.random((23, 41)) < 0.5).astype(np.uint8)
    out = oracle.life(g, 5, boundary)
    assert np.array_equal(oracle.life(g.T.copy(), 5, boundary), out.T)
    assert np.array_equal(oracle.life(g[::-1].copy(), 5, boundary), out[::-1])
    assert np.array_equal(oracle.life(g[:, ::-1].copy(), 5, boundary), out[:, ::-1])


def test_roll_equivariance_wrap():
    rng = np.random.default_rng(8)
    g = (rng.random((37, 29)) < 0.5).astype(np.uint8)
    out = oracle.life(g, 6, "wrap")
    for s in [(1, 0), (0, 1), (5, -7), (36, 28)]:
        assert np.array_equal(oracle.life(np.roll(g, s, (0, 1)), 6, "wrap"), np.roll(out, s, (0, 1)))


def test_n0_returns_normalised_input():
    g = np.array([[0, 3, 255], [1, 0, 7]], np.uint8)
    assert np.array_equal(oracle.life(g, 0, "wrap"), (g != 0).astype(np.uint8))


def test_per_side_modes_cut_patch_matches_full_grid():
    """The per-side interface used for sampled cones: a patch with ZERO on cut
    sides reproduces the full-grid result at distance >= n from the cut."""
    rng = np.random.default_rng(9)
    g = (rng.random((60, 70)) < 0.5).astype(np.uint8)
    n = 6
    full = oracle.life(g, n, "clamp")
    patch = g[0:30, 20:50]  # top edge real (CLAMP), other three sides cut
    out = oracle.life(patch, n, sides=("clamp", "zero", "zero", "zero"))
    assert np.array_equal(out[0:30 - n, n:30 - n], full[0:30 - n, 20 + n:50 - n])


def test_rejects_bad_modes():
    g = np.zeros((4, 4), np.uint8)
    with pytest.raises(ValueError):
        oracle.life(g, 1, sides=("wrap", "zero", "wrap", "wrap"))
