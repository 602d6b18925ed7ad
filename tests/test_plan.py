"""Partition + halo plan (plan.cpp through the C ABI, no GPU): the
Segmenter / Memory Analyzer / static Location Monitor of P:L59, P:L161-169,
Alg 2, checked against their definitions."""
import itertools

import pytest

from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

BOUNDS = [M.WRAP, M.CLAMP, M.ZERO]


def plans(h, g, r, b):
    return [M.mapsm_plan_query(h, g, r, b, k) for k in range(g)]


def owner(ps, row):
    for k, p in enumerate(ps):
        if p.y0 <= row < p.y0 + p.rows:
            return k
    raise AssertionError(row)


@pytest.mark.parametrize("g", range(1, 9))
@pytest.mark.parametrize("h", [8, 9, 17, 64, 100, 1023])
@pytest.mark.parametrize("r", [0, 1, 2, 4])
@pytest.mark.parametrize("b", BOUNDS)
def test_partition_and_halo_sources(g, h, r, b):
    if g > 1 and h // g < r:
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_plan_query(h, g, r, b, 0)
        assert e.value.status == M.EINVAL
        return
    ps = plans(h, g, r, b)
    # even split, first h mod g slabs one row longer (reading c8), contiguous cover
    assert sum(p.rows for p in ps) == h
    y = 0
    for k, p in enumerate(ps):
        assert p.y0 == y
        assert p.rows == h // g + (1 if k < h % g else 0)
        assert p.alloc_rows == p.rows + 2 * r  # both buffers get both halos (Fig 3)
        y += p.rows
    for k, p in enumerate(ps):
        if r == 0:
            assert p.n_recv == 0
            continue
        if g == 1:
            exp = {M.WRAP: M.HALO_WRAP_LOCAL, M.CLAMP: M.HALO_CLAMP, M.ZERO: M.HALO_ZERO}[b]
            assert p.top_kind == exp and p.bottom_kind == exp and p.n_recv == 0
            continue
        # each halo row's source is the owner of that global row (mod h under WRAP)
        for side, first in (("top", p.y0 - r), ("bottom", p.y0 + p.rows)):
            kind = getattr(p, side + "_kind")
            rows = [first + i for i in range(r)]
            if b != M.WRAP and any(x < 0 or x >= h for x in rows):
                assert kind == (M.HALO_CLAMP if b == M.CLAMP else M.HALO_ZERO)
                assert getattr(p, side + "_src_row") == -1
                continue
            assert kind == M.HALO_EXCHANGE
            src = getattr(p, side + "_src_row")
            assert src == first % h
            owners = {owner(ps, x % h) for x in rows}
            assert owners == {p.up if side == "top" else p.down}
        assert p.n_send == p.n_recv == (p.top_kind == M.HALO_EXCHANGE) + (p.bottom_kind == M.HALO_EXCHANGE)


@pytest.mark.parametrize("g", [2, 3, 4, 8])
def test_two_line_exchange_per_iteration(g):
    """'two-line boundary exchanges per iteration': r=1 WRAP -> every
    slab receives exactly 2 rows per iteration."""
    for p in plans(65536, g, 1, M.WRAP):
        assert p.n_recv == 2 and p.n_send == 2


def test_g2_wrap_neighbours_coincide():
    p0, p1 = plans(10, 2, 1, M.WRAP)
    assert p0.up == p0.down == 1 and p1.up == p1.down == 0


def test_min_slab_height_equals_r():
    for r in (1, 2, 4):
        ps = plans(8 * r, 8, r, M.WRAP)
        assert all(p.rows == r for p in ps)


@pytest.mark.parametrize("g,h", list(itertools.product([2, 4, 8], [65536, 16384, 32768])))
def test_bench_configs_partition(g, h):
    for p in plans(h, g, 4 if h == 32768 else 1, M.WRAP):
        assert p.rows == h // g


def test_no_checks_is_radius_zero_only():
    p = M.mapsm_plan_query(100, 4, 0, M.NO_CHECKS, 2)
    assert p.rows == 25 and p.n_recv == 0 and p.alloc_rows == 25
    with pytest.raises(M.MapsmError):
        M.mapsm_plan_query(100, 4, 1, M.NO_CHECKS, 0)
