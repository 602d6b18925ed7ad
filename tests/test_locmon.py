"""Segment Location Monitor (Alg 2, §4.4) — CPU tests, no GPU.

1. The cell-level oracle (oracle/locmon.py) pinned to what the paper fixes:
   the halo rows of Fig 3 / "two-line boundary exchanges",
   duplicate-and-aggregate for Reductive outputs, upToDate reuse
   (P:L331), the single-location case (Alg 2 lines 5-7).
2. The product monitor (C ABI mapsm_locmon_*) against the oracle on random
   partitions in 1-3 dimensions: the (source, cell) pairs must be identical
   and no cell copied twice.
3. The static halo plan (mapsm_plan_query, the hot path's special case) is
   what the general monitor infers for every g, r and boundary.
"""
from __future__ import annotations

import random

import pytest

from oracle.locmon import CellMonitor, cells
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M


# ------------------------------------------------------------ oracle pins

def test_oracle_fig3_two_gpu_halo_rows():
    """GoL on 2 GPUs, 8 rows x 4 columns: each GPU needs its rows plus one
    halo row on each side (Window radius 1); under WRAP GPU 0's top halo is
    row 7 and its bottom halo row 4, both owned by GPU 1."""
    m = CellMonitor()
    m.output(0, [(0, ((0, 4), (0, 4))), (1, ((4, 8), (0, 4)))])
    pairs, agg = m.query(0, ((0, 5), (0, 4)), 0)   # owned rows + bottom halo
    assert not agg and pairs == {(1, (4, x)) for x in range(4)}
    pairs, agg = m.query(0, ((7, 8), (0, 4)), 0)   # top halo (row -1 mod 8)
    assert pairs == {(1, (7, x)) for x in range(4)}
    pairs, _ = m.query(0, ((3, 8), (0, 4)), 1)     # GPU 1: top halo row 3 from GPU 0
    assert pairs == {(0, (3, x)) for x in range(4)}


def test_oracle_reductive_aggregation():
    """Histogram bins duplicated on 3 GPUs (partials): the target receives
    every other partial and must aggregate (Alg 2 line 15)."""
    m = CellMonitor()
    m.output(7, [(g, ((0, 256),)) for g in range(3)], needs_aggregation=True)
    pairs, agg = m.query(7, ((0, 256),), 0)
    assert agg and pairs == {(g, (b,)) for g in (1, 2) for b in range(256)}
    m.copied(7, 0, pairs)                          # partials never become up to date
    pairs2, agg2 = m.query(7, ((0, 256),), 0)
    assert agg2 and pairs2 == pairs


def test_oracle_up_to_date_reuse_and_invalidation():
    m = CellMonitor()
    m.output(0, [(0, ((0, 5),)), (1, ((5, 10),))])
    pairs, _ = m.query(0, ((3, 8),), 2)
    assert pairs == {(0, (3,)), (0, (4,)), (1, (5,)), (1, (6,)), (1, (7,))}
    m.copied(0, 2, pairs)
    assert m.query(0, ((3, 8),), 2) == (set(), False)          # line 2: up to date
    pairs, _ = m.query(0, ((2, 9),), 2)                        # only the cells it lacks
    assert pairs == {(0, (2,)), (1, (8,))}
    m.output(0, [(0, ((0, 5),)), (1, ((5, 10),))])             # new version: stale copies
    assert len(m.query(0, ((3, 8),), 2)[0]) == 5


def test_oracle_single_location_and_errors():
    m = CellMonitor()
    m.output(3, [(-1, ((0, 6), (0, 2)))])                      # bound on the host only
    pairs, _ = m.query(3, ((2, 4), (0, 2)), 5)
    assert pairs == {(-1, c) for c in cells(((2, 4), (0, 2)))}  # lines 5-7
    with pytest.raises(ValueError):
        m.query(3, ((5, 7), (0, 2)), 5)                        # row 6 does not exist
    with pytest.raises(KeyError):
        m.query(4, ((0, 1), (0, 1)), 0)


# ------------------------------------------------- product vs the oracle

def _pairs_of(ops):
    out, vol = set(), 0
    for src, _dst, box in ops:
        cs = cells(box)
        vol += len(cs)
        out |= {(src, c) for c in cs}
    return out, vol


def _random_partition(rng, shape, nparts):
    """Split the box into up to nparts disjoint boxes by random cuts."""
    boxes = [tuple((0, n) for n in shape)]
    while len(boxes) < nparts:
        i = rng.randrange(len(boxes))
        b = boxes[i]
        d = rng.randrange(len(shape))
        lo, hi = b[d]
        if hi - lo < 2:
            if all(h - l < 2 for l, h in b):
                break
            continue
        cut = rng.randrange(lo + 1, hi)
        b1 = tuple((lo, cut) if k == d else b[k] for k in range(len(shape)))
        b2 = tuple((cut, hi) if k == d else b[k] for k in range(len(shape)))
        boxes[i:i + 1] = [b1, b2]
    return boxes


def _random_box(rng, shape):
    out = []
    for n in shape:
        a, b = sorted(rng.sample(range(n + 1), 2))
        out.append((a, b))
    return tuple(out)


@pytest.mark.parametrize("nd", [1, 2, 3])
def test_product_matches_cell_oracle_random(nd):
    rng = random.Random(1234 + nd)
    shape = {1: (23,), 2: (9, 7), 3: (5, 4, 6)}[nd]
    for trial in range(40):
        lm = M.mapsm_locmon_create(nd)
        ref = CellMonitor()
        try:
            for version in range(3):
                parts = _random_partition(rng, shape, rng.randint(1, 6))
                locs = rng.sample(range(8), len(parts)) if len(parts) <= 8 else list(range(len(parts)))
                if rng.random() < 0.2:                      # single location holds everything
                    parts, locs = [tuple((0, n) for n in shape)], [-1]
                segs = list(zip(locs, parts))
                M.mapsm_locmon_output(lm, 0, segs)
                ref.output(0, segs)
                for q in range(6):
                    req = _random_box(rng, shape)
                    target = rng.choice(list(range(-1, 10)))
                    ops, agg = M.mapsm_locmon_query(lm, 0, req, target, nd)
                    want, wagg = ref.query(0, req, target)
                    got, vol = _pairs_of(ops)
                    assert got == want and agg == wagg, (trial, version, req, target)
                    assert vol == len(got), "a cell is copied twice"
                    assert all(d == target and s != target for s, d, _ in ops)
                    if rng.random() < 0.6:
                        M.mapsm_locmon_copied(lm, 0, ops)
                        ref.copied(0, target, want)
        finally:
            M.mapsm_locmon_destroy(lm)


def test_product_aggregation_and_errors():
    lm = M.mapsm_locmon_create(1)
    try:
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_locmon_query(lm, 0, ((0, 4),), 0, 1)
        assert e.value.status == M.ESTATE
        M.mapsm_locmon_output(lm, 0, [(g, ((0, 256),)) for g in range(4)], needs_aggregation=True)
        ops, agg = M.mapsm_locmon_query(lm, 0, ((0, 256),), 2, 1)
        assert agg and sorted(s for s, _, _ in ops) == [0, 1, 3]
        M.mapsm_locmon_output(lm, 1, [(0, ((0, 10),)), (1, ((10, 20),))])
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_locmon_query(lm, 1, ((15, 25),), 2, 1)      # rows 20..24 have no source
        assert e.value.status == M.EINVAL
        assert M.mapsm_locmon_query(lm, 1, ((3, 3),), 2, 1) == ([], False)   # empty segment
        # many ops: the binding retries with a larger array (ENOMEM protocol)
        M.mapsm_locmon_output(lm, 2, [(k, ((k, k + 1),)) for k in range(40)])
        ops, _ = M.mapsm_locmon_query(lm, 2, ((0, 40),), 99, 1)
        assert len(ops) == 40
    finally:
        M.mapsm_locmon_destroy(lm)
    with pytest.raises(M.MapsmError):
        M.mapsm_locmon_create(4)


# ------------------------------------- the halo plan is what Alg 2 infers

def _halo_boxes(y_from, nrows, h):
    """Rows [y_from, y_from + nrows) mod h as at most 2 boxes (WRAP)."""
    rows = [(y_from + k) % h for k in range(nrows)]
    boxes, start = [], rows[0]
    for a, b in zip(rows, rows[1:] + [None]):
        if b != a + 1:
            boxes.append((start, a + 1))
            start = b
    return boxes


@pytest.mark.parametrize("boundary", [M.WRAP, M.CLAMP, M.ZERO])
def test_static_halo_plan_equals_inferred_copies(boundary):
    W = 3
    for g in range(1, 9):
        for r in range(1, 5):
            for h in (g * r, g * r + 1, 4 * g + 3, 37):
                if h < g * r:
                    continue
                plans = [M.mapsm_plan_query(h, g, r, boundary, k) for k in range(g)]
                lm = M.mapsm_locmon_create(2)
                try:
                    M.mapsm_locmon_output(lm, 0, [(k, ((p.y0, p.y0 + p.rows), (0, W))) for k, p in enumerate(plans)])
                    for k, p in enumerate(plans):
                        for side in ("top", "bottom"):
                            y_from = p.y0 - r if side == "top" else p.y0 + p.rows
                            inside = 0 <= y_from and y_from + r <= h
                            if boundary != M.WRAP and not inside:
                                # global edge: no source in the datum (CLAMP/ZERO halos are local)
                                assert (p.top_kind if side == "top" else p.bottom_kind) in (M.HALO_CLAMP, M.HALO_ZERO)
                                continue
                            ops = []
                            for lo, hi in _halo_boxes(y_from, r, h):
                                o, agg = M.mapsm_locmon_query(lm, 0, ((lo, hi), (0, W)), k)
                                assert not agg
                                ops += o
                            kind = p.top_kind if side == "top" else p.bottom_kind
                            src_row = p.top_src_row if side == "top" else p.bottom_src_row
                            nb = p.up if side == "top" else p.down
                            if kind == M.HALO_WRAP_LOCAL:
                                assert ops == []          # g = 1: the slab's own rows are up to date
                                continue
                            assert kind == M.HALO_EXCHANGE
                            assert {s for s, _, _ in ops} == {nb}, (g, r, h, k, side)
                            got_rows = sorted(y for _, _, b in ops for y in range(*b[0]))
                            assert got_rows == sorted((src_row + i) % h for i in range(r))
                finally:
                    M.mapsm_locmon_destroy(lm)
