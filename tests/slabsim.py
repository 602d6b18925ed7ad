"""Slab-decomposition simulator — the CPU "fake backend" for the multi-slab
logic (SURVEY §4 test pyramid tier 1).  It partitions a grid with the
library's plan (mapsm_plan_query, pure host code), fills every slab's halos
exactly as the plan says (exchange / local wrap / clamp / zero) and advances
each slab with the ORACLE on its own rows.  It never calls a kernel."""
import numpy as np

import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

_NAMES = {M.WRAP: "wrap", M.CLAMP: "clamp", M.ZERO: "zero"}


def halo_rows(plan, slab, slabs_by_rank, plans, side, r, h):
    kind = plan.top_kind if side == "top" else plan.bottom_kind
    w = slab.shape[1]
    if kind == M.HALO_EXCHANGE:
        src = plan.top_src_row if side == "top" else plan.bottom_src_row
        nb = plan.up if side == "top" else plan.down
        q = plans[nb]
        rows = [((src + i) % h) - q.y0 for i in range(r)]
        assert all(0 <= x < q.rows for x in rows), "halo row not owned by the neighbour"
        return slabs_by_rank[nb][rows]
    if kind == M.HALO_WRAP_LOCAL:
        idx = [(-r + i) % plan.rows for i in range(r)] if side == "top" else [(plan.rows + i) % plan.rows for i in range(r)]
        return slab[idx]
    if kind == M.HALO_CLAMP:
        return np.repeat(slab[:1] if side == "top" else slab[-1:], r, axis=0)
    return np.zeros((r, w), dtype=slab.dtype)


def step_slab(op, patch, r, boundary, weights):
    sides = ("zero", "zero", _NAMES[boundary], _NAMES[boundary])
    if op == "life":
        return oracle.life(patch, 1, sides=sides)[r:-r]
    return oracle.conv(patch, weights, 1, sides=sides)[r:-r]


def simulate(op, grid0, n, r, boundary, g, weights=None):
    h = grid0.shape[0]
    plans = [M.mapsm_plan_query(h, g, r, boundary, k) for k in range(g)]
    slabs = [grid0[p.y0:p.y0 + p.rows].copy() for p in plans]
    if op == "life":
        slabs = [(s != 0).astype(np.uint8) for s in slabs]
    for _ in range(n):
        new = []
        for k, p in enumerate(plans):
            top = halo_rows(p, slabs[k], slabs, plans, "top", r, h)
            bot = halo_rows(p, slabs[k], slabs, plans, "bottom", r, h)
            new.append(step_slab(op, np.concatenate([top, slabs[k], bot]), r, boundary, weights))
        slabs = new
    return np.concatenate(slabs)
