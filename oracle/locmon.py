"""Segment Location Monitor, cell by cell — TEST INFRASTRUCTURE ONLY.

Plain-Python oracle of Alg 2 (§4.4, "Location Monitor
Dependency Computation"), evaluated on individual cells instead of boxes so a
reader can check it against the paper line by line.  Only ``tests/`` may import
it; it shares no code with the product (``csrc/locmon.cpp``), which works on
N-D rectangles.

State per datum: ``last`` = for every cell, the locations whose last
output holds it (``lastOutput``); ``upto`` = for every cell, the locations
holding an up-to-date instance (``upToDate``); ``agg`` = the outputs are
partials that need aggregation (Alg 2 line 15).

Alg 2, in the paper's order, for (datum, required segment, target):
  1  needsAggregation <- false
  2  if the segment on the target is up to date: return
  5  if the datum's up-to-date buffer is on a single location:
  6      copy from that location to the target; return
  9  foreach device != target: intersect the segment with the device's
 10-12   lastOutput and copy the intersection from that device
 15  if the datum needs aggregation: needsAggregation <- true
and after the copies the target's upToDate grows by what was copied.

Reading l1: line 2 is applied cell by cell — cells the target
already holds up to date are never copied (the purpose of upToDate, "to avoid
unnecessary memory transfers"); for partials nothing is up to date.
The result of a query is the SET of (source, cell) pairs, which is unique
given that reading, so the product's box list can be compared with it exactly.
"""
from __future__ import annotations

import itertools


def cells(box) -> list[tuple]:
    """All cells of a box given as ((lo, hi), ...) per dimension."""
    return list(itertools.product(*[range(lo, hi) for lo, hi in box]))


class CellMonitor:
    def __init__(self):
        self.data = {}

    def output(self, datum: int, segs, needs_aggregation: bool = False) -> None:
        """A task wrote `segs` = [(location, box), ...] of `datum`."""
        last: dict[tuple, set] = {}
        for loc, box in segs:
            for c in cells(box):
                last.setdefault(c, set()).add(loc)
        upto = {} if needs_aggregation else {c: set(v) for c, v in last.items()}
        self.data[datum] = {"last": last, "upto": upto, "agg": needs_aggregation}

    def query(self, datum: int, required, target: int) -> tuple[set, bool]:
        """Alg 2 -> ({(src, cell), ...}, needsAggregation)."""
        d = self.data[datum]                                   # KeyError = unknown datum
        agg = False                                            # line 1
        req = cells(required)
        missing = [c for c in req if target not in d["upto"].get(c, set())]
        if not missing:                                        # line 2
            return set(), False
        locs = {loc for v in d["last"].values() for loc in v}
        if len(locs) == 1 and not d["agg"]:                    # line 5
            (src,) = locs
            for c in missing:
                if src not in d["last"].get(c, set()):
                    raise ValueError(f"cell {c} has no source")
            return {(src, c) for c in missing}, False          # line 6
        pairs = set()
        for c in missing:                                      # lines 9-14
            srcs = d["last"].get(c, set()) - {target}
            if not srcs and not d["agg"]:
                raise ValueError(f"cell {c} has no source")
            for s in srcs:
                pairs.add((s, c))
        if d["agg"]:
            agg = True                                         # line 16
        return pairs, agg

    def copied(self, datum: int, target: int, pairs) -> None:
        """The copies completed: the target holds those cells."""
        d = self.data[datum]
        if d["agg"]:
            return
        for _, c in pairs:
            d["upto"].setdefault(c, set()).add(target)
