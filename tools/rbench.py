"""Time the one-slab Life paths (SMEM-resident / grid-barrier persistent) of a
libmapsm build (MAPSM_LIB) on BASELINE configs[1] (8192^2 WRAP, 1000
generations), with a bit-exact spot check against the oracle.  Tuning helper.

python tools/rbench.py [--w 8192 --h 8192 --n 1000 --mode 1 --reps 5]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

ap = argparse.ArgumentParser()
ap.add_argument("--w", type=int, default=8192)
ap.add_argument("--h", type=int, default=8192)
ap.add_argument("--n", type=int, default=1000)
ap.add_argument("--mode", type=int, default=1)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--b", default="wrap")
args = ap.parse_args()
torch.cuda.set_device(0)
ctx = M.mapsm_ctx_create(0, 1, 0, None, None)
# parity spot check on a smaller grid (all three boundaries)
for b in ("wrap", "clamp", "zero"):
    g0 = mi.life_u8(7, 2048, 1111)
    with M.Grid(ctx, 2048, 1111, "life", 1, b) as g:
        g.set_option(M.OPT_PERSISTENT, args.mode)
        g.bind(g0)
        g.iterate(37)
        ok = np.array_equal(g.gather(), oracle.life(g0, 37, b))
    assert ok, b
g0 = mi.life_u8(mi.SEED_LIFE_8K, args.w, args.h)
g = M.Grid(ctx, args.w, args.h, "life", 1, args.b)
g.set_option(M.OPT_PERSISTENT, args.mode)
g.bind(g0)
stream = torch.cuda.ExternalStream(M.mapsm_grid_stream(g.handle))
g.iterate(args.n)
g.sync()
ts = []
for _ in range(args.reps):
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    g.iterate(args.n)
    e1.record(stream)
    e1.synchronize()
    ts.append(e0.elapsed_time(e1))
li = g.launch()
g.close()
M.mapsm_ctx_destroy(ctx)
t = sorted(ts)[len(ts) // 2]
print(json.dumps({"lib": os.environ.get("MAPSM_LIB", "default"), "kernel": M.KERNEL_NAMES.get(li.kernel),
                  "ctas": li.ctas, "threads": li.threads, "smem": li.smem_bytes, "K": li.rows_per_stage,
                  "ms": t, "us_per_gen": t * 1e3 / args.n,
                  "cells_per_s": args.w * args.h * args.n / (t / 1e3)}))
