"""Kernel-level timing of one workload (tuning helper, not the bench).

python tools/kbench.py [life64k|life8k|conv5|conv9] [iters]
Prints per-launch device time of the bulk stencil kernel (CUDA events around
each launch, MAPSM_OPT_TIMING) and the achieved algorithmic GB/s."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import mapsm_inputs as mi
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

import argparse

ap = argparse.ArgumentParser()
ap.add_argument("wl", nargs="?", default="life64k")
ap.add_argument("iters", nargs="?", type=int, default=20)
ap.add_argument("--local", type=int, default=0, help="g slabs in one process on cuda:0")
ap.add_argument("--exchange", default="copy", choices=["copy", "p2p"])
ap.add_argument("--deep", type=int, default=1, help="MAPSM_OPT_DEEP_HALO (generations per pass)")
args = ap.parse_args()
wl, iters = args.wl, args.iters
cfg = {"life64k": ("life", 65536, 65536, 1, "wrap", 0.25), "life8k": ("life", 8192, 8192, 1, "wrap", 0.25),
       "conv5": ("conv", 16384, 16384, 2, "clamp", 8.0), "conv9": ("conv", 32768, 4096, 4, "zero", 8.0)}[wl]
op, w, h, r, b, bc = cfg
torch.cuda.set_device(0)
ctx = M.mapsm_ctx_create_local([0] * args.local) if args.local else M.mapsm_ctx_create(0, 1, 0, None, None)
W = mi.weights_f32(1, r) if op == "conv" else None
g = M.Grid(ctx, w, h, op, r, b, W, deep_halo=args.deep)
if args.exchange == "p2p":
    g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
if op == "life":
    x = torch.randint(0, 2, (h, w), dtype=torch.uint8, device="cuda")
else:
    x = torch.rand((h, w), dtype=torch.float32, device="cuda")
g.bind(x)
g.iterate(4)
g.sync()
if args.local:
    per, gbs = float("nan"), float("nan")  # per-kernel events only for one slab
else:
    per_l = []
    for rep in range(5):
        g.set_option(M.OPT_TIMING, 1)
        g.iterate(iters)
        ms, n, bms, bn = M.mapsm_get_timing(g.handle)
        per_l.append(ms / n / max(1, g.info().gens_per_pass))  # per generation
    per = sorted(per_l)[len(per_l) // 2]
    gbs = bc * w * h / (per / 1e3) / 1e9
    g.set_option(M.OPT_TIMING, 0)
# graphs region (SM clock sampled during it: FMA-bound kernels run under the power cap)
from bench import ClockSampler  # noqa: E402
smp = ClockSampler(0).start()
time.sleep(0.3)
g.iterate(16)
g.sync()
torch.cuda.synchronize()
t0 = time.perf_counter()
tw0 = time.time()
g.iterate(iters * 2)
g.sync()
reg = (time.perf_counter() - t0) * 1e3 / (iters * 2)  # wall: all slabs' streams
clk = smp.region(tw0, time.time())
smp.stop()
print(json.dumps({"lib": os.environ.get("MAPSM_LIB", "default"), "workload": wl, "local": args.local,
                  "exchange": args.exchange, "deep": args.deep, "ms_per_launch": per,
                  "GBps": gbs, "region_ms_per_iter": reg, "region_GBps": bc * w * h / (reg / 1e3) / 1e9,
                  "cells_per_s": w * h / (reg / 1e3), "sm_mhz": clk.get("sm_mhz"), "reasons": clk.get("reasons")}))
g.close()
M.mapsm_ctx_destroy(ctx)
