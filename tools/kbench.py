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

wl = sys.argv[1] if len(sys.argv) > 1 else "life64k"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 20
cfg = {"life64k": ("life", 65536, 65536, 1, "wrap", 0.25), "life8k": ("life", 8192, 8192, 1, "wrap", 0.25),
       "conv5": ("conv", 16384, 16384, 2, "clamp", 8.0), "conv9": ("conv", 32768, 4096, 4, "zero", 8.0)}[wl]
op, w, h, r, b, bc = cfg
torch.cuda.set_device(0)
ctx = M.mapsm_ctx_create(0, 1, 0, None, None)
W = mi.weights_f32(1, r) if op == "conv" else None
g = M.Grid(ctx, w, h, op, r, b, W)
if op == "life":
    x = torch.randint(0, 2, (h, w), dtype=torch.uint8, device="cuda")
else:
    x = torch.rand((h, w), dtype=torch.float32, device="cuda")
g.bind(x)
g.iterate(4)
g.sync()
per_l = []
for rep in range(5):
    g.set_option(M.OPT_TIMING, 1)
    g.iterate(iters)
    ms, n, bms, bn = M.mapsm_get_timing(g.handle)
    per_l.append(ms / n)
per = sorted(per_l)[len(per_l) // 2]
gbs = bc * w * h / (per / 1e3) / 1e9
g.set_option(M.OPT_TIMING, 0)
# graphs region
g.iterate(16)
g.sync()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s = torch.cuda.ExternalStream(M.mapsm_grid_stream(g.handle))
e0.record(s)
g.iterate(iters * 2)
e1.record(s)
e1.synchronize()
reg = e0.elapsed_time(e1) / (iters * 2)
print(json.dumps({"lib": os.environ.get("MAPSM_LIB", "default"), "workload": wl, "ms_per_launch": per,
                  "GBps": gbs, "region_ms_per_iter": reg, "region_GBps": bc * w * h / (reg / 1e3) / 1e9,
                  "cells_per_s": w * h / (reg / 1e3)}))
g.close()
M.mapsm_ctx_destroy(ctx)
