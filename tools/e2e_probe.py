"""Probe of the pipelined e2e path (tuning helper): times of mapsm_bind_async /
mapsm_read_async alone and of one grid's bind overlapping another's read."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import mapsm_inputs as mi
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

w = h = 65536
torch.cuda.set_device(0)
ctx = M.mapsm_ctx_create(0, 1, 0, None, None)
hin = torch.empty((h, w), dtype=torch.uint8).pin_memory()
mi.life_u8(3, w, h, out=hin.numpy())
hout = torch.empty_like(hin).pin_memory()
A = M.Grid(ctx, w, h, "life", 1, "wrap")
B = M.Grid(ctx, w, h, "life", 1, "wrap")
for g in (A, B):
    g.set_option(M.OPT_OWN_STREAM, 1)
    g.bind(hin)


def t(fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fn()
    A.sync()
    B.sync()
    return (time.perf_counter() - t0) * 1e3


for _ in range(2):
    tb = t(lambda: M.mapsm_bind_async(B.handle, hin))
    tr = t(lambda: M.mapsm_read_async(A.handle, hout))
    tboth = t(lambda: (M.mapsm_bind_async(B.handle, hin), M.mapsm_read_async(A.handle, hout)))
    tit = t(lambda: A.iterate(200))
    tall = t(lambda: (M.mapsm_bind_async(B.handle, hin), A.iterate(200), M.mapsm_read_async(A.handle, hout)))
print(f"bind {tb:.1f} ms  read {tr:.1f} ms  bind||read {tboth:.1f} ms  iterate200 {tit:.1f} ms  bind||(iter+read) {tall:.1f} ms")
A.close()
B.close()
M.mapsm_ctx_destroy(ctx)

# the bench's pipelined loop with host enqueue timestamps
ctx = M.mapsm_ctx_create(0, 1, 0, None, None)
gs = [M.Grid(ctx, w, h, "life", 1, "wrap") for _ in range(3)]
outs = [hout] + [torch.empty_like(hin).pin_memory() for _ in range(2)]
for g in gs:
    g.set_option(M.OPT_OWN_STREAM, 1)
    g.bind(hin)
    g.iterate(200)
    g.sync()
torch.cuda.synchronize()
t0 = time.perf_counter()
log = []
for k in range(6):
    g = gs[k % 3]
    M.mapsm_bind_async(g.handle, hin)
    log.append(("bind", k, (time.perf_counter() - t0) * 1e3))
    g.iterate(200)
    log.append(("iter", k, (time.perf_counter() - t0) * 1e3))
    M.mapsm_read_async(g.handle, outs[k % 3])
    log.append(("read", k, (time.perf_counter() - t0) * 1e3))
for g in gs:
    g.sync()
print(f"6 steps {(time.perf_counter() - t0) * 1e3:.1f} ms")
print(" ".join(f"{a}{k}@{t:.0f}" for a, k, t in log))

for mode in ("bind+read", "bind+iter+read", "iter+read"):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for k in range(6):
        g = gs[k % 3]
        if "bind" in mode:
            M.mapsm_bind_async(g.handle, hin)
        if "iter" in mode:
            g.iterate(200)
        M.mapsm_read_async(g.handle, outs[k % 3])
    for g in gs:
        g.sync()
    print(f"{mode}: 6 steps {(time.perf_counter() - t0) * 1e3:.1f} ms")

# FIFO-chained uploads and downloads across the grids (events)
streams = [torch.cuda.ExternalStream(M.mapsm_grid_stream(g.handle)) for g in gs]
torch.cuda.synchronize()
t0 = time.perf_counter()
pb = pr = None
for k in range(6):
    g, s = gs[k % 3], streams[k % 3]
    if pb is not None:
        s.wait_event(pb)
    M.mapsm_bind_async(g.handle, hin)
    pb = torch.cuda.Event()
    pb.record(s)
    g.iterate(200)
    if pr is not None:
        s.wait_event(pr)
    M.mapsm_read_async(g.handle, outs[k % 3])
    pr = torch.cuda.Event()
    pr.record(s)
for g in gs:
    g.sync()
print(f"chained bind+iter+read: 6 steps {(time.perf_counter() - t0) * 1e3:.1f} ms")
