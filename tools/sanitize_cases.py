"""Small cases of every kernel path for compute-sanitizer (memcheck /
racecheck / synccheck).  Exits non-zero on any parity failure."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

ctx = M.mapsm_ctx_create(0, 1, 0, None, None)
loc = M.mapsm_ctx_create_local([0, 0, 0])
ok = True


def check(name, got, exp):
    global ok
    same = np.array_equal(np.asarray(got).view(np.uint8), np.asarray(exp).view(np.uint8))
    print(f"{name}: {'ok' if same else 'MISMATCH'}", flush=True)
    ok &= same


for b in ("wrap", "clamp", "zero"):
    for (w, h) in ((256, 40), (192, 33)):  # TMA kernel / register kernel
        g0 = mi.life_u8(3, w, h)
        for persistent in (0, 1):
            with M.Grid(ctx, w, h, "life", 1, b) as g:
                g.set_option(M.OPT_PERSISTENT, persistent)
                g.bind(g0)
                g.iterate(5)
                check(f"life {w}x{h} {b} persistent={persistent}", g.gather(), oracle.life(g0, 5, b))
    with M.Grid(loc, 256, 40, "life", 1, b) as g:
        g0 = mi.life_u8(4, 256, 40)
        g.bind(g0)
        g.iterate(3)
        check(f"life local g=3 {b}", g.gather(), oracle.life(g0, 3, b))
    for r in (1, 2, 4):
        W = mi.weights_f32(5, r)
        for (w, h) in ((256, 24), (21, 13)):  # TMA kernel / generic kernel
            f0 = mi.field_f32(6, w, h)
            with M.Grid(ctx, w, h, "conv", r, b, W) as g:
                g.bind(f0)
                g.iterate(2)
                check(f"conv r={r} {w}x{h} {b}", g.gather(), oracle.conv(f0, W, 2, b))
img = mi.image_u8(7, 300, 50)
with M.Grid(ctx, 300, 50, "histogram") as g:
    g.bind(img)
    check("histogram", g.histogram(), oracle.histogram(img))
with M.Grid(loc, 300, 50, "histogram") as g:
    g.bind(img)
    check("histogram local g=3", g.histogram(), oracle.histogram(img))
M.mapsm_ctx_destroy(loc)
M.mapsm_ctx_destroy(ctx)
print("ALL OK" if ok else "FAILURES")
sys.exit(0 if ok else 1)
