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
    # round 2: SMEM-resident Life (one CTA and several), conv r = 3 (constant-slot
    # FFMA2 kernel), conv deep halos (local slabs), Window(3D) r = 3, deep-halo Life
    for (w, h) in ((256, 40), (2048, 300)):
        g0 = mi.life_u8(8, w, h)
        with M.Grid(ctx, w, h, "life", 1, b) as g:
            g.bind(g0)
            g.iterate(11)
            check(f"life resident {w}x{h} {b}", g.gather(), oracle.life(g0, 11, b))
    W = mi.weights_f32(9, 3)
    f0 = mi.field_f32(10, 1024, 40)
    with M.Grid(ctx, 1024, 40, "conv", 3, b, W) as g:
        g.bind(f0)
        g.iterate(2)
        check(f"conv r=3 1024x40 {b}", g.gather(), oracle.conv(f0, W, 2, b))
    W = mi.weights_f32(11, 2)
    f0 = mi.field_f32(12, 256, 30)
    with M.Grid(loc, 256, 30, "conv", 2, b, W, deep_halo=3) as g:
        g.bind(f0)
        g.iterate(7)
        check(f"conv deep halo K=3 local g=3 {b}", g.gather(), oracle.conv(f0, W, 7, b))
    for r in (1, 2):  # fused two-generation conv kernel (conv_tb.cuh)
        W = mi.weights_f32(16 + r, r)
        for (w, h) in ((516, 21), (12, 14)):
            f0 = mi.field_f32(18, w, h)
            with M.Grid(loc, w, h, "conv", r, b, W, deep_halo=2) as g:
                g.bind(f0)
                g.iterate(5)
                check(f"conv tb2 r={r} {w}x{h} local g=3 {b}", g.gather(), oracle.conv(f0, W, 5, b))
    W = mi.weights3d_f32(13, 3)
    v0 = mi.volume_f32(14, 40, 10, 9)
    with M.Grid(ctx, 40, 10, "conv", 3, b, W, d=9) as g:
        g.bind(v0)
        g.iterate(2)
        check(f"conv3d r=3 {b}", g.gather(), oracle.conv3d(v0, W, 2, b))
    g0 = mi.life_u8(15, 512, 60)
    with M.Grid(loc, 512, 60, "life", 1, b, deep_halo=4) as g:
        g.bind(g0)
        g.iterate(9)
        check(f"life deep halo K=4 local g=3 {b}", g.gather(), oracle.life(g0, 9, b))
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
