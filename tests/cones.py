"""Light-cone sampling for full-size parity (test helper).

After n iterations of a radius-r stencil, an output block depends only on the
input within distance R = n*r.  ``cone_eval`` evaluates such a block with the
ORACLE one iteration at a time on a patch cut out of the (generated) input,
cropping r cells from every cut side after each step (cells within k*r of a
cut are invalid after k steps); real grid edges keep their boundary mode and a
fully covered axis keeps its true WRAP.  Only the oracle does arithmetic."""
import numpy as np

import oracle


def _axis(lo, hi, R, n_axis, b):
    """Index array along one axis and (mode_lo, mode_hi, cut_lo, cut_hi)."""
    if hi - lo + 2 * R >= n_axis:
        return np.arange(n_axis), (b, b, False, False), 0
    if b == "wrap":
        return np.arange(lo - R, hi + R) % n_axis, ("zero", "zero", True, True), lo - R
    a, z = max(0, lo - R), min(n_axis, hi + R)
    return np.arange(a, z), (b if a == 0 else "zero", b if z == n_axis else "zero", a > 0, z < n_axis), a


def rows_from(gen, yidx):
    """Stack generated global rows yidx (gen(y0, nrows) -> array) in order."""
    out, i = [], 0
    while i < len(yidx):
        j = i
        while j + 1 < len(yidx) and yidx[j + 1] == yidx[j] + 1:
            j += 1
        out.append(gen(int(yidx[i]), j - i + 1))
        i = j + 1
    return np.concatenate(out)


def cone_eval(op, gen, h, w, r, n, boundary, ys, ye, xs, xe, weights=None):
    R = n * r
    yidx, (ty, by, cut_t, cut_b), y_start = _axis(ys, ye, R, h, boundary)
    xidx, (lx, rx, cut_l, cut_r), x_start = _axis(xs, xe, R, w, boundary)
    patch = rows_from(gen, yidx)[:, xidx]
    # coordinates of patch[0,0] in "unwrapped" global space
    y0, x0 = y_start, x_start
    for _ in range(n):
        if op == "life":
            patch = oracle.life(patch, 1, sides=(ty, by, lx, rx))
        else:
            patch = oracle.conv(patch, weights, 1, sides=(ty, by, lx, rx))
        t, b_, l, rr = (r if cut_t else 0), (r if cut_b else 0), (r if cut_l else 0), (r if cut_r else 0)
        patch = patch[t:patch.shape[0] - b_, l:patch.shape[1] - rr]
        y0 += t
        x0 += l
    # full axes start at 0 (no unwrapping); cut axes start at y0/x0
    oy = ys - y0 if (cut_t or cut_b) else ys
    ox = xs - x0 if (cut_l or cut_r) else xs
    return patch[oy:oy + (ye - ys), ox:ox + (xe - xs)]


def cone_eval3d(vol_rows, d, h, w, r, n, boundary, zr, yr, xr, weights):
    """Window(3D) light cone: the oracle's generation-n values of the block
    zr x yr x xr ((start, end) per axis) of a d x h x w volume, evaluated on
    the cut-out patch as cone_eval does in 2-D.  vol_rows(z, y0, nrows) ->
    generated rows [y0, y0+nrows) of plane z (shape (nrows, w))."""
    R = n * r
    axes = [_axis(zr[0], zr[1], R, d, boundary), _axis(yr[0], yr[1], R, h, boundary),
            _axis(xr[0], xr[1], R, w, boundary)]
    (zidx, zm, z_start), (yidx, ym, y_start), (xidx, xm, x_start) = axes
    patch = np.stack([rows_from(lambda y0, nr, z=int(z): vol_rows(z, y0, nr), yidx)[:, xidx] for z in zidx])
    origin = [z_start, y_start, x_start]
    modes = [zm, ym, xm]
    sides = (zm[0], zm[1], ym[0], ym[1], xm[0], xm[1])
    for _ in range(n):
        patch = oracle.conv3d(patch, weights, 1, sides=sides)
        sl = []
        for a, m in enumerate(modes):
            lo = r if m[2] else 0
            hi = r if m[3] else 0
            sl.append(slice(lo, patch.shape[a] - hi))
            origin[a] += lo
        patch = patch[tuple(sl)]
    out = []
    for a, (m, rng) in enumerate(zip(modes, (zr, yr, xr))):
        o = rng[0] - origin[a] if (m[2] or m[3]) else rng[0]
        out.append(slice(o, o + rng[1] - rng[0]))
    return patch[tuple(out)]
