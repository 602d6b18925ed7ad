"""CPU oracle — TEST INFRASTRUCTURE ONLY.

Plain, slow C implementation (``oracle.c``) of what the Window(2D) ->
Structured-Injective hot path computes (Game of Life and the fp32 window
convolution), written from PAPER.md (see the header of oracle.c for the
definitions and citations).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` leg may import this
package.  It shares no code with ``paper_conf_sc_ben_nunlbr15_b200`` and never
imports it.

Parity status: Life pinned (closed forms, scipy neighbour count,
known methuselah, exhaustive tiny tori); fp32 conv pinned (exact-rational fma
chain, scipy correlate in fp64, roll/identity closed forms, mass invariant);
fp64 conv pinned (scipy correlate); histogram pinned (numpy.bincount, closed
forms, invariants); fp32-field histogram pinned (closed forms at bin edges,
numpy.floor/clip binning); Segment Location Monitor (``oracle/locmon.py``)
pinned by the paper's worked cases (Fig 3 halos, Reductive aggregation,
upToDate reuse) and brute-force cell enumeration.  No function is "parity
unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

WRAP, CLAMP, ZERO = 0, 1, 2
_MODES = {"wrap": WRAP, "clamp": CLAMP, "zero": ZERO}

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")


def build(force: bool = False) -> str:
    """Compile oracle.c (gcc, OpenMP, no fast-math, no FP contraction)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-Wall", "-o", _SO, _SRC, "-lm"])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i64, p, ci = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int
        _lib.oracle_life_ex.argtypes = [p, p, i64, i64, i64, ci, ci, ci, ci]
        _lib.oracle_conv_ex.argtypes = [p, p, i64, i64, i64, ci, p, ci, ci, ci, ci]
        _lib.oracle_conv_f64_ex.argtypes = [p, p, i64, i64, i64, ci, p, ci, ci, ci, ci]
        for f in (_lib.oracle_life_ex, _lib.oracle_conv_ex, _lib.oracle_conv_f64_ex):
            f.restype = ci
        _lib.oracle_num_threads.restype = ci
        _lib.oracle_histogram.argtypes = [p, i64, i64, i64, ci, p]
        _lib.oracle_histogram.restype = ci
        _lib.oracle_conv3d_ex.argtypes = [p, p, i64, i64, i64, i64, ci, p, p]
        _lib.oracle_conv3d_ex.restype = ci
        _lib.oracle_histogram_f32.argtypes = [p, i64, i64, i64, ci, p]
        _lib.oracle_histogram_f32.restype = ci
    return _lib


def _mode(m) -> int:
    return _MODES[m] if isinstance(m, str) else int(m)


def _sides(boundary, sides):
    if sides is None:
        b = _mode(boundary)
        return (b, b, b, b)
    return tuple(_mode(s) for s in sides)


def life(grid: np.ndarray, n: int, boundary="wrap", sides=None) -> np.ndarray:
    """Generation n of a u8 Life grid (nonzero = alive) -> 0/1 u8.

    ``sides`` = (top, bottom, left, right) modes overrides ``boundary``."""
    g = np.ascontiguousarray(grid, dtype=np.uint8)
    h, w = g.shape
    out = np.empty_like(g)
    rc = _L().oracle_life_ex(g.ctypes.data, out.ctypes.data, w, h, n, *_sides(boundary, sides))
    if rc != 0:
        raise ValueError("oracle_life_ex rejected its arguments")
    return out


def conv(field: np.ndarray, weights: np.ndarray, n: int, boundary="wrap", sides=None) -> np.ndarray:
    """n fixed-order fp32 window-convolution steps (reading c11)."""
    f = np.ascontiguousarray(field, dtype=np.float32)
    wt = np.ascontiguousarray(weights, dtype=np.float32)
    k = wt.shape[0]
    assert wt.shape == (k, k) and k % 2 == 1
    h, w = f.shape
    out = np.empty_like(f)
    rc = _L().oracle_conv_ex(f.ctypes.data, out.ctypes.data, w, h, n, k // 2, wt.ctypes.data,
                             *_sides(boundary, sides))
    if rc != 0:
        raise ValueError("oracle_conv_ex rejected its arguments")
    return out


def conv_f64(field: np.ndarray, weights: np.ndarray, n: int, boundary="wrap", sides=None) -> np.ndarray:
    """n window-convolution steps accumulated and carried in fp64."""
    f = np.ascontiguousarray(field, dtype=np.float32)
    wt = np.ascontiguousarray(weights, dtype=np.float32)
    k = wt.shape[0]
    h, w = f.shape
    out = np.empty((h, w), dtype=np.float64)
    rc = _L().oracle_conv_f64_ex(f.ctypes.data, out.ctypes.data, w, h, n, k // 2, wt.ctypes.data,
                                 *_sides(boundary, sides))
    if rc != 0:
        raise ValueError("oracle_conv_f64_ex rejected its arguments")
    return out


def conv3d(vol: np.ndarray, weights: np.ndarray, n: int, boundary="wrap", sides=None) -> np.ndarray:
    """n steps of the fp32 Window(3D) convolution of a (d, h, w) volume with
    (2r+1)^3 weights ordered (dz, dy, dx); `sides` = 6 modes (z lo, z hi, y lo,
    y hi, x lo, x hi) overriding `boundary`."""
    v = np.ascontiguousarray(vol, dtype=np.float32)
    wt = np.ascontiguousarray(weights, dtype=np.float32).ravel()
    k = round(len(wt) ** (1 / 3))
    assert k ** 3 == len(wt) and k % 2 == 1
    d, h, w = v.shape
    modes = np.array([_mode(m) for m in (sides if sides is not None else [boundary] * 6)], dtype=np.int32)
    out = np.empty_like(v)
    rc = _L().oracle_conv3d_ex(v.ctypes.data, out.ctypes.data, w, h, d, n, k // 2, wt.ctypes.data,
                               modes.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_conv3d_ex rejected its arguments")
    return out


def histogram(img: np.ndarray, nbins: int = 256) -> np.ndarray:
    """256-bin histogram of a u8 image (Reductive-Static pattern, Fig 4)."""
    a = np.asarray(img)
    assert a.dtype == np.uint8 and a.ndim == 2 and a.strides[1] == 1
    h, w = a.shape
    out = np.zeros(nbins, dtype=np.uint64)
    rc = _L().oracle_histogram(a.ctypes.data, w, h, a.strides[0] if h > 0 else w, nbins, out.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_histogram rejected its arguments")
    return out


def histogram_f32(field: np.ndarray, nbins: int = 256) -> np.ndarray:
    """256-bin histogram of an fp32 field over [0, 1): bin = floor(v * 256),
    clamped to [0, 255], NaN -> 0 (reading h4)."""
    a = np.ascontiguousarray(field, dtype=np.float32)
    h, w = a.shape
    out = np.zeros(nbins, dtype=np.uint64)
    rc = _L().oracle_histogram_f32(a.ctypes.data, w, h, w, nbins, out.ctypes.data)
    if rc != 0:
        raise ValueError("oracle_histogram_f32 rejected its arguments")
    return out


def num_threads() -> int:
    return int(_L().oracle_num_threads())
