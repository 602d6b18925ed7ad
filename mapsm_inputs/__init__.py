"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and
bench.py (SURVEY §8(c) reading c12).

This module holds none of the method's arithmetic: it only produces the
counter-based random grids/weights and the hand-placed patterns of
BASELINE.json configs[0].  Both the oracle side and the CUDA side consume its
outputs; neither imports the other.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libmapsm_inputs.so")
_SRC = os.path.join(_HERE, "gen.c")

# Seeds of SURVEY §8(d) / BASELINE.md §4.
SEED_LIFE_8K = 0x5EED0002
SEED_LIFE_64K = 0x5EED0003
SEED_CONV5_FIELD = 0x5EED0004
SEED_CONV5_W = 0x5EED0044
SEED_CONV9_FIELD = 0x5EED0005
SEED_CONV9_W = 0x5EED0055
SEED_HIST_UNIFORM = 0x5EED0006
SEED_HIST_SKEWED = 0x5EED0066
SEED_CONV3D_FIELD = 0x5EED0007
SEED_CONV3D_W = 0x5EED0077


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _SO, _SRC])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i64, u64, p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p
        _lib.mapsm_gen_splitmix64.argtypes = [u64]
        _lib.mapsm_gen_splitmix64.restype = u64
        _lib.mapsm_gen_life_u8.argtypes = [u64, i64, i64, i64, p, i64]
        _lib.mapsm_gen_life_u8.restype = None
        _lib.mapsm_gen_field_f32.argtypes = [u64, i64, i64, i64, p, i64]
        _lib.mapsm_gen_field_f32.restype = None
        _lib.mapsm_gen_weights_f32.argtypes = [u64, ctypes.c_int, p]
        _lib.mapsm_gen_weights_f32.restype = None
        _lib.mapsm_gen_weights_n_f32.argtypes = [u64, ctypes.c_int, p]
        _lib.mapsm_gen_weights_n_f32.restype = ctypes.c_int
        _lib.mapsm_gen_image_u8.argtypes = [u64, i64, i64, i64, p, i64, ctypes.c_int]
        _lib.mapsm_gen_image_u8.restype = None
    return _lib


def splitmix64(x: int) -> int:
    return int(_L().mapsm_gen_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def life_u8(seed: int, w: int, h: int, y0: int = 0, out: np.ndarray | None = None) -> np.ndarray:
    """Rows [y0, y0+h) of the random Life grid of width w (0/1 bytes)."""
    if out is None:
        out = np.empty((h, w), dtype=np.uint8)
    assert out.dtype == np.uint8 and out.shape[0] >= h and out.shape[1] >= w and out.strides[1] == 1
    _L().mapsm_gen_life_u8(seed, w, y0, h, out.ctypes.data, out.strides[0])
    return out


def field_f32(seed: int, w: int, h: int, y0: int = 0, out: np.ndarray | None = None) -> np.ndarray:
    """Rows [y0, y0+h) of the random U[0,1) fp32 field of width w."""
    if out is None:
        out = np.empty((h, w), dtype=np.float32)
    assert out.dtype == np.float32 and out.strides[1] == 4
    _L().mapsm_gen_field_f32(seed, w, y0, h, out.ctypes.data, out.strides[0] // 4)
    return out


def weights_f32(seed: int, r: int) -> np.ndarray:
    """(2r+1)^2 non-negative asymmetric weights summing to ~1, row-major."""
    k = 2 * r + 1
    out = np.empty(k * k, dtype=np.float32)
    _L().mapsm_gen_weights_f32(seed, r, out.ctypes.data)
    return out.reshape(k, k)


def weights3d_f32(seed: int, r: int) -> np.ndarray:
    """(2r+1)^3 non-negative asymmetric weights summing to ~1, (dz, dy, dx) order."""
    k = 2 * r + 1
    out = np.empty(k ** 3, dtype=np.float32)
    assert _L().mapsm_gen_weights_n_f32(seed, k ** 3, out.ctypes.data) == 0
    return out.reshape(k, k, k)


def volume_f32(seed: int, w: int, h: int, d: int, z0: int = 0) -> np.ndarray:
    """Planes [z0, z0+d) of a synthetic (depth, h, w) fp32 volume: the 2-D
    field recipe over global row index z*h + y, so plane z of the volume is
    rows [z*h, (z+1)*h) of field_f32(seed, w, ...)."""
    return field_f32(seed, w, d * h, y0=z0 * h).reshape(d, h, w)


def image_u8(seed: int, w: int, h: int, y0: int = 0, kind: str = "uniform",
             out: np.ndarray | None = None) -> np.ndarray:
    """Rows [y0, y0+h) of a synthetic u8 image (histogram path)."""
    if out is None:
        out = np.empty((h, w), dtype=np.uint8)
    assert out.dtype == np.uint8 and out.strides[1] == 1
    _L().mapsm_gen_image_u8(seed, w, y0, h, out.ctypes.data, out.strides[0], {"uniform": 0, "skewed": 1}[kind])
    return out


# Hand-placed patterns (SURVEY §8(c) "BJ.configs[1]" pin).
GLIDER = [(0, 1), (1, 2), (2, 0), (2, 1), (2, 2)]  # .O. / ..O / OOO, moves (+1,+1) per 4 gens


def place(grid: np.ndarray, cells, y: int, x: int) -> None:
    h, w = grid.shape
    for dy, dx in cells:
        grid[(y + dy) % h, (x + dx) % w] = 1


def config0_grid() -> np.ndarray:
    """BASELINE.json configs[0]: 64x64, glider at (60,60), horizontal blinker at
    row 10 cols 40-42, block at rows 40-41 cols 10-11."""
    g = np.zeros((64, 64), dtype=np.uint8)
    place(g, GLIDER, 60, 60)
    place(g, [(0, 0), (0, 1), (0, 2)], 10, 40)
    place(g, [(0, 0), (0, 1), (1, 0), (1, 1)], 40, 10)
    return g
