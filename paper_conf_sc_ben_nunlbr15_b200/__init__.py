"""mapsm — B200-native Window(2D) -> Structured-Injective stencil path of
MAPS-Multi (SC'15): Game of Life and fp32 window convolution, row-slab
partitioned over GPUs with per-iteration halo exchange.

The product is ``libmapsm.so`` (C ABI in ``include/mapsm.h``); this package is
its thin ctypes binding (``mapsm``) and the in-tree build (``build``).  The
multi-process bootstrap is the caller's: ``torch.distributed`` broadcasts
``mapsm_nccl_unique_id()`` and every rank calls ``mapsm_ctx_create`` (see
bench.py).  There is no CPU fallback.
"""
from . import mapsm  # noqa: F401
from .mapsm import Grid, MapsmError  # noqa: F401

__all__ = ["mapsm", "Grid", "MapsmError"]
