"""Thin ctypes binding of libmapsm (include/mapsm.h) — argument marshalling only.

Every function here has the name of the C entry point it wraps and raises
``MapsmError`` on a non-OK status.  All compute happens in libmapsm's sm_100a
kernels; there is no Python or CPU fallback: if ``libmapsm.so`` is missing
the import fails loudly (build it with ``python -m
paper_conf_sc_ben_nunlbr15_b200.build``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

# MAPSM_LIB may point at an alternative build of the same library (kernel
# tuning experiments); the default is the in-tree build.
_LIB_PATH = os.environ.get("MAPSM_LIB") or os.path.join(os.path.dirname(os.path.abspath(__file__)), "libmapsm.so")

# enums (include/mapsm.h)
OK, EINVAL, ENOMEM, ECUDA, ENCCL, ESTATE, EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
U8, F32 = 1, 2
WRAP, CLAMP, ZERO, NO_CHECKS = 0, 1, 2, 3
OP_LIFE, OP_CONV, OP_HISTOGRAM = 0, 1, 2
HALO_EXCHANGE, HALO_WRAP_LOCAL, HALO_CLAMP, HALO_ZERO = 0, 1, 2, 3
OPT_GRAPHS, OPT_GRAPH_ITERS, OPT_NO_EXCHANGE, OPT_TIMING, OPT_PERSISTENT, OPT_EXCHANGE, OPT_DEEP_HALO = 1, 2, 3, 4, 5, 6, 7
OPT_OWN_STREAM = 8
OPT_EXCHANGE_SMS = 9
OPT_HOST_PACKED = 10
EXCHANGE_COPY, EXCHANGE_P2P, EXCHANGE_CE = 0, 1, 2

BOUNDARY = {"wrap": WRAP, "clamp": CLAMP, "zero": ZERO, "no_checks": NO_CHECKS}

EXPORTED = [
    "mapsm_plan_query", "mapsm_ctx_create", "mapsm_ctx_create_local", "mapsm_ctx_destroy",
    "mapsm_nccl_unique_id", "mapsm_grid_create", "mapsm_window_set", "mapsm_op_set", "mapsm_grid_slab",
    "mapsm_bind", "mapsm_iterate", "mapsm_sync", "mapsm_gather", "mapsm_read", "mapsm_histogram", "mapsm_grid_destroy",
    "mapsm_get_info", "mapsm_set_option", "mapsm_get_timing", "mapsm_grid_stream", "mapsm_status_string",
    "mapsm_last_error", "mapsm_version", "mapsm_locmon_create", "mapsm_locmon_destroy", "mapsm_locmon_output",
    "mapsm_locmon_query", "mapsm_locmon_copied", "mapsm_task_histogram", "mapsm_gather_async",
    "mapsm_grid_create_3d", "mapsm_matrix_create", "mapsm_matrix_destroy", "mapsm_matrix_bind",
    "mapsm_invoke_unmodified", "mapsm_matrix_sync", "mapsm_matrix_gather", "mapsm_routine_sgemm",
    "mapsm_routine_saxpy", "mapsm_launch_query", "mapsm_exchange_plan", "mapsm_gather_plan",
    "mapsm_bind_async", "mapsm_read_async",
]
MSG_SEND, MSG_RECV = 0, 1
(KERNEL_NONE, KERNEL_LIFE_TMA, KERNEL_LIFE_REG, KERNEL_LIFE_ANYW, KERNEL_LIFE_PERSIST, KERNEL_LIFE_TB,
 KERNEL_CONV_TMA, KERNEL_CONV_REG, KERNEL_CONV_GENERIC, KERNEL_CONV_WIDE, KERNEL_CONV3D,
 KERNEL_LIFE_TB_PERSIST, KERNEL_CONV_TB2) = range(13)
KERNEL_NAMES = {0: "none", 1: "life_tma_kernel", 2: "life_step_kernel", 3: "life_anyw_kernel",
                4: "life_persist_kernel", 5: "life_tb_kernel", 6: "conv_tma_kernel", 7: "conv_step_kernel",
                8: "conv_generic_kernel", 9: "conv_wide_kernel", 10: "conv3d_kernel", 11: "life_tb_persist_kernel",
                12: "conv_tb2_kernel"}
MAX_DIMS = 3
MAX_PARAMS = 8
PAT_BLOCK2D, PAT_BLOCK2D_T, PAT_OUT_SI, PAT_INOUT_SI = 0, 1, 2, 3


class MapsmError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: {status} {detail}")
        self.status = status


class mapsm_slab_plan(ctypes.Structure):
    _fields_ = [("y0", ctypes.c_int64), ("rows", ctypes.c_int64), ("up", ctypes.c_int), ("down", ctypes.c_int),
                ("top_kind", ctypes.c_int), ("bottom_kind", ctypes.c_int), ("top_src_row", ctypes.c_int64),
                ("bottom_src_row", ctypes.c_int64), ("n_send", ctypes.c_int), ("n_recv", ctypes.c_int),
                ("alloc_rows", ctypes.c_int64)]


class mapsm_grid_info(ctypes.Structure):
    _fields_ = [("w", ctypes.c_int64), ("h", ctypes.c_int64), ("dtype", ctypes.c_int), ("op", ctypes.c_int),
                ("radius", ctypes.c_int), ("boundary", ctypes.c_int), ("world", ctypes.c_int),
                ("local_slabs", ctypes.c_int), ("pitch_bytes", ctypes.c_int64), ("generation", ctypes.c_int64),
                ("launches", ctypes.c_int64), ("exchanges", ctypes.c_int64), ("device_bytes", ctypes.c_int64),
                ("used_graphs", ctypes.c_int), ("gens_per_pass", ctypes.c_int), ("halo_rows", ctypes.c_int64),
                ("d", ctypes.c_int64)]


class mapsm_msg(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("peer", ctypes.c_int), ("row", ctypes.c_int64), ("rows", ctypes.c_int64),
                ("offset", ctypes.c_int64), ("bytes", ctypes.c_int64), ("global_row", ctypes.c_int64)]


class mapsm_launch_info(ctypes.Structure):
    _fields_ = [("kernel", ctypes.c_int), ("threads", ctypes.c_int), ("smem_bytes", ctypes.c_int),
                ("ring_stages", ctypes.c_int), ("rows_per_stage", ctypes.c_int), ("consumer_warps", ctypes.c_int),
                ("gens_per_launch", ctypes.c_int), ("ctas", ctypes.c_int64), ("strips", ctypes.c_int64),
                ("min_cta_seg_rows", ctypes.c_int64), ("max_cta_seg_rows", ctypes.c_int64),
                ("min_cta_rows", ctypes.c_int64), ("segments", ctypes.c_int64)]


class mapsm_box(ctypes.Structure):
    _fields_ = [("lo", ctypes.c_int64 * MAX_DIMS), ("hi", ctypes.c_int64 * MAX_DIMS)]


class mapsm_copy_op(ctypes.Structure):
    _fields_ = [("src", ctypes.c_int), ("dst", ctypes.c_int), ("box", mapsm_box)]


class mapsm_segment(ctypes.Structure):
    _fields_ = [("row0", ctypes.c_int64), ("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("ld", ctypes.c_int64),
                ("ptr", ctypes.c_void_p)]


# int routine(void* context, int slab, int device, void* stream, const mapsm_segment*, int, const float*, int)
ROUTINE = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                           ctypes.POINTER(mapsm_segment), ctypes.c_int, ctypes.POINTER(ctypes.c_float), ctypes.c_int)

_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} is missing: build it with `python -m paper_conf_sc_ben_nunlbr15_b200.build` "
                          "(no CPU fallback exists)")
    L = ctypes.CDLL(_LIB_PATH)
    i64, ci, vp = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p
    P = ctypes.POINTER
    sig = {
        "mapsm_plan_query": [i64, ci, ci, ci, ci, P(mapsm_slab_plan)],
        "mapsm_exchange_plan": [i64, ci, ci, ci, ci, i64, i64, i64, P(mapsm_msg), ci, P(ci)],
        "mapsm_gather_plan": [i64, ci, ci, ci, ci, ci, i64, i64, P(mapsm_msg), ci, P(ci)],
        "mapsm_ctx_create": [ci, ci, ci, vp, vp, P(vp)],
        "mapsm_ctx_create_local": [ci, P(ci), P(vp)],
        "mapsm_ctx_destroy": [vp],
        "mapsm_nccl_unique_id": [vp],
        "mapsm_grid_create": [vp, i64, i64, ci, P(vp)],
        "mapsm_window_set": [vp, ci, ci],
        "mapsm_op_set": [vp, ci, vp],
        "mapsm_grid_slab": [vp, ci, P(i64), P(i64)],
        "mapsm_bind": [vp, vp, i64],
        "mapsm_bind_async": [vp, vp, i64],
        "mapsm_read_async": [vp, vp, i64],
        "mapsm_iterate": [vp, i64],
        "mapsm_sync": [vp],
        "mapsm_gather": [vp, vp, i64, ci],
        "mapsm_read": [vp, vp, i64],
        "mapsm_histogram": [vp, vp, ci],
        "mapsm_grid_destroy": [vp],
        "mapsm_get_info": [vp, P(mapsm_grid_info)],
        "mapsm_set_option": [vp, ci, i64],
        "mapsm_get_timing": [vp, P(ctypes.c_double), P(i64), P(ctypes.c_double), P(i64)],
        "mapsm_grid_stream": [vp, ci, P(vp)],
        "mapsm_launch_query": [vp, ci, ci, P(mapsm_launch_info)],
        "mapsm_locmon_create": [ci, P(vp)],
        "mapsm_locmon_destroy": [vp],
        "mapsm_locmon_output": [vp, ci, ci, P(ci), P(mapsm_box), ci],
        "mapsm_locmon_query": [vp, ci, P(mapsm_box), ci, P(mapsm_copy_op), ci, P(ci), P(ci)],
        "mapsm_locmon_copied": [vp, ci, ci, P(mapsm_copy_op)],
        "mapsm_task_histogram": [vp, ci, vp, ci, P(i64)],
        "mapsm_gather_async": [vp, vp, i64, ci],
        "mapsm_grid_create_3d": [vp, i64, i64, i64, ci, P(vp)],
        "mapsm_matrix_create": [vp, i64, i64, P(vp)],
        "mapsm_matrix_destroy": [vp],
        "mapsm_matrix_bind": [vp, vp, i64],
        "mapsm_invoke_unmodified": [vp, i64, vp, vp, ci, P(vp), P(ci), P(ctypes.c_float), ci, P(i64)],
        "mapsm_matrix_sync": [vp],
        "mapsm_matrix_gather": [vp, vp, i64, ci],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = ci
    L.mapsm_status_string.argtypes = [ci]
    L.mapsm_status_string.restype = ctypes.c_char_p
    L.mapsm_last_error.argtypes = []
    L.mapsm_last_error.restype = ctypes.c_char_p
    L.mapsm_version.argtypes = []
    L.mapsm_version.restype = ctypes.c_char_p
    _lib = L
    return L


def _check(status: int, where: str) -> None:
    if status != OK:
        L = lib()
        raise MapsmError(status, where, f"{L.mapsm_status_string(status).decode()}: {L.mapsm_last_error().decode()}")


def _ptr(buf) -> int:
    """Address of a numpy array, torch tensor (host or device) or int."""
    if isinstance(buf, int):
        return buf
    if isinstance(buf, np.ndarray):
        return buf.ctypes.data
    if hasattr(buf, "data_ptr"):
        return buf.data_ptr()
    raise TypeError(f"unsupported buffer type {type(buf)}")


def _pitch(buf, default: int) -> int:
    if isinstance(buf, np.ndarray):
        return buf.strides[0]
    if hasattr(buf, "stride") and hasattr(buf, "element_size"):
        return buf.stride(0) * buf.element_size()
    return default


# ---------------------------------------------------------------- C-named API

def mapsm_plan_query(h: int, g: int, radius: int, boundary: int, rank: int) -> mapsm_slab_plan:
    p = mapsm_slab_plan()
    _check(lib().mapsm_plan_query(h, g, radius, boundary, rank, ctypes.byref(p)), "mapsm_plan_query")
    return p


def mapsm_exchange_plan(h: int, g: int, radius: int, boundary: int, rank: int, depth: int, halo: int,
                        pitch: int) -> list[mapsm_msg]:
    """The ordered halo-exchange messages of slab `rank` for one pass."""
    out = (mapsm_msg * 4)()
    n = ctypes.c_int()
    _check(lib().mapsm_exchange_plan(h, g, radius, boundary, rank, depth, halo, pitch, out, 4, ctypes.byref(n)),
           "mapsm_exchange_plan")
    return [out[i] for i in range(n.value)]


def mapsm_gather_plan(h: int, g: int, radius: int, boundary: int, rank: int, root: int, halo: int,
                      pitch: int) -> list[mapsm_msg]:
    """The gather-to-root messages of slab `rank`."""
    cap = max(1, g)
    out = (mapsm_msg * cap)()
    n = ctypes.c_int()
    _check(lib().mapsm_gather_plan(h, g, radius, boundary, rank, root, halo, pitch, out, cap, ctypes.byref(n)),
           "mapsm_gather_plan")
    return [out[i] for i in range(n.value)]


def mapsm_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().mapsm_nccl_unique_id(buf), "mapsm_nccl_unique_id")
    return buf.raw


def mapsm_ctx_create(rank: int, world: int, device: int, nccl_unique_id: bytes | None = None,
                     cuda_stream: int | None = None) -> int:
    """One rank of `world` (include/mapsm.h).  world > 1 needs the rank-0
    mapsm_nccl_unique_id(); world == 1 with an id = the one-rank NCCL ring
    (WRAP halos through ncclSend/ncclRecv to the rank itself)."""
    out = ctypes.c_void_p()
    uid = ctypes.create_string_buffer(nccl_unique_id, 128) if nccl_unique_id is not None else None
    _check(lib().mapsm_ctx_create(rank, world, device, uid, cuda_stream, ctypes.byref(out)), "mapsm_ctx_create")
    return out.value


def mapsm_ctx_create_local(devices) -> int:
    arr = (ctypes.c_int * len(devices))(*devices)
    out = ctypes.c_void_p()
    _check(lib().mapsm_ctx_create_local(len(devices), arr, ctypes.byref(out)), "mapsm_ctx_create_local")
    return out.value


def mapsm_ctx_destroy(ctx: int) -> None:
    _check(lib().mapsm_ctx_destroy(ctx), "mapsm_ctx_destroy")


def mapsm_grid_create(ctx: int, w: int, h: int, dtype: int) -> int:
    out = ctypes.c_void_p()
    _check(lib().mapsm_grid_create(ctx, w, h, dtype, ctypes.byref(out)), "mapsm_grid_create")
    return out.value


def mapsm_grid_create_3d(ctx: int, w: int, h: int, d: int, dtype: int = F32) -> int:
    out = ctypes.c_void_p()
    _check(lib().mapsm_grid_create_3d(ctx, w, h, d, dtype, ctypes.byref(out)), "mapsm_grid_create_3d")
    return out.value


def mapsm_window_set(grid: int, radius: int, boundary: int) -> None:
    _check(lib().mapsm_window_set(grid, radius, boundary), "mapsm_window_set")


def mapsm_op_set(grid: int, op: int, weights=None) -> None:
    wptr = None
    if weights is not None:
        w = np.ascontiguousarray(weights, dtype=np.float32)
        wptr = w.ctypes.data
        _check(lib().mapsm_op_set(grid, op, wptr), "mapsm_op_set")
        return
    _check(lib().mapsm_op_set(grid, op, None), "mapsm_op_set")


def mapsm_grid_slab(grid: int, local_index: int = 0) -> tuple[int, int]:
    y0, rows = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().mapsm_grid_slab(grid, local_index, ctypes.byref(y0), ctypes.byref(rows)), "mapsm_grid_slab")
    return y0.value, rows.value


def mapsm_bind(grid: int, buf, row_pitch_bytes: int | None = None) -> None:
    _check(lib().mapsm_bind(grid, _ptr(buf), row_pitch_bytes or _pitch(buf, 0)), "mapsm_bind")


def mapsm_bind_async(grid: int, buf, row_pitch_bytes: int | None = None) -> None:
    """Stream-ordered Bind: `buf` (pinned host or device) must stay valid until mapsm_sync."""
    _check(lib().mapsm_bind_async(grid, _ptr(buf), row_pitch_bytes or _pitch(buf, 0)), "mapsm_bind_async")


def mapsm_iterate(grid: int, n: int) -> None:
    _check(lib().mapsm_iterate(grid, n), "mapsm_iterate")


def mapsm_sync(grid: int) -> None:
    _check(lib().mapsm_sync(grid), "mapsm_sync")


def mapsm_gather(grid: int, buf, row_pitch_bytes: int | None = None, root: int = 0) -> None:
    p = None if buf is None else _ptr(buf)
    pitch = row_pitch_bytes or (0 if buf is None else _pitch(buf, 0))
    _check(lib().mapsm_gather(grid, p, pitch, root), "mapsm_gather")


def mapsm_gather_async(grid: int, buf, row_pitch_bytes: int | None = None, root: int = 0) -> None:
    """GatherAsync: enqueue only; `buf` is complete after mapsm_sync."""
    p = None if buf is None else _ptr(buf)
    pitch = row_pitch_bytes or (0 if buf is None else _pitch(buf, 0))
    _check(lib().mapsm_gather_async(grid, p, pitch, root), "mapsm_gather_async")


def mapsm_read(grid: int, buf, row_pitch_bytes: int | None = None) -> None:
    _check(lib().mapsm_read(grid, _ptr(buf), row_pitch_bytes or _pitch(buf, 0)), "mapsm_read")


def mapsm_read_async(grid: int, buf, row_pitch_bytes: int | None = None) -> None:
    """Stream-ordered read of this process's rows: `buf` is complete after mapsm_sync."""
    _check(lib().mapsm_read_async(grid, _ptr(buf), row_pitch_bytes or _pitch(buf, 0)), "mapsm_read_async")


def _is_cuda_tensor(buf) -> bool:
    return bool(getattr(buf, "is_cuda", False))


def mapsm_histogram(grid: int, bins=None, sync: bool = True) -> np.ndarray:
    """Reductive-Static aggregate: 256 uint64 counts (into `bins` if given:
    a numpy array or a torch tensor, host or device).  For a device tensor
    the C call is stream-ordered on the grid's stream; with sync=True (the
    default) this wrapper waits for it (mapsm_sync) so the counts can be read
    on any stream; sync=False leaves them pending (read after mapsm_sync)."""
    out = np.zeros(256, dtype=np.uint64) if bins is None else bins
    _check(lib().mapsm_histogram(grid, _ptr(out), 256), "mapsm_histogram")
    if sync and _is_cuda_tensor(out):
        mapsm_sync(grid)
    return out


def mapsm_task_histogram(grid: int, target_slabs: int = 0, bins=None, sync: bool = True) -> tuple[np.ndarray, int]:
    """Chained Reductive-Static task over the grid's current generation with
    its own partition (0 = the grid's); returns (bins, bytes moved here).
    Device-tensor bins: as mapsm_histogram (sync=False leaves them pending)."""
    out = np.zeros(256, dtype=np.uint64) if bins is None else bins
    moved = ctypes.c_int64()
    _check(lib().mapsm_task_histogram(grid, target_slabs, _ptr(out), 256, ctypes.byref(moved)),
           "mapsm_task_histogram")
    if sync and _is_cuda_tensor(out):
        mapsm_sync(grid)
    return out, moved.value


# Segment Location Monitor (Alg 2).  Boxes are given as sequences of (lo, hi)
# pairs, one per dimension (missing dimensions are [0, 1)).

def _box(b) -> mapsm_box:
    x = mapsm_box()
    for d in range(MAX_DIMS):
        lo, hi = (b[d] if d < len(b) else (0, 1))
        x.lo[d], x.hi[d] = lo, hi
    return x


def _unbox(x: mapsm_box, nd: int) -> tuple:
    return tuple((x.lo[d], x.hi[d]) for d in range(nd))


def mapsm_locmon_create(ndims: int) -> int:
    out = ctypes.c_void_p()
    _check(lib().mapsm_locmon_create(ndims, ctypes.byref(out)), "mapsm_locmon_create")
    return out.value


def mapsm_locmon_destroy(m: int) -> None:
    _check(lib().mapsm_locmon_destroy(m), "mapsm_locmon_destroy")


def mapsm_locmon_output(m: int, datum: int, segs, needs_aggregation: bool = False) -> None:
    """segs: [(location, box), ...]"""
    n = len(segs)
    locs = (ctypes.c_int * max(n, 1))(*[l for l, _ in segs])
    boxes = (mapsm_box * max(n, 1))(*[_box(b) for _, b in segs])
    _check(lib().mapsm_locmon_output(m, datum, n, locs, boxes, int(needs_aggregation)), "mapsm_locmon_output")


def mapsm_locmon_query(m: int, datum: int, required, target: int, nd: int = 2) -> tuple[list, bool]:
    """Alg 2: ([(src, dst, box), ...], needs_aggregation)."""
    req = _box(required)
    n, agg = ctypes.c_int(), ctypes.c_int()
    cap = 16
    while True:
        ops = (mapsm_copy_op * cap)()
        st = lib().mapsm_locmon_query(m, datum, ctypes.byref(req), target, ops, cap, ctypes.byref(n),
                                      ctypes.byref(agg))
        if st == ENOMEM and n.value > cap:
            cap = n.value
            continue
        _check(st, "mapsm_locmon_query")
        return [(ops[i].src, ops[i].dst, _unbox(ops[i].box, nd)) for i in range(n.value)], bool(agg.value)


def mapsm_locmon_copied(m: int, datum: int, ops) -> None:
    n = len(ops)
    arr = (mapsm_copy_op * max(n, 1))()
    for i, (src, dst, b) in enumerate(ops):
        arr[i].src, arr[i].dst, arr[i].box = src, dst, _box(b)
    _check(lib().mapsm_locmon_copied(m, datum, n, arr), "mapsm_locmon_copied")


# Unmodified routines (NEXT-4): fp32 matrix datums and InvokeUnmodified.

def mapsm_matrix_create(ctx: int, rows: int, cols: int) -> int:
    out = ctypes.c_void_p()
    _check(lib().mapsm_matrix_create(ctx, rows, cols, ctypes.byref(out)), "mapsm_matrix_create")
    return out.value


def mapsm_matrix_destroy(m: int) -> None:
    _check(lib().mapsm_matrix_destroy(m), "mapsm_matrix_destroy")


def mapsm_matrix_bind(m: int, buf, ld: int | None = None) -> None:
    _check(lib().mapsm_matrix_bind(m, _ptr(buf), ld or _pitch(buf, 0) // 4), "mapsm_matrix_bind")


def mapsm_matrix_sync(m: int) -> None:
    _check(lib().mapsm_matrix_sync(m), "mapsm_matrix_sync")


def mapsm_matrix_gather(m: int, buf, ld: int | None = None, root: int = 0) -> None:
    p = None if buf is None else _ptr(buf)
    _check(lib().mapsm_matrix_gather(m, p, ld or (0 if buf is None else _pitch(buf, 0) // 4), root),
           "mapsm_matrix_gather")


def routine_ptr(routine) -> int:
    """'sgemm' / 'saxpy' (built-in cuBLAS wrappers), a ROUTINE callback, or an address."""
    if isinstance(routine, str):
        return ctypes.cast(getattr(lib(), f"mapsm_routine_{routine}"), ctypes.c_void_p).value
    if isinstance(routine, ROUTINE):
        return ctypes.cast(routine, ctypes.c_void_p).value
    return int(routine)


def mapsm_invoke_unmodified(ctx: int, task_rows: int, routine, params, patterns, scalars=(), context=None) -> int:
    """Run `routine` per slab on the segments the patterns imply; returns bytes moved."""
    n = len(params)
    P = (ctypes.c_void_p * n)(*params)
    pats = (ctypes.c_int * n)(*patterns)
    sc = (ctypes.c_float * max(1, len(scalars)))(*scalars)
    moved = ctypes.c_int64()
    _check(lib().mapsm_invoke_unmodified(ctx, task_rows, routine_ptr(routine), context, n, P, pats, sc,
                                         len(scalars), ctypes.byref(moved)), "mapsm_invoke_unmodified")
    return moved.value


def mapsm_grid_destroy(grid: int) -> None:
    _check(lib().mapsm_grid_destroy(grid), "mapsm_grid_destroy")


def mapsm_get_info(grid: int) -> mapsm_grid_info:
    info = mapsm_grid_info()
    _check(lib().mapsm_get_info(grid, ctypes.byref(info)), "mapsm_get_info")
    return info


def mapsm_set_option(grid: int, opt: int, value: int) -> None:
    _check(lib().mapsm_set_option(grid, opt, value), "mapsm_set_option")


def mapsm_get_timing(grid: int) -> tuple[float, int, float, int]:
    a, b = ctypes.c_double(), ctypes.c_int64()
    c, d = ctypes.c_double(), ctypes.c_int64()
    _check(lib().mapsm_get_timing(grid, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c), ctypes.byref(d)),
           "mapsm_get_timing")
    return a.value, b.value, c.value, d.value


def mapsm_grid_stream(grid: int, local_index: int = 0) -> int:
    out = ctypes.c_void_p()
    _check(lib().mapsm_grid_stream(grid, local_index, ctypes.byref(out)), "mapsm_grid_stream")
    return out.value or 0


def mapsm_launch_query(grid: int, local_index: int = 0, which: int = 0) -> mapsm_launch_info:
    """Geometry of the last bulk (which=0) or boundary (which=1) launch."""
    out = mapsm_launch_info()
    _check(lib().mapsm_launch_query(grid, local_index, which, ctypes.byref(out)), "mapsm_launch_query")
    return out


def mapsm_version() -> str:
    return lib().mapsm_version().decode()


# ------------------------------------------------------------ convenience

class Grid:
    """One datum with its Window(2D) pattern — create -> window_set -> op_set ->
    bind -> iterate -> gather, as in Fig 2a."""

    def __init__(self, ctx: int, w: int, h: int, op: str = "life", radius: int = 1, boundary: str = "wrap",
                 weights=None, deep_halo: int = 1, d: int = 0):
        """d > 0: a Window(3D) d x h x w fp32 volume (op "conv", (2r+1)^3 weights)."""
        self.ctx, self.w, self.h, self.d = ctx, w, h, d
        self.op = op
        self.dtype = F32 if op == "conv" else U8
        if op == "histogram":
            radius, boundary = 0, "no_checks"
        self.handle = (mapsm_grid_create_3d(ctx, w, h, d, self.dtype) if d else
                       mapsm_grid_create(ctx, w, h, self.dtype))
        try:
            mapsm_window_set(self.handle, radius, BOUNDARY[boundary] if isinstance(boundary, str) else boundary)
            if deep_halo > 1:
                mapsm_set_option(self.handle, OPT_DEEP_HALO, deep_halo)
            if op == "life":
                mapsm_op_set(self.handle, OP_LIFE, None)
            elif op == "histogram":
                mapsm_op_set(self.handle, OP_HISTOGRAM, None)
            else:
                mapsm_op_set(self.handle, OP_CONV, weights)
        except Exception:
            mapsm_grid_destroy(self.handle)
            raise

    def local_rows(self) -> tuple[int, int]:
        """(y0, rows) of this process's rows (all local slabs)."""
        info = mapsm_get_info(self.handle)
        y0, _ = mapsm_grid_slab(self.handle, 0)
        ylast, rlast = mapsm_grid_slab(self.handle, info.local_slabs - 1)
        return y0, ylast + rlast - y0

    def bind(self, buf, pitch: int | None = None):
        mapsm_bind(self.handle, buf, pitch or self._rp(buf))

    def iterate(self, n: int):
        mapsm_iterate(self.handle, n)

    def sync(self):
        mapsm_sync(self.handle)

    def read(self, out=None):
        y0, rows = self.local_rows()
        if out is None:
            shape = (rows, self.h, self.w) if self.d else (rows, self.w)
            out = np.empty(shape, dtype=np.uint8 if self.dtype == U8 else np.float32)
        mapsm_read(self.handle, out, self._rp(out))
        return out

    def _rp(self, buf):
        """Row pitch of a (planes, h, w) volume buffer (None = the binding's default for 2-D)."""
        if not self.d or buf is None:
            return None
        return buf.strides[1] if isinstance(buf, np.ndarray) else buf.stride(1) * buf.element_size()

    def gather(self, out=None, root: int = 0, rank: int = 0):
        if out is None and rank == root:
            shape = (self.d, self.h, self.w) if self.d else (self.h, self.w)
            out = np.empty(shape, dtype=np.uint8 if self.dtype == U8 else np.float32)
        mapsm_gather(self.handle, out, self._rp(out), root)
        return out

    def histogram(self, bins=None):
        return mapsm_histogram(self.handle, bins)

    def task_histogram(self, target_slabs: int = 0, bins=None):
        return mapsm_task_histogram(self.handle, target_slabs, bins)

    def gather_async(self, out, root: int = 0):
        mapsm_gather_async(self.handle, out, self._rp(out), root)
        return out

    def info(self) -> mapsm_grid_info:
        return mapsm_get_info(self.handle)

    def launch(self, which: int = 0, local_index: int = 0) -> mapsm_launch_info:
        return mapsm_launch_query(self.handle, local_index, which)

    def set_option(self, opt: int, value: int):
        mapsm_set_option(self.handle, opt, value)

    def close(self):
        if self.handle:
            mapsm_grid_destroy(self.handle)
            self.handle = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
