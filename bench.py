"""bench.py — Game of Life cell-updates/s and % HBM roofline on 1..8 B200.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` (torchrun
for N > 1) prints ONE JSON line on rank 0.  Default workload = BASELINE.json
configs[2] at N=1 (``life64k``); ``--workload`` selects the other configs
(``life8k``, ``conv5``, ``conv9``) and the §8(f) NEXT-1 histogram (``hist8k``).

* step      = one pass of the hot path over the resident grid: for the stencils
              one ``mapsm_iterate(grid, n)`` call (n generations: boundary rows,
              halo exchange when N > 1, interior, buffer swap); for the histogram
              one ``mapsm_histogram`` (per-slab bins, cross-GPU aggregation).
* value     = work units (cell-updates or pixels) of all ranks in K steps / the
              max-over-ranks device time of the K steps (CUDA events on the
              library's compute stream; L2 flushed between steps outside the
              events).
* e2e       = the same metric through the public C ABI with pinned HOST buffers
              and the host<->device copies inside the timed region (mapsm_bind
              of the host rows, the step, mapsm_read / histogram to host).
* roofline  = the dominant kernel vs the measured HBM copy bandwidth
              (MEASURED_PEAKS.json hbm_gbs); algorithmic bytes: 0.25 B per Life
              cell-update, 8 B per conv cell-update, 1 B per histogram pixel.
* cpu_baseline = the CPU oracle (oracle/, OpenMP) timed on a bounded sample of
              the same workload on rank 0 only.
* deep_halo = (Life) the same workload on the deep-halo path (MAPSM_OPT_DEEP_HALO
              = --deep-halo K, default 8: K generations per pass of the
              temporally blocked kernel, K-row halos exchanged once per pass),
              reported separately with its ALU-pipe roofline.
``--impl reference`` times only the oracle (this tier's reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    "life64k": dict(op="life", w=65536, h=65536, r=1, b="wrap", n=200, seed=0x5EED0003, wseed=None,
                    scaling="strong", bcell=0.25,
                    label="Game of Life 65536x65536 WRAP, random p=0.5 (splitmix64 seed 0x5EED0003), "
                          "200 generations per step (BASELINE configs[2])"),
    "life8k": dict(op="life", w=8192, h=8192, r=1, b="wrap", n=1000, seed=0x5EED0002, wseed=None,
                   scaling="strong", bcell=0.25,
                   label="Game of Life 8192x8192 WRAP, random p=0.5 (seed 0x5EED0002), 1000 generations per step "
                         "(BASELINE configs[1]; L2-resident)"),
    "conv5": dict(op="conv", w=16384, h=16384, r=2, b="clamp", n=500, seed=0x5EED0004, wseed=0x5EED0044,
                  scaling="strong", bcell=8.0,
                  label="fp32 5x5 window convolution 16384x16384 CLAMP, 500 iterations per step (BASELINE configs[3])"),
    "conv9": dict(op="conv", w=32768, h=4096, r=4, b="zero", n=100, seed=0x5EED0005, wseed=0x5EED0055,
                  scaling="weak", bcell=8.0,
                  label="fp32 9x9 (r=4) window stencil, 32768 wide x 4096 rows per GPU, ZERO, 100 iterations per "
                        "step (BASELINE configs[4], weak scaling)"),
    "conv9sq": dict(op="conv", w=32768, h=32768, r=4, b="zero", n=100, seed=0x5EED0005, wseed=0x5EED0055,
                    scaling="weak", bcell=8.0,
                    label="fp32 9x9 (r=4) window stencil, 32768x32768 per GPU, ZERO, 100 iterations per step "
                          "(BASELINE configs[4], SURVEY 8(d) alternative reading: 32768^2 per GPU)"),
    "conv3d": dict(op="conv", w=512, h=512, d=512, r=1, b="zero", n=100, seed=0x5EED0007, wseed=0x5EED0077,
                   scaling="strong", bcell=8.0,
                   label="fp32 3x3x3 Window(3D) convolution 512x512x512 ZERO, 100 iterations per step (SURVEY "
                         "§8(f) NEXT-2; plane-slab partition; not a BASELINE config)"),
    "conv3d5": dict(op="conv", w=512, h=512, d=512, r=2, b="clamp", n=20, seed=0x5EED0007, wseed=0x5EED0078,
                    scaling="strong", bcell=8.0,
                    label="fp32 5x5x5 Window(3D) convolution 512x512x512 CLAMP, 20 iterations per step (SURVEY "
                          "§8(f) NEXT-2; FMA-bound; not a BASELINE config)"),
    "sgemm8k": dict(op="sgemm", w=8192, h=8192, r=0, b="none", n=10, seed=0x5EED0008, wseed=None,
                    scaling="weak", bcell=0.0,
                    label="chain of fp32 8192x8192 matrix multiplications C = A B through InvokeUnmodified "
                          "(cuBLAS SGEMM wrapper, Block2D / Block2D-T / SI patterns; the paper's 8K chain, "
                          "P:L491-508; SURVEY §8(f) NEXT-4), 10 multiplications per step"),
    "hist8k": dict(op="histogram", w=8192, h=8192, r=0, b="no_checks", n=1, seed=0x5EED0006, wseed=None,
                   scaling="strong", bcell=1.0,
                   label="256-bin histogram of an 8192x8192 u8 image, uniform pixels (seed 0x5EED0006), one "
                         "Reductive-Static task per step (SURVEY §8(f) NEXT-1; the paper's 8K image, P:L477-479)"),
}


def metric_of(wl):
    if wl["op"] == "sgemm":
        return "fp32 matrix-multiplication FLOP/s (unmodified cuBLAS routine)", "FLOP/s"
    if wl["op"] == "life":
        return "Game of Life cell-updates/s", "cell-updates/s"
    if wl["op"] == "conv":
        k = 2 * wl["r"] + 1
        return f"fp32 {k}x{k} window-conv cell-updates/s", "cell-updates/s"
    return "256-bin histogram pixels/s", "pixels/s"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-lms", "100", "-i", str(self.dev)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        # a timed region shorter than nvidia-smi's start-up (the histogram's
        # ~0.3 ms) has no sample yet: take the first one right after it
        late = not self.lines
        t_end = time.time() + 3.0
        while not self.lines and time.time() < t_end:
            time.sleep(0.01)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        out = {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
               "reasons": sorted(reasons), "samples": len(sm)}
        if late and sm:
            out["note"] = "timed region shorter than the sampling start-up; sampled just after it"
        return out


# ------------------------------------------------------------------ oracle leg

def _oracle_sample(wl):
    """(run(k), work units per iteration, description) for a bounded sample."""
    import mapsm_inputs as mi
    import oracle

    w = wl["w"]
    if wl["op"] == "sgemm":
        from oracle import blas
        import numpy as np

        rows = 512
        rng = np.random.default_rng(wl["seed"])
        a = (rng.random((rows, w), dtype=np.float32) - 0.5)
        bm = (rng.random((w, w), dtype=np.float32) - 0.5)

        def run_mm(k):
            for _ in range(k):
                blas.sgemm(a, bm)
        return run_mm, 2.0 * rows * w * w, f"{rows} x {w} @ {w} x {w} float64 products"
    if wl["op"] == "life":
        rows = 512
        g0 = mi.life_u8(wl["seed"], w, rows)
        return (lambda k: oracle.life(g0, k, wl["b"])), w * rows, f"{w} x {rows} rows"
    if wl["op"] == "conv" and wl.get("d"):
        planes = 8
        v0 = mi.volume_f32(wl["seed"], w, wl["h"], planes)
        W = mi.weights3d_f32(wl["wseed"], wl["r"])
        return (lambda k: oracle.conv3d(v0, W, k, wl["b"])), w * wl["h"] * planes, f"{planes} planes of {wl['h']} x {w}"
    if wl["op"] == "conv":
        rows = 256
        g0 = mi.field_f32(wl["seed"], w, rows)
        W = mi.weights_f32(wl["wseed"], wl["r"])
        return (lambda k: oracle.conv(g0, W, k, wl["b"])), w * rows, f"{w} x {rows} rows"
    img = mi.image_u8(wl["seed"], w, wl["h"])

    def run(k):
        for _ in range(k):
            oracle.histogram(img)
    return run, w * wl["h"], f"the full {w} x {wl['h']} image"


def _oracle_threads(wl):
    import oracle

    if wl["op"] == "sgemm":
        return os.cpu_count()  # numpy's BLAS threads
    return 1 if wl["op"] == "histogram" else oracle.num_threads()  # the histogram oracle is sequential


def cpu_baseline(wl, budget_s=12.0):
    """Time the oracle (as it stands) on a bounded sample of the workload."""
    run, units, what = _oracle_sample(wl)
    t0 = time.perf_counter()
    run(1)
    t1 = time.perf_counter() - t0
    cap = wl["n"] if wl["op"] != "histogram" else 50
    n = max(1, min(cap, int(budget_s / max(t1, 1e-6))))
    t0 = time.perf_counter()
    run(n)
    dt = time.perf_counter() - t0
    _, unit = metric_of(wl)
    return {"value": units * n / dt, "unit": unit, "cores": _oracle_threads(wl), "kind": "oracle",
            "sample": f"{what} of the same {wl['op']} workload ({wl['b']} boundary on the sample), {n} iterations, "
                      f"{dt:.1f} s wall (oracle/oracle.c)"}


def run_sgemm(args, wl, rank, world, local_rank):
    """NEXT-4 measurement: a chain of C = A B (m = 8192 rows per GPU, weak)
    through mapsm_invoke_unmodified with the cuBLAS SGEMM wrapper; A, B
    resident (the Location Monitor moves nothing after the first call)."""
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    uid = None
    if world > 1:
        obj = [M.mapsm_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    ctx = M.mapsm_ctx_create(rank, world, local_rank, uid, stream.cuda_stream)
    k = n = wl["w"]
    m = wl["h"] * world
    chain = wl["n"]
    g = torch.Generator().manual_seed(wl["seed"])
    hA = (torch.rand((m, k), generator=g) - 0.5).pin_memory()
    hB = (torch.rand((k, n), generator=g) - 0.5).pin_memory()
    hC = torch.empty((m, n), dtype=torch.float32).pin_memory()
    A = M.mapsm_matrix_create(ctx, m, k)
    B = M.mapsm_matrix_create(ctx, k, n)
    C = M.mapsm_matrix_create(ctx, m, n)
    M.mapsm_matrix_bind(A, hA)
    M.mapsm_matrix_bind(B, hB)
    pats = [M.PAT_BLOCK2D, M.PAT_BLOCK2D_T, M.PAT_OUT_SI]

    def step():
        moved = 0
        for _ in range(chain):
            moved += M.mapsm_invoke_unmodified(ctx, m, "sgemm", [A, B, C], pats, (1.0, 0.0))
        return moved

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local_rank])
        torch.cuda.synchronize()

    first_moved = M.mapsm_invoke_unmodified(ctx, m, "sgemm", [A, B, C], pats, (1.0, 0.0))
    for _ in range(args.warmup):
        step()
    barrier()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    sampler = ClockSampler(local_rank)
    sampler.start()
    total_ms, moved = 0.0, 0
    barrier()
    for _ in range(args.steps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        moved += step()
        e1.record(stream)
        e1.synchronize()
        total_ms += e0.elapsed_time(e1)
    barrier()
    clocks = sampler.stop()
    t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms = float(t.item())
    flop_step = 2.0 * m * n * k * chain
    value = flop_step * args.steps / (total_ms / 1e3)
    # e2e: host matrices bound, chain, gather C to pinned host memory
    e2e_ms = 0.0
    for _ in range(args.e2e_steps):
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        M.mapsm_matrix_bind(A, hA)
        M.mapsm_matrix_bind(B, hB)
        step()
        M.mapsm_matrix_gather(C, hC if rank == 0 else None)
        e1.record(stream)
        e1.synchronize()
        e2e_ms += e0.elapsed_time(e1)
    te = torch.tensor([e2e_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_value = flop_step * args.e2e_steps / (float(te.item()) / 1e3)
    for h in (A, B, C):
        M.mapsm_matrix_destroy(h)
    M.mapsm_ctx_destroy(ctx)
    if rank == 0:
        sm_mhz = clocks.get("sm_mhz") or 1965.0
        peak = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12
        ach = value / world / 1e12
        cb = None
        if not args.no_cpu_baseline:
            from oracle import blas

            rows = 512
            a = hA[:rows].numpy()
            b = hB.numpy()
            t0 = time.perf_counter()
            reps = 0
            while time.perf_counter() - t0 < 8.0 or reps == 0:
                blas.sgemm(a, b)
                reps += 1
            dt = time.perf_counter() - t0
            cb = {"value": 2.0 * rows * n * k * reps / dt, "unit": "FLOP/s", "cores": os.cpu_count(),
                  "kind": "oracle", "sample": f"{rows} x {k} @ {k} x {n} in float64 (oracle/blas.py, numpy), "
                                              f"{reps} reps, {dt:.1f} s"}
        line = {"metric": metric_of(wl)[0], "value": value, "unit": "FLOP/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": wl["label"], "m": m, "n": n, "k": k, "multiplications_per_step": chain,
                           "parallelism": f"row-slab x{world}",
                           "l2": "L2 flushed between steps (256 MiB write); 768 MiB of operands per GPU"},
                "e2e": {"value": e2e_value, "unit": "FLOP/s", "h2d_bytes_per_step": 4 * (m * k + k * n) * world,
                        "d2h_bytes_per_step": 4 * m * n,
                        "how": "mapsm_matrix_bind(A, B pinned host) + chain + mapsm_matrix_gather(C -> pinned host)"},
                "gpu_launches": 0,
                "gpu_launches_note": "the kernels are cuBLAS's (an unmodified library routine by design, P:L405)",
                "moved_bytes": {"first_call": int(first_moved), "timed_region": int(moved)},
                "roofline": {"bound": "fma", "kernel": "cuBLAS SGEMM (fp32 CUDA-core FMA, no TF32)", "achieved": ach,
                             "peak": peak, "unit": "TFLOP/s", "frac": ach / peak,
                             "peak_source": "148 SMs x 128 FP32 lanes x 2 flop x sampled SM clock (nominal)"},
                "clocks": clocks, "cpu_baseline": cb,
                "paper_context": "Table 4 P:L503-508: single-GPU 8K multiplication 245-366 ms on GTX 780/Titan "
                                 "Black/GTX 980 (CUBLAS over MAPS-Multi 248.62 ms on GTX 980)"}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier(device_ids=[local_rank])
        dist.destroy_process_group()


def run_reference(args, wl, rank, world):
    """Reference arm of this tier: the oracle as it stands, on the host cores,
    rank 0 only; each step is a bounded sample of the same workload, sized so
    W+K steps take ~1 minute."""
    if rank != 0:
        return
    run, units, what = _oracle_sample(wl)
    t0 = time.perf_counter()
    run(1)
    t1 = time.perf_counter() - t0
    cap = wl["n"] if wl["op"] != "histogram" else 50
    per_step = max(1, min(cap, int(60.0 / max(1, args.steps + args.warmup) / max(t1, 1e-6))))
    for _ in range(args.warmup):
        run(per_step)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        run(per_step)
    dt = time.perf_counter() - t0
    value = units * per_step * args.steps / dt
    metric, unit = metric_of(wl)
    cb = {"value": value, "unit": unit, "cores": _oracle_threads(wl), "kind": "oracle",
          "sample": f"per step: {what}, {per_step} iterations of the same workload; {args.steps} timed steps, "
                    f"{dt:.1f} s"}
    line = {"impl": "reference", "metric": metric, "value": value, "unit": unit,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
            "higher_is_better": True, "scaling": wl["scaling"], "vs_baseline": None,
            "dtype": "f32" if wl["op"] in ("conv", "sgemm") else "u8", "data": "synthetic",
            "config": {"workload": wl["label"]}, "cpu_baseline": cb,
            "e2e": {"value": value, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU leg

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mapsm", choices=["mapsm", "reference"])
    ap.add_argument("--workload", default="life64k", choices=sorted(WORKLOADS))
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--graph-iters", type=int, default=0)
    ap.add_argument("--deep-halo", type=int, default=8,
                    help="Life workloads: also measure the deep-halo path with K generations per pass "
                         "(reported under 'deep_halo'; 0/1 = skip)")
    args = ap.parse_args()
    wl = dict(WORKLOADS[args.workload])

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, wl, rank, world)
        return
    if wl["op"] == "sgemm":
        run_sgemm(args, wl, rank, world, local_rank)
        return

    import torch
    import torch.distributed as dist

    import mapsm_inputs as mi
    from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    # A dedicated (non-default) stream: libmapsm launches on it, and the CUDA
    # events of the timed region are recorded on it.
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    uid = None
    if world > 1:
        obj = [M.mapsm_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    ctx = M.mapsm_ctx_create(rank, world, local_rank, uid, stream.cuda_stream)

    op = wl["op"]
    w = wl["w"]
    h = wl["h"] * (world if wl["scaling"] == "weak" else 1)
    n = wl["n"]
    d = wl.get("d", 0)   # Window(3D): partition units are planes of h rows
    if op == "conv":
        W = mi.weights3d_f32(wl["wseed"], wl["r"]) if d else mi.weights_f32(wl["wseed"], wl["r"])
    else:
        W = None
    grid = M.Grid(ctx, w, h, op, wl["r"], wl["b"], W, d=d)
    cpu_ = w * (h if d else 1)             # cells per partition unit (row or plane)
    cells_total = w * h * (d if d else 1)
    if args.graph_iters:
        grid.set_option(M.OPT_GRAPH_ITERS, args.graph_iters)
    y0, rows = grid.local_rows()
    host_dtype = torch.float32 if op == "conv" else torch.uint8
    # pinned host rows of this rank (input and result buffers for e2e)
    h_in = torch.empty((rows, h, w) if d else (rows, w), dtype=host_dtype, pin_memory=True)
    if d:
        h_in.numpy()[:] = mi.volume_f32(wl["seed"], w, h, rows, z0=y0)
    elif op == "life":
        mi.life_u8(wl["seed"], w, rows, y0=y0, out=h_in.numpy())
    elif op == "conv":
        mi.field_f32(wl["seed"], w, rows, y0=y0, out=h_in.numpy())
    else:
        mi.image_u8(wl["seed"], w, rows, y0=y0, out=h_in.numpy())
    h_out = torch.empty_like(h_in, pin_memory=True) if op != "histogram" else None
    d_bins = torch.zeros(256, dtype=torch.int64, device=dev)
    h_bins = torch.zeros(256, dtype=torch.int64, pin_memory=True)
    grid.bind(h_in)
    info0 = grid.info()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2

    def step():
        if op == "histogram":
            M.mapsm_histogram(grid.handle, d_bins, sync=False)
        else:
            grid.iterate(n)

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local_rank])
        torch.cuda.synchronize()

    # warm-up (graph capture, NCCL connections, clocks)
    for _ in range(args.warmup):
        step()
    barrier()

    # timed region: K steps, L2 flushed between steps outside the events
    sampler = ClockSampler(local_rank)
    sampler.start()
    launches0 = grid.info().launches
    total_ms = 0.0
    barrier()
    for _ in range(args.steps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step()
        e1.record(stream)
        e1.synchronize()
        total_ms += e0.elapsed_time(e1)
    barrier()
    clocks = sampler.stop()
    launches = grid.info().launches - launches0
    used_graphs = bool(grid.info().used_graphs)
    t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
    tl = torch.tensor([launches], dtype=torch.int64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(tl, op=dist.ReduceOp.SUM)
    total_ms = float(t.item())
    total_launches = int(tl.item())
    units_per_step = cells_total * n
    value = units_per_step * args.steps / (total_ms / 1e3)
    ms_per_step = total_ms / args.steps

    peak_gbs, peak_src = load_peaks()
    bcell = wl["bcell"]
    slab_cells = rows * cpu_
    # achieved over the timed region: each stencil step is n back-to-back bulk
    # launches (N == 1), the histogram step one launch (plus its aggregation)
    bulk_launches_per_step = n if op != "histogram" else 1
    per_launch_s = (total_ms / 1e3) / (args.steps * bulk_launches_per_step)
    achieved_region = bcell * slab_cells / per_launch_s / 1e9
    kernel = {"life": "life_tma_kernel", "conv": "conv3d_kernel" if d else "conv_tma_kernel",
              "histogram": "histogram_kernel"}[op]
    roofline = {"bound": "hbm", "peak": peak_gbs, "unit": "GB/s", "kernel": kernel,
                "bytes_per_unit": bcell, "algorithmic_bytes_per_launch": bcell * slab_cells, "peak_source": peak_src}
    per_kernel_s = None
    if op != "histogram":
        # CUDA events around every bulk launch on the launching stream
        # (direct launches, same kernels and configuration) for one step
        grid.set_option(M.OPT_TIMING, 1)
        grid.iterate(n)
        bulk_ms, bulk_n, bnd_ms, bnd_n = M.mapsm_get_timing(grid.handle)
        grid.set_option(M.OPT_TIMING, 0)
        bulk_rows = rows if bnd_n == 0 else rows - 2 * wl["r"]
        per_kernel_s = (bulk_ms / 1e3) / max(1, bulk_n)
        achieved_kernel = bcell * bulk_rows * cpu_ / per_kernel_s / 1e9
        roofline["achieved_events_per_launch_GBps"] = achieved_kernel
        roofline["kernel_ms_per_launch"] = per_kernel_s * 1e3
        achieved = achieved_region if world == 1 else achieved_kernel
    else:
        achieved = achieved_region
        roofline["note"] = ("whole step timed (memset + kernel + aggregation + bins copy); the 64 MiB image "
                            "is re-read from HBM after each L2 flush")
    roofline["achieved"] = achieved
    roofline["frac"] = achieved / peak_gbs
    roofline["frac_vs_8TBps_spec"] = achieved / 8000.0
    roofline["traffic"] = None
    tfile = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tfile):
        try:
            roofline["traffic"] = json.load(open(tfile)).get(args.workload)
        except Exception:
            pass
    if op == "conv":
        fma_per_cell = (2 * wl["r"] + 1) ** (3 if d else 2)
        sm_mhz = clocks.get("sm_mhz") or 1965.0
        fma_peak = 148 * 128 * sm_mhz * 1e6
        roofline["fma_frac_at_sampled_clock"] = (bulk_rows * cpu_ * fma_per_cell / per_kernel_s) / fma_peak
        if fma_per_cell / 8.0 > 5.7:   # above the FMA/HBM balance (37.2 TFMA/s / 6.5 TB/s)
            # FMA-bound: the binding roofline is the FP32 FMA pipe,
            # 148 SMs x 128 FMA/clk x 2 flop x the SM clock sampled during the run
            # (guide unit counts; nominal, not measured). The HBM figures stay as
            # secondary keys.
            flops_per_cell = 2.0 * fma_per_cell
            t_launch = per_launch_s if world == 1 else per_kernel_s
            rows_launch = slab_cells if world == 1 else bulk_rows * cpu_
            alu_ach = flops_per_cell * rows_launch / t_launch / 1e12
            alu_peak = 2.0 * fma_peak / 1e12
            roofline = {"bound": "alu", "kernel": kernel, "achieved": alu_ach, "peak": alu_peak,
                        "unit": "TFLOP/s", "frac": alu_ach / alu_peak,
                        "flops_per_unit": flops_per_cell,
                        "algorithmic_flops_per_launch": flops_per_cell * rows_launch,
                        "peak_source": (f"derived: 148 SM x 128 FP32 FMA/clk x 2 flop x {sm_mhz:.0f} MHz "
                                        "(sampled SM clock; B200_PROFILING.md unit counts)"),
                        "traffic": roofline["traffic"],
                        "hbm": {"achieved": achieved, "peak": peak_gbs, "unit": "GB/s",
                                "frac": achieved / peak_gbs, "bytes_per_unit": bcell,
                                "peak_source": peak_src},
                        "kernel_ms_per_launch": per_kernel_s * 1e3,
                        "note": f"FP32-FMA bound ({fma_per_cell / 8.0:.2f} FMA/B > 5.7 balance)"}

    # halo-exchange exposure (N > 1): same steps without the exchange
    exposure = None
    if world > 1 and op != "histogram":
        grid.set_option(M.OPT_NO_EXCHANGE, 1)
        grid.iterate(n)
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        grid.iterate(n)
        e1.record(stream)
        barrier()
        tt = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        grid.set_option(M.OPT_NO_EXCHANGE, 0)
        exposure = {"ms_per_step_no_exchange": float(tt.item()),
                    "exposed_pct": 100.0 * (ms_per_step - float(tt.item())) / ms_per_step}

    # e2e: host buffers through the public API, copies inside the timed region
    e2e_ms = 0.0
    barrier()
    for _ in range(args.e2e_steps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        barrier()
        e0.record(stream)
        grid.bind(h_in)
        if op == "histogram":
            M.mapsm_histogram(grid.handle, h_bins)
        else:
            grid.iterate(n)
            M.mapsm_read(grid.handle, h_out, grid._rp(h_out))
        e1.record(stream)
        e1.synchronize()
        e2e_ms += e0.elapsed_time(e1)
    te = torch.tensor([e2e_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_value = units_per_step * args.e2e_steps / (float(te.item()) / 1e3)
    elem = 4 if op == "conv" else 1
    h2d = cells_total * elem
    d2h = 256 * 8 * world if op == "histogram" else cells_total * elem

    # Chained task: a Reductive-Static histogram task over
    # the current generation, its data movement inferred by the Segment Location
    # Monitor (Alg 2) — 0 bytes on the grid's own partition.  Timed per call
    # (memset + kernel + aggregation + bins copy), after an L2 flush.
    chained = None
    if op != "histogram":
        d_b = torch.zeros(256, dtype=torch.int64, device=dev)
        _, moved = M.mapsm_task_histogram(grid.handle, 0, d_b)
        c_ms = 0.0
        for _ in range(args.steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            M.mapsm_task_histogram(grid.handle, 0, d_b, sync=False)
            e1.record(stream)
            e1.synchronize()
            c_ms += e0.elapsed_time(e1)
        tc = torch.tensor([c_ms], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tc, op=dist.ReduceOp.MAX)
        c_s = float(tc.item()) / 1e3 / args.steps
        tb = 0.125 if op == "life" else 4.0   # bytes read per cell (1 bit / one fp32)
        ach = tb * rows * cpu_ / c_s / 1e9
        chained = {"task": "histogram of the current generation (mapsm_task_histogram, grid's own partition)",
                   "moved_bytes": int(moved), "ms_per_call": c_s * 1e3, "cells_per_s": cells_total / c_s,
                   "roofline": {"bound": "hbm", "kernel": "histogram_life_kernel" if op == "life"
                                else "histogram_f32_kernel", "bytes_per_unit": tb, "achieved": ach,
                                "peak": peak_gbs, "unit": "GB/s", "frac": ach / peak_gbs,
                                "note": "whole call timed (memset + kernel + bins copy + sync)"}}

    grid.close()

    # Deep halos    grid.close()

    # Deep halos (MAPSM_OPT_DEEP_HALO): the same workload
    # with K generations per pass and K-row halos exchanged once per pass —
    # reported separately because it is not the per-iteration exchange of the
    # north_star design and is bound by the ALU pipe, not HBM.
    deep = None
    if op == "life" and args.deep_halo > 1:
        K = args.deep_halo
        dg = M.Grid(ctx, w, h, op, wl["r"], wl["b"], None, deep_halo=K)
        dg.bind(h_in)
        for _ in range(args.warmup):
            dg.iterate(n)
        barrier()
        d_ms = 0.0
        for _ in range(args.steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            dg.iterate(n)
            e1.record(stream)
            e1.synchronize()
            d_ms += e0.elapsed_time(e1)
        dinfo = dg.info()
        # per-launch kernel time of the temporally blocked kernel (direct launches)
        dg.set_option(M.OPT_TIMING, 1)
        dg.iterate(n - n % K)
        b_ms, b_n, bb_ms, bb_n = M.mapsm_get_timing(dg.handle)
        dg.set_option(M.OPT_TIMING, 0)
        dg.close()
        td = torch.tensor([d_ms], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(td, op=dist.ReduceOp.MAX)
        d_ms = float(td.item())
        d_value = units_per_step * args.steps / (d_ms / 1e3)
        # ALU roofline: 12 ALU-pipe ops (2 funnel shifts + 2 LOP3 for the
        # 3-cell row sum, 8 LOP3 for the rule) per 32-cell word per generation;
        # the ALU pipe retires 64 lanes/clk/SM (tools/pipebench.cu: LOP3 and
        # SHF ~1.9 warp-instructions/clk/SM).
        sm_mhz = clocks.get("sm_mhz") or 1965.0
        alu_peak = 148 * 64 * sm_mhz * 1e6 / 1e12  # T lane-ops/s
        kern_s = (b_ms / 1e3) / max(1, b_n)
        bulk_rows = rows if bb_n == 0 else rows - 2 * K
        cells_per_launch = bulk_rows * w * K
        alu_achieved = cells_per_launch * 12 / 32 / kern_s / 1e12
        deep = {"generations_per_pass": int(dinfo.gens_per_pass), "halo_rows": int(dinfo.halo_rows),
                "value": d_value, "unit": metric_of(wl)[1], "ms_per_step": d_ms / args.steps,
                "vs_per_generation_path": d_value / value,
                "roofline": {"bound": "alu", "kernel": "life_tb_kernel", "achieved": alu_achieved,
                             "peak": alu_peak, "unit": "T ALU lane-ops/s", "frac": alu_achieved / alu_peak,
                             "ops_per_cell_update": 12 / 32, "kernel_ms_per_launch": kern_s * 1e3,
                             "peak_source": "148 SMs x 64 ALU lanes/clk x sampled SM clock (B300_MICROARCH.md "
                                            "alu rt=2/SMSP; tools/pipebench.cu)",
                             "hbm_bytes_per_cell_update": 0.25 / K,
                             "hbm_achieved_GBps": cells_per_launch * 0.25 / K / kern_s / 1e9}}
    M.mapsm_ctx_destroy(ctx)

    if rank == 0:
        cb = None if args.no_cpu_baseline else cpu_baseline(wl)
        nbuf = 1 if op == "histogram" else 2
        ws_mib = nbuf * (rows + 2 * wl["r"]) * info0.pitch_bytes / 2**20
        metric, unit = metric_of(wl)
        dtype = {"life": "u32 bit-sliced (1 bit/cell)", "conv": "f32", "histogram": "u8 in, u32/u64 counts"}[op]
        para = f"row-slab x{world}"
        if world > 1:
            para += " + NCCL allreduce of bins" if op == "histogram" else " + NCCL halo exchange"
        line = {
            "metric": metric, "value": value, "unit": unit, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": wl["scaling"], "vs_baseline": None, "dtype": dtype, "data": "synthetic",
            "config": {"workload": wl["label"], "w": w, "h": h, **({"d": d} if d else {}),
                       "iterations_per_step": n, "radius": wl["r"],
                       "boundary": wl["b"], "parallelism": para,
                       "l2": f"L2 flushed between steps (256 MiB write, outside the events); per-GPU working set "
                             f"{ws_mib:.0f} MiB vs 126 MB L2",
                       "cuda_graphs": used_graphs},
            "e2e": {"value": e2e_value, "unit": unit, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                    "how": ("mapsm_bind(pinned host) + mapsm_histogram(-> host bins) per step" if op == "histogram"
                            else "mapsm_bind(pinned host) + mapsm_iterate(n) + mapsm_read(pinned host) per step")},
            "gpu_launches": total_launches,
            "roofline": roofline,
            "clocks": clocks,
            "cpu_baseline": cb,
        }
        if exposure is not None:
            line["halo_exposure"] = exposure
        if deep is not None:
            line["deep_halo"] = deep
        if chained is not None:
            line["chained_task"] = chained
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier(device_ids=[local_rank])
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
