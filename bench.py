"""bench.py — Game of Life cell-updates/s and % of roofline on 1..8 B200.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` (torchrun
for N > 1) prints ONE JSON line on rank 0.  Default workload = BASELINE.json
configs[2] at N=1 (``life64k``, the metric's configuration).  The same line
carries, under ``configs``, every other BASELINE configuration measured under
the same clock (``life8k`` = configs[1], ``conv5`` = configs[3], ``conv9`` =
configs[4]), each with its own value, ms_per_step, clocks, roofline (its own
dominant kernel and bound) and cpu_baseline.  ``--workload`` runs one
workload alone (also the §8(f) NEXT items: ``hist8k``, ``conv3d``, ``sgemm8k``).

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
* roofline  = the dominant kernel of the step (named from the library's launch
              record, mapsm_launch_query) against its bound: HBM (measured copy
              bandwidth, MEASURED_PEAKS.json hbm_gbs) for Life 65536^2 and the
              5x5 conv; the ALU pipe for the L2/SMEM-resident 8192^2 Life; the
              FP32 FMA pipe for the 9x9 conv.  achieved = algorithmic bytes (or
              ops) per launch / the average launch duration over the timed
              region (step time / launches per step, launch gaps included).
* cpu_baseline = the CPU oracle (oracle/, OpenMP) timed on a bounded sample of
              the same workload on rank 0 at N = 1.
* deep_halo = (Life 65536^2) the deep-halo path (MAPSM_OPT_DEEP_HALO = K: K
              generations per pass, K-row halos exchanged once per pass),
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
                   scaling="strong", bcell=0.25, single_gpu=True,
                   label="Game of Life 8192x8192 WRAP, random p=0.5 (seed 0x5EED0002), 1000 generations per step "
                         "(BASELINE configs[1], 1 B200; SMEM-resident)"),
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
    """nvidia-smi SM clocks / throttle reasons, sampled every 50 ms for the
    whole run (started before any warm-up) with the host time of every
    sample; ``region(t0, t1)`` summarises the samples taken inside one timed
    region.  A region without a sample (shorter than the period) reports
    sm_mhz = None (no off-region clock is substituted)."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.samples = []  # (host time, sm, smax, reasons)

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-lms", "50", "-i", str(self.dev)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            now = time.time()
            parts = [p.strip() for p in line.strip().split(",")]
            if len(parts) < 6:
                continue
            try:
                sm, smax = float(parts[0]), float(parts[1])
            except ValueError:
                continue
            reasons = {nm for nm, v in zip(self.NAMES, parts[2:6]) if v.lower().startswith("active")}
            self.samples.append((now, sm, smax, reasons))

    def region(self, t0, t1):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.06)  # let the sample that closes the region arrive
        inside = [s for s in list(self.samples) if t0 <= s[0] <= t1 + 0.055]
        if not inside:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0,
                    "note": f"no nvidia-smi sample inside the {1e3 * (t1 - t0):.0f} ms region (50 ms period)"}
        reasons = set()
        for s in inside:
            reasons |= s[3]
        return {"sm_mhz": statistics.median(s[1] for s in inside), "sm_max_mhz": max(s[2] for s in inside),
                "reasons": sorted(reasons), "samples": len(inside)}

    def stop(self):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()


def sm_clock_for_peak(clocks):
    """SM clock for a derived (ALU / FP32) peak: the region's median sample,
    else MEASURED_PEAKS.json sm_max_mhz (stated in peak_source)."""
    if clocks.get("sm_mhz"):
        return float(clocks["sm_mhz"]), "the SM clock sampled during the timed region"
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    mhz = float(json.load(open(p)).get("sm_max_mhz", 1965.0)) if os.path.exists(p) else 1965.0
    return mhz, "MEASURED_PEAKS.json sm_max_mhz (no clock sample inside the region)"


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


def cpu_baseline(wl, budget_s=8.0):
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
    sampler = ClockSampler(local_rank).start()
    time.sleep(0.3)
    total_ms, moved = 0.0, 0
    barrier()
    t_region = time.time()
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
    clocks = sampler.region(t_region, time.time())
    sampler.stop()
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
        sm_mhz, clk_src = sm_clock_for_peak(clocks)
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
                             "peak_source": f"148 SMs x 128 FP32 lanes x 2 flop x {sm_mhz:.0f} MHz ({clk_src})"},
                "clocks": clocks, "cpu_baseline": cb,
                "paper_context": "Table 4 P:L503-508: single-GPU 8K multiplication 245-366 ms on GTX 780/Titan "
                                 "Black/GTX 980 (CUBLAS over MAPS-Multi 248.62 ms on GTX 980)"}
        emit(line)
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
    emit(line)


# ------------------------------------------------------------------ GPU leg

SUB_CONFIGS = ["life8k", "conv5", "conv9"]  # BASELINE configs[1], [3], [4] beside the headline configs[2]
ALU_OPS_PER_WORD = 12  # Life: 2 funnel shifts + 2 LOP3 (3-cell row sum) + 8 LOP3 (rule) per 32-cell word


class Env:
    """Per-process GPU state shared by every measured workload."""

    def __init__(self, args, rank, world, local_rank):
        import torch
        import torch.distributed as dist

        from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

        self.torch, self.dist, self.M = torch, dist, M
        self.args, self.rank, self.world, self.local_rank = args, rank, world, local_rank
        torch.cuda.set_device(local_rank)
        self.dev = torch.device("cuda", local_rank)
        if world > 1:
            dist.init_process_group("nccl", device_id=self.dev)
        # A dedicated (non-default) stream: libmapsm launches on it, and the CUDA
        # events of the timed regions are recorded on it.
        self.stream = torch.cuda.Stream(device=self.dev)
        torch.cuda.set_stream(self.stream)
        uid = None
        if world > 1:
            obj = [M.mapsm_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            uid = obj[0]
        self.ctx = M.mapsm_ctx_create(rank, world, local_rank, uid, self.stream.cuda_stream)
        self.flush = torch.empty(256 << 20, dtype=torch.uint8, device=self.dev)  # > 126 MB L2
        self.sampler = ClockSampler(local_rank).start()

    def barrier(self):
        if self.world > 1:
            self.dist.barrier(device_ids=[self.local_rank])
        self.torch.cuda.synchronize()

    def max_over_ranks(self, x, dtype=None):
        t = self.torch.tensor([x], dtype=dtype or self.torch.float64, device=self.dev)
        if self.world > 1:
            self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX)
        return t.item()

    def sum_over_ranks(self, x):
        t = self.torch.tensor([x], dtype=self.torch.int64, device=self.dev)
        if self.world > 1:
            self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM)
        return int(t.item())

    def timed(self, fn, steps, flush=True):
        """K steps, each bracketed by CUDA events on the library's stream, L2
        flushed before each step outside the events; returns (sum ms, t0, t1)."""
        torch = self.torch
        total = 0.0
        self.barrier()
        t0 = time.time()
        for _ in range(steps):
            if flush:
                self.flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(self.stream)
            fn()
            e1.record(self.stream)
            e1.synchronize()
            total += e0.elapsed_time(e1)
        self.barrier()
        return total, t0, time.time()

    def close(self):
        self.M.mapsm_ctx_destroy(self.ctx)
        self.sampler.stop()
        if self.world > 1:
            self.dist.barrier(device_ids=[self.local_rank])
            self.dist.destroy_process_group()


def host_input(env, wl, rows, y0):
    """Pinned host rows [y0, y0+rows) of the workload's synthetic input."""
    import mapsm_inputs as mi

    torch = env.torch
    d = wl.get("d", 0)
    w, h = wl["w"], wl["h"]
    dt = torch.float32 if wl["op"] == "conv" else torch.uint8
    t = torch.empty((rows, h, w) if d else (rows, w), dtype=dt, pin_memory=True)
    if d:
        t.numpy()[:] = mi.volume_f32(wl["seed"], w, h, rows, z0=y0)
    elif wl["op"] == "life":
        mi.life_u8(wl["seed"], w, rows, y0=y0, out=t.numpy())
    elif wl["op"] == "conv":
        mi.field_f32(wl["seed"], w, rows, y0=y0, out=t.numpy())
    else:
        mi.image_u8(wl["seed"], w, rows, y0=y0, out=t.numpy())
    return t


def roofline_of(env, name, wl, kernel, cells_launch, t_launch_s, clocks, launch_unit, gens=1):
    """The dominant kernel's roofline: algorithmic work of one launch over the
    average launch duration in the timed region.  `gens`:
    generations one launch computes with one HBM read and one write of the
    field (conv_tb2_kernel: 2), which multiplies the arithmetic, not the bytes."""
    peak_gbs, peak_src = load_peaks()
    bcell = wl["bcell"]
    hbm_ach = bcell * cells_launch / t_launch_s / 1e9
    hbm = {"achieved": hbm_ach, "peak": peak_gbs, "unit": "GB/s", "frac": hbm_ach / peak_gbs,
           "bytes_per_unit": bcell, "peak_source": peak_src}
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tfile):
        try:
            traffic = json.load(open(tfile)).get(name)
        except Exception:
            traffic = None
    base = {"kernel": kernel, "launch_unit": launch_unit, "ms_per_launch": t_launch_s * 1e3, "traffic": traffic}
    mhz, clk_src = sm_clock_for_peak(clocks)
    if wl["op"] == "life" and kernel in ("life_tb_persist_kernel", "life_persist_kernel", "life_tb_kernel"):
        # L2 / SMEM resident (or temporally blocked): bound by the ALU pipe
        ach = cells_launch * ALU_OPS_PER_WORD / 32 / t_launch_s / 1e12
        peak = 148 * 64 * mhz * 1e6 / 1e12
        return {"bound": "alu", **base, "achieved": ach, "peak": peak, "unit": "T ALU lane-ops/s", "frac": ach / peak,
                "ops_per_unit": ALU_OPS_PER_WORD / 32,
                "algorithmic_ops_per_launch": cells_launch * ALU_OPS_PER_WORD / 32,
                "peak_source": f"148 SMs x 64 ALU lanes/clk x {mhz:.0f} MHz ({clk_src}; B200_PROFILING.md unit "
                               "counts, LOP3/SHF issue measured with tools/pipebench.cu)",
                "hbm_equivalent": {**hbm, "note": "working set resident in L2 / shared memory: the HBM "
                                                  "fraction is not a bound (it can exceed 1)"}}
    if wl["op"] == "conv":
        fma_cell = (2 * wl["r"] + 1) ** (3 if wl.get("d") else 2)
        if fma_cell * gens / bcell > 5.7:  # above the FMA/HBM balance (37.2 TFMA/s / 6.5 TB/s): FP32-FMA bound
            fma_cell *= gens
            ach = 2.0 * fma_cell * cells_launch / t_launch_s / 1e12
            peak = 148 * 128 * 2 * mhz * 1e6 / 1e12
            return {"bound": "alu", **base, "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak,
                    "flops_per_unit": 2.0 * fma_cell, "algorithmic_flops_per_launch": 2.0 * fma_cell * cells_launch,
                    "peak_source": f"derived: 148 SM x 128 FP32 FMA/clk x 2 flop x {mhz:.0f} MHz ({clk_src}; "
                                   "B200_PROFILING.md unit counts; FFMA2 issue measured with tools/pipebench3.cu)",
                    "hbm": hbm, "note": f"FP32-FMA bound ({fma_cell / bcell:.2f} FMA/B > 5.7 balance)"}
    return {"bound": "hbm", **base, "achieved": hbm_ach, "peak": peak_gbs, "unit": "GB/s",
            "frac": hbm_ach / peak_gbs, "frac_vs_8TBps_spec": hbm_ach / 8000.0, "bytes_per_unit": bcell,
            "algorithmic_bytes_per_launch": bcell * cells_launch, "peak_source": peak_src}


def measure(env, name, wl, steps, warmup, e2e_steps, min_region_s=0.0, extras=False, deep_k=0):
    """One workload: K timed steps + e2e (+ the headline's extras)."""
    M, torch, args = env.M, env.torch, env.args
    world, rank = env.world, env.rank
    op = wl["op"]
    w = wl["w"]
    h = wl["h"] * (world if wl["scaling"] == "weak" else 1)
    n = wl["n"]
    d = wl.get("d", 0)
    if op == "conv":
        import mapsm_inputs as mi
        W = mi.weights3d_f32(wl["wseed"], wl["r"]) if d else mi.weights_f32(wl["wseed"], wl["r"])
    else:
        W = None
    # Halo exchange of the multi-process run (at N = 1 nothing is exchanged;
    # the nccl_ring sub-line covers the modes on one GPU): "auto" = the fused
    # peer-store kernel (MAPSM_EXCHANGE_P2P, CUDA IPC over NVLink; the fastest
    # exchange on the ring at the N = 8 slab sizes) where the
    # grid allows it, else — or if the collective IPC linking fails on any
    # rank — NCCL send/recv with the concurrent-boundary schedule.
    xmode = args.exchange
    if xmode == "auto":
        xmode = "p2p" if (world > 1 and op in ("life", "conv") and not d and wl["r"] <= 4) else "nccl"
    if world == 1 or op == "histogram":
        xmode = "nccl"

    def make_grid(mode):
        gr = M.Grid(env.ctx, w, h, op, wl["r"], wl["b"], W, d=d)
        if mode != "nccl":
            gr.set_option(M.OPT_EXCHANGE, {"p2p": M.EXCHANGE_P2P, "ce": M.EXCHANGE_CE}[mode])
        if args.graph_iters:
            gr.set_option(M.OPT_GRAPH_ITERS, args.graph_iters)
        return gr

    grid = make_grid(xmode)
    cpu_ = w * (h if d else 1)             # cells per partition unit (row or plane)
    cells_total = w * h * (d if d else 1)
    y0, rows = grid.local_rows()
    h_in = host_input(env, {**wl, "h": h}, rows, y0)
    h_out = torch.empty_like(h_in, pin_memory=True) if op != "histogram" else None
    d_bins = torch.zeros(256, dtype=torch.int64, device=env.dev)
    h_bins = torch.zeros(256, dtype=torch.int64, pin_memory=True)
    x_fallback = None
    try:
        grid.bind(h_in)
    except M.MapsmError as e:  # (the same error on every rank: the linking agrees collectively)
        if xmode == "nccl" or args.exchange != "auto":
            raise
        x_fallback = str(e)[:200]
        grid.close()
        xmode = "nccl"
        grid = make_grid(xmode)
        grid.bind(h_in)
    info0 = grid.info()

    def step():
        if op == "histogram":
            M.mapsm_histogram(grid.handle, d_bins, sync=False)
        else:
            grid.iterate(n)

    for _ in range(warmup):
        step()
    env.barrier()
    if min_region_s > 0:  # sub-configurations: at least min_region_s of timed steps (clock samples)
        one, _, _ = env.timed(step, 1)
        one = env.max_over_ranks(one)
        steps = max(steps, min(400, int(min_region_s * 1e3 / max(one, 1e-3)) + 1))
    launches0 = grid.info().launches
    total_ms, t0, t1 = env.timed(step, steps)
    clocks = env.sampler.region(t0, t1)
    launches = grid.info().launches - launches0
    used_graphs = bool(grid.info().used_graphs)
    total_ms = env.max_over_ranks(total_ms)
    total_launches = env.sum_over_ranks(launches)
    units_per_step = cells_total * n
    value = units_per_step * steps / (total_ms / 1e3)
    ms_per_step = total_ms / steps
    li = grid.launch(0)
    kernel = M.KERNEL_NAMES.get(li.kernel, "?") if op != "histogram" else "histogram_kernel"
    slab_cells = rows * cpu_
    # the unit of the roofline: one launch of the dominant kernel.  At N = 1
    # every generation is one launch (or a whole persistent step is one);
    # with exchanged halos a generation is boundary + interior launches + the
    # exchange, and the generation is the unit.
    per_process_launches = max(1, launches // steps)
    if op == "histogram":
        gens_per_launch, unit = 1, "one histogram call (one launch)"
    elif li.gens_per_launch > 1 and per_process_launches == 1:
        gens_per_launch, unit = n, f"one launch = {n} generations (SMEM-resident persistent kernel)"
    elif per_process_launches == n:
        gens_per_launch, unit = 1, "one launch = one generation"
    else:
        gens_per_launch, unit = 1, "one generation (boundary + interior launches + halo exchange)"
    t_launch = (ms_per_step / 1e3) / (n / gens_per_launch)
    roofline = roofline_of(env, name, wl, kernel, slab_cells * gens_per_launch, t_launch, clocks, unit)

    exposure = None
    if world > 1 and op != "histogram":  # halo-exchange exposure: the same steps without the exchange
        grid.set_option(M.OPT_NO_EXCHANGE, 1)
        grid.iterate(n)
        ne_ms, _, _ = env.timed(step, 2, flush=False)
        ne = env.max_over_ranks(ne_ms) / 2
        grid.set_option(M.OPT_NO_EXCHANGE, 0)
        exposure = {"ms_per_step_no_exchange": ne, "exposed_pct": 100.0 * (ms_per_step - ne) / ms_per_step}

    chained = deep = None
    if extras and op != "histogram":
        # Chained task: a Reductive-Static histogram of the
        # current generation, data movement inferred by Alg 2 (0 bytes on the
        # grid's own partition); whole call timed after an L2 flush.
        d_b = torch.zeros(256, dtype=torch.int64, device=env.dev)
        _, moved = M.mapsm_task_histogram(grid.handle, 0, d_b)
        c_ms, _, _ = env.timed(lambda: M.mapsm_task_histogram(grid.handle, 0, d_b, sync=False), steps)
        c_s = env.max_over_ranks(c_ms) / 1e3 / steps
        peak_gbs, _ = load_peaks()
        tb = 0.125 if op == "life" else 4.0
        ach = tb * rows * cpu_ / c_s / 1e9
        chained = {"task": "histogram of the current generation (mapsm_task_histogram, grid's own partition)",
                   "moved_bytes": int(moved), "ms_per_call": c_s * 1e3, "cells_per_s": cells_total / c_s,
                   "roofline": {"bound": "hbm", "kernel": "histogram_life_kernel" if op == "life"
                                else "histogram_f32_kernel", "bytes_per_unit": tb, "achieved": ach,
                                "peak": peak_gbs, "unit": "GB/s", "frac": ach / peak_gbs,
                                "note": "whole call timed (kernel + bins, one launch)"}}
    # e2e: host buffers through the public API, copies inside the timed region.
    # Sequential: bind -> iterate -> read, one step at a time (host waits).
    def e2e_step():
        grid.bind(h_in)
        if op == "histogram":
            M.mapsm_histogram(grid.handle, h_bins)
        else:
            grid.iterate(n)
            M.mapsm_read(grid.handle, h_out, grid._rp(h_out))

    seq_ms, _, _ = env.timed(e2e_step, 1, flush=False)
    seq_value = units_per_step / (env.max_over_ranks(seq_ms) / 1e3)
    e2e_value, e2e_how = seq_value, ("mapsm_bind(pinned host) + mapsm_histogram(-> host bins) per step"
                                     if op == "histogram" else
                                     "mapsm_bind(pinned host) + mapsm_iterate(n) + mapsm_read(pinned host) per step")
    pipe = packed_e2e = None
    if op != "histogram" and args.e2e_pipeline > 1 and world == 1:
        # (N = 1 only: with N > 1 every Bind is a collective; several grids'
        # NCCL exchanges on different streams of one communicator are not
        # pipelined here — the multi-GPU e2e stays sequential)
        # Pipelined: P grids of the same workload on their own streams
        # (MAPSM_OPT_OWN_STREAM), each step = mapsm_bind_async(pinned host
        # input) + mapsm_iterate(n) + mapsm_read_async(pinned host output) on
        # the next grid: one step's upload, another's generations and a third's
        # download run together (PCIe is full duplex).  Every step still moves
        # its whole input in and its whole result out inside the timed region
        # (events: start on the bench stream, every grid stream waits on it;
        # end after every grid stream's last read).  The library orders the
        # own-stream grids' host transfers FIFO per direction (xfer_begin).
        P = args.e2e_pipeline
        k_steps = max(e2e_steps, 8 * P)
        pgrids = [grid]
        grid.set_option(M.OPT_OWN_STREAM, 1)
        for _ in range(P - 1):
            pg = M.Grid(env.ctx, w, h, op, wl["r"], wl["b"], W, d=d)
            pg.set_option(M.OPT_OWN_STREAM, 1)
            pg.bind(h_in)
            pgrids.append(pg)
        pouts = [h_out] + [torch.empty_like(h_in, pin_memory=True) for _ in range(P - 1)]
        gstreams = [torch.cuda.ExternalStream(M.mapsm_grid_stream(pg.handle)) for pg in pgrids]
        for pg in pgrids:  # warm the graphs / streams
            pg.iterate(n)
            pg.sync()
        env.barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(env.stream)
        for gs in gstreams:
            gs.wait_event(e0)
        for k in range(k_steps):
            pg = pgrids[k % P]
            M.mapsm_bind_async(pg.handle, h_in)
            pg.iterate(n)
            M.mapsm_read_async(pg.handle, pouts[k % P], pg._rp(pouts[k % P]))
        for gs in gstreams:
            ev = torch.cuda.Event()
            ev.record(gs)
            env.stream.wait_event(ev)
        e1.record(env.stream)
        e1.synchronize()
        for pg in pgrids:
            pg.sync()
        pipe_ms = env.max_over_ranks(e0.elapsed_time(e1))
        pipe = {"value": units_per_step * k_steps / (pipe_ms / 1e3), "steps": k_steps, "grids": P,
                "ms_per_step": pipe_ms / k_steps}
        e2e_value = pipe["value"]
        e2e_how = (f"{P} grids on their own streams, each step mapsm_bind_async(pinned host input) + "
                   f"mapsm_iterate(n) + mapsm_read_async(pinned host output) on the next grid; {k_steps} steps "
                   "timed end to end (device events, all grid streams joined)")
        if op == "life" and w % 32 == 0:
            # The same pipeline with bit-packed host rows (MAPSM_OPT_HOST_PACKED:
            # the device row format, 1/8 of the u8 bytes over PCIe).
            import numpy as np

            hp_in = torch.from_numpy(np.packbits(h_in.numpy() != 0, axis=1, bitorder="little")).pin_memory()
            hp_outs = [torch.empty_like(hp_in, pin_memory=True) for _ in range(P)]
            for pg in pgrids:
                pg.set_option(M.OPT_HOST_PACKED, 1)
                M.mapsm_bind(pg.handle, hp_in)
                pg.iterate(n)
                pg.sync()
            env.barrier()
            e0.record(env.stream)
            for gs in gstreams:
                gs.wait_event(e0)
            for k in range(k_steps):
                pg = pgrids[k % P]
                M.mapsm_bind_async(pg.handle, hp_in)
                pg.iterate(n)
                M.mapsm_read_async(pg.handle, hp_outs[k % P])
            for gs in gstreams:
                ev = torch.cuda.Event()
                ev.record(gs)
                env.stream.wait_event(ev)
            e1.record(env.stream)
            e1.synchronize()
            for pg in pgrids:
                pg.sync()
            pk_ms = env.max_over_ranks(e0.elapsed_time(e1))
            packed_e2e = {"value": units_per_step * k_steps / (pk_ms / 1e3), "ms_per_step": pk_ms / k_steps,
                          "h2d_bytes_per_step": int(hp_in.numel()), "d2h_bytes_per_step": int(hp_in.numel()),
                          "how": "as `how`, with MAPSM_OPT_HOST_PACKED: host rows bit-packed (w/32 uint32 "
                                 "words, bit j of word k = column 32k+j), the device row format"}
            for pg in pgrids:
                pg.set_option(M.OPT_HOST_PACKED, 0)
        for pg in pgrids[1:]:
            pg.close()
    elem = 4 if op == "conv" else 1
    h2d = cells_total * elem
    d2h = 256 * 8 * world if op == "histogram" else cells_total * elem

    grid.close()
    if (extras and op == "life" and args.deep_halo > 1) or (op == "conv" and deep_k > 1 and not d):
        # Deep halos: K generations per pass, K*r-row
        # halos exchanged once per pass — reported separately (not the
        # per-iteration exchange of the north_star design).  Life: ONE
        # temporally blocked kernel per pass (ALU-bound); conv r <= 2 with
        # K = 2: the fused two-generation kernel (one HBM pass per two
        # generations); other conv: K launches per pass over a trapezoid.
        K = args.deep_halo if op == "life" else deep_k
        dg = M.Grid(env.ctx, w, h, op, wl["r"], wl["b"], W, deep_halo=K)
        dg.bind(h_in)
        for _ in range(warmup):
            dg.iterate(n)
        dl0 = dg.info().launches
        d_ms, dt0, dt1 = env.timed(lambda: dg.iterate(n), steps)
        dclocks = env.sampler.region(dt0, dt1)
        dinfo = dg.info()
        dl = (dinfo.launches - dl0) // steps
        dkernel = M.KERNEL_NAMES.get(dg.launch(0).kernel, "?")
        dg.close()
        d_ms = env.max_over_ranks(d_ms)
        d_value = units_per_step * steps / (d_ms / 1e3)
        passes = n // K
        t_pass = (d_ms / steps / 1e3) / max(1, passes)
        if op == "life":
            droof = roofline_of(env, f"{name}_tb{K}", wl, "life_tb_kernel", slab_cells * K, t_pass, dclocks,
                                f"one pass = {K} generations ({dl} launches per step)")
        elif dkernel == "conv_tb2_kernel":  # one launch = the two generations of a pass
            droof = roofline_of(env, name + "_tb2", wl, dkernel, slab_cells, t_pass, dclocks,
                                f"one pass = {K} generations in one launch ({dl} launches per step)", gens=K)
        else:
            droof = roofline_of(env, name, wl, dkernel, slab_cells, t_pass / K, dclocks,
                                f"one generation (a pass = {K} launches; {dl} launches per step)")
        deep = {"generations_per_pass": int(dinfo.gens_per_pass), "halo_rows": int(dinfo.halo_rows),
                "value": d_value, "unit": metric_of(wl)[1], "ms_per_step": d_ms / steps,
                "vs_per_generation_path": d_value / value, "roofline": droof, "clocks": dclocks,
                "kernel": dkernel,
                "hbm_bytes_per_cell_update": (0.25 / K if op == "life" else
                                              wl["bcell"] / K if dkernel == "conv_tb2_kernel" else wl["bcell"]),
                "exchanged_rows_per_pass": K * wl["r"]}

    ring = None
    if extras and world == 1 and op != "histogram" and wl["b"] == "wrap" and not d:
        try:  # (an NCCL failure here must not cost the bench line)
            # The NCCL data plane on one GPU (include/mapsm.h, one-rank NCCL
            # context): the WRAP row ring closes through ncclSend/ncclRecv to
            # itself every generation — boundary rows first, the exchange group on
            # the side stream, interior overlapped, all inside the CUDA graphs — so
            # the multi-process path runs on hardware; exposure = the same steps
            # with the exchange switched off.
            rctx = M.mapsm_ctx_create(0, 1, env.local_rank, M.mapsm_nccl_unique_id(), env.stream.cuda_stream)
            try:
                rg = M.Grid(rctx, w, h, op, wl["r"], wl["b"], W)
                rg.bind(h_in)
                for _ in range(warmup):
                    rg.iterate(n)
                x0, l0 = rg.info().exchanges, rg.info().launches
                r_ms, rt0, rt1 = env.timed(lambda: rg.iterate(n), steps)
                rclocks = env.sampler.region(rt0, rt1)
                rinfo = rg.info()
                rg.set_option(M.OPT_EXCHANGE_SMS, 0)
                rg.iterate(n)
                ser_ms, _, _ = env.timed(lambda: rg.iterate(n), 2)
                rg.set_option(M.OPT_EXCHANGE_SMS, -1)
                rg.set_option(M.OPT_NO_EXCHANGE, 1)
                rg.iterate(n)
                ne_ms, _, _ = env.timed(lambda: rg.iterate(n), 2)
                rg.close()
                # the fused peer-store kernel over the same ring (MAPSM_EXCHANGE_P2P:
                # boundary CTAs store their rows into the halos and signal the mailbox)
                rg = M.Grid(rctx, w, h, op, wl["r"], wl["b"], W)
                rg.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
                rg.bind(h_in)
                rg.iterate(n)
                fp_ms, _, _ = env.timed(lambda: rg.iterate(n), 2)
                rg.close()
                dring = None
                if op == "life" and args.deep_halo > 1:  # deep halos over the same ring: one exchange per K generations
                    rg = M.Grid(rctx, w, h, op, wl["r"], wl["b"], W, deep_halo=args.deep_halo)
                    rg.bind(h_in)
                    rg.iterate(n)
                    dr_ms, _, _ = env.timed(lambda: rg.iterate(n), 3)
                    dring = {"generations_per_pass": args.deep_halo, "ms_per_step": dr_ms / 3,
                             "value": units_per_step * 3 / (dr_ms / 1e3)}
                    rg.close()
            finally:
                M.mapsm_ctx_destroy(rctx)
            r_step = r_ms / steps
            ring = {"how": "one-rank NCCL communicator (mapsm_ctx_create with world 1 and an id): per generation the "
                           "boundary rows and one NCCL group (send-up, send-down, recv-bottom, recv-top to rank 0) on "
                           "the side stream on a few SMs, the interior on the others (concurrent-boundary schedule, "
                           "MAPSM_OPT_EXCHANGE_SMS default); CUDA graphs",
                    "serial_ms_per_step": ser_ms / 2,
                    "fused_p2p_ms_per_step": fp_ms / 2,
                    "value": units_per_step * steps / (r_ms / 1e3), "unit": metric_of(wl)[1], "ms_per_step": r_step,
                    "vs_plain_path": (units_per_step * steps / (r_ms / 1e3)) / value,
                    "launches_per_step": (rinfo.launches - l0) // steps,
                    "halo_messages_per_step": (rinfo.exchanges - x0) // steps,
                    "halo_bytes_per_message": wl["r"] * int(info0.pitch_bytes),
                    "halo_exposure": {"ms_per_step_no_exchange": ne_ms / 2,
                                      "exposed_pct": 100.0 * (r_step - ne_ms / 2) / r_step},
                    "clocks": rclocks}
            if dring is not None:
                ring["deep_halo"] = dring

        except Exception as e:  # noqa: BLE001
            ring = {"error": f"{type(e).__name__}: {e}"[:300]}

    metric, unit_name = metric_of(wl)
    nbuf = 1 if op == "histogram" else 2
    ws_mib = nbuf * (rows + 2 * wl["r"]) * info0.pitch_bytes / 2**20
    dtype = {"life": "u32 bit-sliced (1 bit/cell)", "conv": "f32", "histogram": "u8 in, u32/u64 counts"}[op]
    para = f"row-slab x{world}"
    if world > 1:
        para += (" + NCCL allreduce of bins" if op == "histogram" else
                 {"nccl": " + NCCL halo exchange (concurrent-boundary schedule)",
                  "p2p": " + fused peer-store halo exchange (CUDA IPC)",
                  "ce": " + copy-engine peer-copy halo exchange"}[xmode])
    line = {
        "metric": metric, "value": value, "unit": unit_name, "n_gpus": world, "steps": steps,
        "warmup": warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": wl["scaling"], "vs_baseline": None, "dtype": dtype, "data": "synthetic",
        "config": {"workload": wl["label"], "w": w, "h": h, **({"d": d} if d else {}),
                   "iterations_per_step": n, "radius": wl["r"], "boundary": wl["b"], "parallelism": para,
                   "l2": f"L2 flushed between steps (256 MiB write, outside the events); per-GPU working set "
                         f"{ws_mib:.0f} MiB vs 126 MB L2", "cuda_graphs": used_graphs,
                   "kernel": kernel, "launch": {"ctas": int(li.ctas), "threads": int(li.threads),
                                                "smem_bytes": int(li.smem_bytes),
                                                "ring_stages": int(li.ring_stages)},
                   **({"exchange": xmode} if world > 1 else {}),
                   **({"exchange_fallback": x_fallback} if x_fallback else {})},
        "e2e": {"value": e2e_value, "unit": unit_name, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "how": e2e_how, "sequential_value": seq_value,
                "sequential_how": "one step: mapsm_bind + mapsm_iterate + mapsm_read, host waits between steps",
                **({"packed_host": packed_e2e} if packed_e2e else {})},
        "gpu_launches": total_launches,
        "roofline": roofline,
        "clocks": clocks,
    }
    if exposure is not None:
        line["halo_exposure"] = exposure
    if deep is not None:
        line["deep_halo"] = deep
    if ring is not None:
        line["nccl_ring"] = ring
    if chained is not None:
        line["chained_task"] = chained
    return line


_JSON_OUT = None


def emit(line):
    """The one JSON line on stdout (everything else the process writes to
    file descriptor 1 — NCCL's version banner, CUDA or library logs — is
    redirected to stderr by main())."""
    out = _JSON_OUT or sys.stdout
    out.write(json.dumps(line) + "\n")
    out.flush()


def main():
    # stdout carries only the JSON line: keep a private handle on the real
    # stdout, then point file descriptor 1 at stderr for everything else
    # (NCCL prints its version banner to stdout under NCCL_DEBUG=VERSION)
    global _JSON_OUT
    sys.stdout.flush()
    _JSON_OUT = os.fdopen(os.dup(1), "w")
    os.dup2(2, 1)
    os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mapsm", choices=["mapsm", "reference"])
    ap.add_argument("--workload", default="life64k", choices=sorted(WORKLOADS))
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--e2e-pipeline", type=int, default=3,
                    help="grids pipelined for the e2e measurement (1 = sequential steps only)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="headline only (no BASELINE sub-configurations)")
    ap.add_argument("--graph-iters", type=int, default=0)
    ap.add_argument("--exchange", default="auto", choices=["auto", "nccl", "p2p", "ce"],
                    help="N > 1: halo exchange of the measured grids (auto = p2p where the grid allows it, "
                         "falling back to nccl if the CUDA-IPC linking fails; nccl = NCCL send/recv with the "
                         "concurrent-boundary schedule; p2p = fused peer stores over CUDA IPC; "
                         "ce = copy-engine peer copies)")
    ap.add_argument("--deep-halo", type=int, default=8,
                    help="Life 65536^2: also measure the deep-halo path with K generations per pass "
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

    env = Env(args, rank, world, local_rank)
    time.sleep(0.2)  # the clock sampler's first samples
    head = measure(env, args.workload, wl, args.steps, args.warmup, args.e2e_steps, extras=True,
                   deep_k=2 if wl["op"] == "conv" and not wl.get("d") else 0)
    subs = {}
    if args.workload == "life64k" and not args.no_configs:
        for name in SUB_CONFIGS:
            swl = dict(WORKLOADS[name])
            if swl.get("single_gpu") and world > 1:
                continue
            subs[name] = measure(env, name, swl, args.steps, args.warmup, 1, min_region_s=0.3,
                                 deep_k=2 if name == "conv5" else 0)
    env.close()
    if rank == 0:
        if not args.no_cpu_baseline and world == 1:
            head["cpu_baseline"] = cpu_baseline(wl)
            for name, sub in subs.items():
                sub["cpu_baseline"] = cpu_baseline(WORKLOADS[name])
        else:
            head["cpu_baseline"] = None
        if subs:
            head["configs"] = {name: {k: v for k, v in sub.items() if k not in ("n_gpus", "higher_is_better",
                                                                                  "vs_baseline", "data")}
                               for name, sub in subs.items()}
        emit(head)


if __name__ == "__main__":
    main()
