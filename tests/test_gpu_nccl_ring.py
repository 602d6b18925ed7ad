"""GPU parity of the NCCL data plane on one B200: a one-rank NCCL communicator
(mapsm_ctx_create(0, 1, dev, id, stream), include/mapsm.h) closes the WRAP row
ring through ncclSend / ncclRecv to itself, so every pass runs exactly what a
rank of the multi-process mode runs (boundary rows
first, the exchange list of mapsm_exchange_plan issued in one NCCL group on
the side stream, interior rows overlapped, CUDA graphs capturing the NCCL
group) — the two-line boundary exchange of P:L461 §5.1 — with the peer being
the rank itself.  Results are compared bit for bit with the CPU oracle
(oracle/oracle.c) and with the same grid on the plain one-GPU context (which
maps the halo rows on the read side and exchanges nothing).  Every case
asserts that halo messages were actually exchanged."""
import numpy as np
import pytest

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ring_ctx():
    import torch

    torch.cuda.set_device(0)
    c = M.mapsm_ctx_create(0, 1, 0, M.mapsm_nccl_unique_id(), None)
    yield c
    M.mapsm_ctx_destroy(c)


def run(c, op, w, h, r, b, x0, steps, W=None, K=1, graphs=True, p2p=False):
    with M.Grid(c, w, h, op, r, b, W, deep_halo=K) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        if p2p:
            g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        g.bind(x0)
        for n in steps:
            g.iterate(n)
        out = g.gather()
        info = g.info()
    return out, info


@pytest.mark.parametrize("graphs", [True, False])
@pytest.mark.parametrize("w,h,n", [(256, 64, 9), (4096, 2048, 20), (1024 + 64, 333, 7)])
def test_life_ring_vs_oracle(ring_ctx, graphs, w, h, n):
    x0 = mi.life_u8(7100 + w + h, w, h)
    out, info = run(ring_ctx, "life", w, h, 1, "wrap", x0, [n], graphs=graphs)
    assert info.exchanges >= 2 * n, info.exchanges  # two halo receives per generation
    assert np.array_equal(out, oracle.life(x0, n, "wrap"))


@pytest.mark.parametrize("b", ["clamp", "zero"])
def test_life_ring_non_wrap_unchanged(ring_ctx, b):
    """No exchanged edge at world == 1 under CLAMP / ZERO: same result, no messages."""
    x0 = mi.life_u8(7200, 512, 96)
    out, info = run(ring_ctx, "life", 512, 96, 1, b, x0, [6])
    assert info.exchanges == 0
    assert np.array_equal(out, oracle.life(x0, 6, b))


@pytest.mark.parametrize("r", [1, 2, 4, 6])
def test_conv_ring_vs_oracle(ring_ctx, r):
    w, h, n = 512 + 4, 8 * r + 37, 5
    f0 = mi.field_f32(7300 + r, w, h)
    W = mi.weights_f32(7310 + r, r)
    out, info = run(ring_ctx, "conv", w, h, r, "wrap", f0, [2, n - 2], W=W)
    assert info.exchanges >= 2 * n
    assert np.array_equal(out.view(np.uint32), oracle.conv(f0, W, n, "wrap").view(np.uint32))


@pytest.mark.parametrize("K", [2, 4, 8])
def test_life_ring_deep_halo(ring_ctx, K):
    """Deep halos over the NCCL ring: K rows exchanged once per pass."""
    w, h, n = 2048, 4 * K + 50, 3 * K + 1
    x0 = mi.life_u8(7400 + K, w, h)
    out, info = run(ring_ctx, "life", w, h, 1, "wrap", x0, [n], K=K)
    assert info.gens_per_pass == K and info.halo_rows == K
    assert info.exchanges >= 2 * (n // K)
    assert np.array_equal(out, oracle.life(x0, n, "wrap"))


@pytest.mark.parametrize("r,K", [(2, 2), (1, 2), (2, 3)])
def test_conv_ring_deep_halo(ring_ctx, r, K):
    """conv deep halos over the NCCL ring (K = 2, r <= 2: the fused two-generation kernel)."""
    w, h, n = 1024, 4 * K * r + 29, 2 * K + 1
    f0 = mi.field_f32(7500 + 10 * r + K, w, h)
    W = mi.weights_f32(7510 + r, r)
    out, info = run(ring_ctx, "conv", w, h, r, "wrap", f0, [n], W=W, K=K)
    assert info.halo_rows == K * r
    assert info.exchanges >= 2 * (n // K)
    assert np.array_equal(out.view(np.uint32), oracle.conv(f0, W, n, "wrap").view(np.uint32))


@pytest.mark.parametrize("op,r", [("life", 1), ("conv", 2)])
def test_ring_fused_p2p_self_link(ring_ctx, op, r):
    """MAPSM_OPT_EXCHANGE = P2P on the one-rank ring: the boundary CTAs store their rows
    into the slab's own halos and signal its own mailbox (no NCCL per pass)."""
    w, h, n = 2048, 300, 11
    if op == "life":
        x0 = mi.life_u8(7600, w, h)
        exp = oracle.life(x0, n, "wrap")
        out, info = run(ring_ctx, op, w, h, 1, "wrap", x0, [n], p2p=True)
        assert np.array_equal(out, exp)
    else:
        x0 = mi.field_f32(7610, w, h)
        W = mi.weights_f32(7611, r)
        out, info = run(ring_ctx, op, w, h, r, "wrap", x0, [n], W=W, p2p=True)
        assert np.array_equal(out.view(np.uint32), oracle.conv(x0, W, n, "wrap").view(np.uint32))
    assert info.exchanges >= 2 * n


def test_ring_equals_plain_context(ring_ctx, ctx):
    """The ring and the read-side row map give the same generation (65536-wide rows, 3 full TMA trips)."""
    w, h, n = 65536, 1024, 6
    x0 = mi.life_u8(7700, w, h)
    a, ia = run(ring_ctx, "life", w, h, 1, "wrap", x0, [n])
    b, ib = run(ctx, "life", w, h, 1, "wrap", x0, [n])
    assert ia.exchanges > 0 and ib.exchanges == 0
    assert np.array_equal(a, b)


@pytest.mark.parametrize("p2p", [False, True])
@pytest.mark.parametrize("k", [1, 2, 4])
@pytest.mark.parametrize("op,r,w,h", [("life", 1, 65536, 300), ("life", 1, 2048, 77), ("conv", 2, 4096, 90),
                                      ("conv", 4, 1024 + 4, 61)])
@pytest.mark.parametrize("graphs", [True, False])
def test_ring_concurrent_boundary(ring_ctx, p2p, k, op, r, w, h, graphs):
    """MAPSM_OPT_EXCHANGE_SMS = k: the boundary rows (and the NCCL group, or
    the fused peer stores) on the side stream on k SMs while the interior runs
    on the others; generation t's interior waits only for t-1's boundary rows
    and t's boundary rows for t-1's interior and halos.  Odd / even n over
    several calls (the side stream is forked and joined per call)."""
    W = mi.weights_f32(7800 + r, r) if op == "conv" else None
    x0 = mi.field_f32(7810 + w, w, h) if op == "conv" else mi.life_u8(7810 + w, w, h)
    steps = [5, 20, 1]
    n = sum(steps)
    with M.Grid(ring_ctx, w, h, op, r, "wrap", W) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        if p2p:
            g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_P2P)
        g.set_option(M.OPT_EXCHANGE_SMS, k)
        g.bind(x0)
        for s in steps:
            g.iterate(s)
        out = g.gather()
        info = g.info()
    exp = oracle.conv(x0, W, n, "wrap") if op == "conv" else oracle.life(x0, n, "wrap")
    assert info.exchanges >= 2 * n and info.launches == 2 * n
    assert np.array_equal(out.view(np.uint8), exp.view(np.uint8))


@pytest.mark.parametrize("op,r,K", [("life", 1, 4), ("life", 1, 8), ("conv", 2, 2), ("conv", 1, 2)])
def test_ring_concurrent_deep_halo(ring_ctx, op, r, K):
    """The concurrent schedule on deep-halo passes (boundary band K*r rows)."""
    w, h = 4096, 6 * K * r + 31
    W = mi.weights_f32(7900 + r, r) if op == "conv" else None
    x0 = mi.field_f32(7910, w, h) if op == "conv" else mi.life_u8(7910, w, h)
    n = 5 * K + 1
    with M.Grid(ring_ctx, w, h, op, r, "wrap", W, deep_halo=K) as g:
        g.set_option(M.OPT_EXCHANGE_SMS, 2)
        g.bind(x0)
        g.iterate(n)
        out = g.gather()
    exp = oracle.conv(x0, W, n, "wrap") if op == "conv" else oracle.life(x0, n, "wrap")
    assert np.array_equal(out.view(np.uint8), exp.view(np.uint8))


@pytest.mark.parametrize("k", [-1, 1, 3])
@pytest.mark.parametrize("op,r,w,h", [("life", 1, 65536, 300), ("life", 1, 2048, 77), ("conv", 2, 4096, 90),
                                      ("conv", 4, 1024 + 4, 61), ("conv", 1, 516, 40)])
@pytest.mark.parametrize("graphs", [True, False])
def test_ring_copy_engine_exchange(ring_ctx, k, op, r, w, h, graphs):
    """MAPSM_EXCHANGE_CE: the boundary launch waits on the mailbox for the
    neighbours' generation counts; the rows move by copy-engine peer copies
    (here: to the rank itself), followed by the count; interior beside it."""
    W = mi.weights_f32(8000 + r, r) if op == "conv" else None
    x0 = mi.field_f32(8010 + w, w, h) if op == "conv" else mi.life_u8(8010 + w, w, h)
    steps = [7, 16, 2]
    n = sum(steps)
    with M.Grid(ring_ctx, w, h, op, r, "wrap", W) as g:
        if not graphs:
            g.set_option(M.OPT_GRAPHS, 0)
        g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_CE)
        g.set_option(M.OPT_EXCHANGE_SMS, k)
        g.bind(x0)
        for s in steps:
            g.iterate(s)
        out = g.gather()
        info = g.info()
    exp = oracle.conv(x0, W, n, "wrap") if op == "conv" else oracle.life(x0, n, "wrap")
    assert info.exchanges >= 2 * n and info.launches == 2 * n
    assert np.array_equal(out.view(np.uint8), exp.view(np.uint8))


def test_copy_engine_exchange_needs_nccl_context(local_ctx):
    with M.Grid(local_ctx(2), 256, 64, "life", 1, "wrap") as g:
        with pytest.raises(M.MapsmError):
            g.set_option(M.OPT_EXCHANGE, M.EXCHANGE_CE)


def test_ring_config2_full_grid_two_generations(ring_ctx):
    """BASELINE configs[2] (65536^2 WRAP, seed 0x5EED0003) through the NCCL
    ring in the bench's nccl_ring configuration (default concurrent-boundary
    schedule, CUDA graphs): generations 1 and 2, every cell."""
    import torch

    w = h = 65536
    g0 = np.empty((h, w), np.uint8)
    mi.life_u8(mi.SEED_LIFE_64K, w, h, out=g0)
    dev = torch.empty((h, w), dtype=torch.uint8, device="cuda")
    with M.Grid(ring_ctx, w, h, "life", 1, "wrap") as g:
        g.bind(g0)
        g.iterate(1)
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
        exp = oracle.life(g0, 1, "wrap")
        del g0
        assert torch.equal(dev, torch.from_numpy(exp).cuda()), "generation 1"
        g.iterate(1)
        M.mapsm_read(g.handle, dev)
        torch.cuda.synchronize()
        assert g.info().exchanges >= 4
    exp = oracle.life(exp, 1, "wrap")
    assert torch.equal(dev, torch.from_numpy(exp).cuda()), "generation 2"


def test_ring_life_slab_deep_halo_full_grid():
    """One GPU's slab at N = 8 (65536 x 8192) with deep halos K = 8 over the
    ring, 16 generations in 2 passes (the E(8) prediction's path), every cell."""
    import torch

    torch.cuda.set_device(0)
    c = M.mapsm_ctx_create(0, 1, 0, M.mapsm_nccl_unique_id(), None)
    try:
        w, h, n = 65536, 8192, 16
        g0 = mi.life_u8(mi.SEED_LIFE_64K, w, h)
        with M.Grid(c, w, h, "life", 1, "wrap", deep_halo=8) as g:
            g.bind(g0)
            g.iterate(n)
            out = g.gather()
            assert g.info().exchanges >= 4
    finally:
        M.mapsm_ctx_destroy(c)
    assert np.array_equal(out, oracle.life(g0, n, "wrap"))


@pytest.mark.parametrize("K", [1, 2])
def test_ring_conv5_full_grid(ring_ctx, K):
    """The 5x5 16384^2 field (seeds 0x5EED0004 / 0x5EED0044) under WRAP through
    the ring: per generation (K = 1) and the two-generation kernel (K = 2)."""
    w = h = 16384
    f0 = mi.field_f32(mi.SEED_CONV5_FIELD, w, h)
    W = mi.weights_f32(mi.SEED_CONV5_W, 2)
    with M.Grid(ring_ctx, w, h, "conv", 2, "wrap", W, deep_halo=K) as g:
        g.bind(f0)
        g.iterate(2)
        got = g.gather()
    assert np.array_equal(got.view(np.uint32), oracle.conv(f0, W, 2, "wrap").view(np.uint32))


def test_no_exchange_toggle_after_graph_capture(ring_ctx):
    """MAPSM_OPT_NO_EXCHANGE set after CUDA graphs were captured must take
    effect (the captured passes hold the old schedule and are dropped): with
    the exchange off the halos go stale and the result leaves the oracle's;
    with it back on and a fresh bind it matches again."""
    w, h = 2048, 64
    x0 = mi.life_u8(8100, w, h)
    with M.Grid(ring_ctx, w, h, "life", 1, "wrap") as g:
        g.bind(x0)
        g.iterate(32)  # graphs captured with the exchange
        assert np.array_equal(g.gather(), oracle.life(x0, 32, "wrap"))
        g.set_option(M.OPT_NO_EXCHANGE, 1)
        g.iterate(32)
        stale = g.gather()
        assert not np.array_equal(stale, oracle.life(x0, 64, "wrap"))
        g.set_option(M.OPT_NO_EXCHANGE, 0)
        g.bind(x0)
        g.iterate(64)
        assert np.array_equal(g.gather(), oracle.life(x0, 64, "wrap"))
