"""Multi-slab host logic on CPU: the plan + halo protocol reproduce the
whole-grid oracle for every g (partition invariance: kernels run
on multiple GPUs without modification), including a real 2-process exchange
over torch.distributed (gloo) with the library's fixed send/recv order."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import mapsm_inputs as mi
import oracle
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M
from slabsim import halo_rows, simulate, step_slab

NAMES = {M.WRAP: "wrap", M.CLAMP: "clamp", M.ZERO: "zero"}


@pytest.mark.parametrize("g", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("b", [M.WRAP, M.CLAMP, M.ZERO])
def test_life_partition_invariance(g, b):
    h, w, n = 37, 48, 7
    g0 = mi.life_u8(99, w, h)
    assert np.array_equal(simulate("life", g0, n, 1, b, g), oracle.life(g0, n, NAMES[b]))


@pytest.mark.parametrize("g", [1, 2, 5, 8])
@pytest.mark.parametrize("b", [M.WRAP, M.CLAMP, M.ZERO])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_conv_partition_invariance_bit_exact(g, b, r):
    h, w, n = 8 * 4 + 3, 21, 3
    if h // g < r:
        pytest.skip("slab shorter than r")
    f0 = mi.field_f32(5, w, h)
    W = mi.weights_f32(6 + r, r)
    got = simulate("conv", f0, n, r, b, g, W)
    exp = oracle.conv(f0, W, n, NAMES[b])
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))


def test_min_height_slabs_g8_r2():
    f0 = mi.field_f32(7, 16, 16)
    W = mi.weights_f32(8, 2)
    got = simulate("conv", f0, 4, 2, M.WRAP, 8, W)
    assert np.array_equal(got, oracle.conv(f0, W, 4, "wrap"))


# ----------------------------------------- the data plane's message lists

@pytest.mark.parametrize("g", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("b", [M.WRAP, M.CLAMP, M.ZERO])
@pytest.mark.parametrize("r,depth", [(1, 1), (2, 2), (4, 4), (1, 8)])
def test_exchange_plan_messages_match_pairwise(g, b, r, depth):
    """Every receive of the list is matched, by NCCL's pair-wise issue-order
    rule, with a send of the same size carrying exactly the global rows the
    receiver's halo needs (P:L461 two-line exchanges; Alg 2 line 10)."""
    h, pitch = 8 * g * depth + 3, 40
    if h // g < depth:
        pytest.skip("slab shorter than the halo")
    halo = depth
    lists = [M.mapsm_exchange_plan(h, g, r, b, k, depth, halo, pitch) for k in range(g)]
    plans = [M.mapsm_plan_query(h, g, r, b, k) for k in range(g)]
    for k, msgs in enumerate(lists):
        p = plans[k]
        kinds = [(m.kind, m.row) for m in msgs]
        # the fixed order: send-up, send-down, recv-bottom, recv-top
        exp = []
        if p.top_kind == M.HALO_EXCHANGE:
            exp.append((M.MSG_SEND, 0))
        if p.bottom_kind == M.HALO_EXCHANGE:
            exp.append((M.MSG_SEND, p.rows - depth))
        if p.bottom_kind == M.HALO_EXCHANGE:
            exp.append((M.MSG_RECV, p.rows))
        if p.top_kind == M.HALO_EXCHANGE:
            exp.append((M.MSG_RECV, -depth))
        assert kinds == exp
        for m in msgs:
            assert m.rows == depth and m.bytes == depth * pitch and m.offset == (m.row + halo) * pitch
        for j, m in enumerate(msgs):
            if m.kind != M.MSG_RECV:
                continue
            nth = sum(1 for q in msgs[:j] if q.kind == M.MSG_RECV and q.peer == m.peer)
            sends = [q for q in lists[m.peer] if q.kind == M.MSG_SEND and q.peer == k]
            src = sends[nth]
            assert src.bytes == m.bytes
            # the sender's rows are the global rows my halo stands for
            assert src.global_row == m.global_row == (p.y0 + m.row) % h


@pytest.mark.parametrize("g", [1, 2, 3, 5])
@pytest.mark.parametrize("root", [0, 1])
def test_gather_plan_covers_every_row_once(g, root):
    if root >= g:
        pytest.skip("root outside the world")
    h, pitch, halo = 29, 16, 1
    plans = [M.mapsm_plan_query(h, g, 1, M.WRAP, k) for k in range(g)]
    covered = np.zeros(h, int)
    covered[plans[root].y0:plans[root].y0 + plans[root].rows] += 1  # the root's own rows
    recvs = M.mapsm_gather_plan(h, g, 1, M.WRAP, root, root, halo, pitch)
    assert [m.peer for m in recvs] == [k for k in range(g) if k != root]
    for k in range(g):
        if k == root:
            continue
        (snd,) = M.mapsm_gather_plan(h, g, 1, M.WRAP, k, root, halo, pitch)
        rcv = recvs[[m.peer for m in recvs].index(k)]
        assert snd.kind == M.MSG_SEND and snd.peer == root and rcv.kind == M.MSG_RECV
        assert snd.bytes == rcv.bytes == plans[k].rows * pitch and snd.offset == halo * pitch
        covered[rcv.global_row:rcv.global_row + rcv.rows] += 1
    assert (covered == 1).all()


# ------------------------------------------------------------ gloo, N ranks

def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run_msgs(buf, msgs):
    """Issue a message list in order over torch.distributed (gloo pairs match
    in issue order, as NCCL's do) and wait for all of it."""
    reqs = []
    for m in msgs:
        view = torch.from_numpy(buf[m.offset:m.offset + m.bytes])
        reqs.append(dist.isend(view, m.peer) if m.kind == M.MSG_SEND else dist.irecv(view, m.peer))
    for q in reqs:
        q.wait()


def _rank_main(rank, world, port, boundary, op, r, n, result_q):
    """One rank of the data plane, driven ONLY by the library's message lists
    (mapsm_exchange_plan / mapsm_gather_plan): the slab buffer is laid out as
    the device buffer is ([r halo rows | owned rows | r halo rows], pitch
    bytes per row), the exchange moves bytes at the listed offsets, the step
    is the oracle on the slab.  A change of order, offsets or sizes in the
    lists (which exchange_nccl and the gather iterate) breaks the result."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    h, w = 23, 24
    if op == "life":
        g0 = mi.life_u8(1234, w, h)
        W, dt = None, np.uint8
    else:
        g0 = mi.field_f32(1235, w, h)
        W, dt = mi.weights_f32(1236, r), np.float32
    pitch = w * np.dtype(dt).itemsize
    plans = [M.mapsm_plan_query(h, world, r, boundary, k) for k in range(world)]
    p = plans[rank]
    buf = np.zeros((p.rows + 2 * r) * pitch, np.uint8)
    rows = buf.view(dt).reshape(p.rows + 2 * r, w)
    rows[r:r + p.rows] = g0[p.y0:p.y0 + p.rows]
    for _ in range(n):
        _run_msgs(buf, M.mapsm_exchange_plan(h, world, r, boundary, rank, r, r, pitch))
        mine = rows[r:r + p.rows]
        if p.top_kind != M.HALO_EXCHANGE:
            rows[:r] = halo_rows(p, mine, None, plans, "top", r, h)
        if p.bottom_kind != M.HALO_EXCHANGE:
            rows[r + p.rows:] = halo_rows(p, mine, None, plans, "bottom", r, h)
        rows[r:r + p.rows] = step_slab(op, rows.copy(), r, boundary, W)
    msgs = M.mapsm_gather_plan(h, world, r, boundary, rank, 0, r, pitch)
    if rank != 0:
        _run_msgs(buf, msgs)
    else:
        full = np.zeros((h, w), dt)
        full[p.y0:p.y0 + p.rows] = rows[r:r + p.rows]
        stage = np.zeros(max(m.bytes for m in msgs) if msgs else 1, np.uint8)
        for m in msgs:  # one at a time through the staging buffer, as the root does
            _run_msgs(stage, [m])
            full[m.global_row:m.global_row + m.rows] = stage[:m.bytes].view(dt).reshape(m.rows, w)
        exp = oracle.life(g0, n, NAMES[boundary]) if op == "life" else oracle.conv(g0, W, n, NAMES[boundary])
        result_q.put(bool(np.array_equal(full.view(np.uint8), exp.view(np.uint8))))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,b,op,r", [(2, M.WRAP, "life", 1), (2, M.CLAMP, "life", 1), (3, M.WRAP, "life", 1),
                                          (3, M.ZERO, "conv", 2), (2, M.WRAP, "conv", 2)])
def test_gloo_data_plane_from_message_lists(world, b, op, r):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(k, world, port, b, op, r, 5, q)) for k in range(world)]
    for pr in procs:
        pr.start()
    ok = q.get(timeout=180)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert ok
