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


# ------------------------------------------------------------ gloo, 2 ranks

def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_main(rank, world, port, boundary, n, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    h, w, r = 20, 64, 1
    g0 = mi.life_u8(1234, w, h)
    plans = [M.mapsm_plan_query(h, world, r, boundary, k) for k in range(world)]
    p = plans[rank]
    mine = g0[p.y0:p.y0 + p.rows].copy()
    for _ in range(n):
        top = np.zeros((r, w), np.uint8)
        bot = np.zeros((r, w), np.uint8)
        reqs = []
        # exactly the order of exchange_nccl(): send-up, send-down, recv-bottom, recv-top
        t_send_top = torch.from_numpy(mine[:r].copy())
        t_send_bot = torch.from_numpy(mine[-r:].copy())
        t_recv_bot = torch.zeros((r, w), dtype=torch.uint8)
        t_recv_top = torch.zeros((r, w), dtype=torch.uint8)
        if p.top_kind == M.HALO_EXCHANGE:
            reqs.append(dist.isend(t_send_top, p.up))
        if p.bottom_kind == M.HALO_EXCHANGE:
            reqs.append(dist.isend(t_send_bot, p.down))
        if p.bottom_kind == M.HALO_EXCHANGE:
            reqs.append(dist.irecv(t_recv_bot, p.down))
        if p.top_kind == M.HALO_EXCHANGE:
            reqs.append(dist.irecv(t_recv_top, p.up))
        for q in reqs:
            q.wait()
        if p.top_kind == M.HALO_EXCHANGE:
            top = t_recv_top.numpy()
        else:
            top = halo_rows(p, mine, None, plans, "top", r, h)
        if p.bottom_kind == M.HALO_EXCHANGE:
            bot = t_recv_bot.numpy()
        else:
            bot = halo_rows(p, mine, None, plans, "bottom", r, h)
        mine = step_slab("life", np.concatenate([top, mine, bot]), r, boundary, None)
    # gather to root over gloo
    out = [torch.zeros((q.rows, w), dtype=torch.uint8) for q in plans]
    dist.all_gather(out, torch.from_numpy(mine)) if all(q.rows == p.rows for q in plans) else None
    if rank == 0:
        full = np.concatenate([o.numpy() for o in out])
        result_q.put(bool(np.array_equal(full, oracle.life(g0, n, NAMES[boundary]))))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("b", [M.WRAP, M.CLAMP])
def test_two_rank_gloo_exchange_order(b):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(k, 2, port, b, 9, q)) for k in range(2)]
    for pr in procs:
        pr.start()
    ok = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert ok
