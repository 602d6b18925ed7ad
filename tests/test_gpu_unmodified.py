"""GPU parity: unmodified routines (§4.6,
Fig 5; §5.4) — cuBLAS SGEMM / SAXPY wrappers run per slab on the
segments the access patterns imply, data moved by the Segment Location
Monitor.  Results within the oracle's fp32 forward-error bound
(oracle/blas.py, reading u1); bytes moved equal to what Alg 2 must move (and
zero for a chain on unchanged inputs)."""
import ctypes

import numpy as np
import pytest

from oracle import blas
from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

pytestmark = pytest.mark.gpu


def rows_of(m, g):
    base, extra = divmod(m, g)
    return [base + (1 if k < extra else 0) for k in range(g)]


def mat(ctx, a):
    h = M.mapsm_matrix_create(ctx, a.shape[0], a.shape[1])
    M.mapsm_matrix_bind(h, np.ascontiguousarray(a, np.float32))
    return h


def gather(h, shape):
    out = np.empty(shape, np.float32)
    M.mapsm_matrix_gather(h, out)
    return out


def within(got, exact, bound):
    assert np.all(np.abs(got.astype(np.float64) - exact) <= bound + 1e-30)


@pytest.mark.parametrize("G", [1, 2, 3, 4])
@pytest.mark.parametrize("mkn", [(64, 32, 48), (1000, 257, 129), (7, 5, 3)])
def test_sgemm_vs_oracle_and_moves(local_ctx, G, mkn):
    m, k, n = mkn
    rng = np.random.default_rng(m + k + n + G)
    A = (rng.random((m, k)) - 0.5).astype(np.float32)
    B = (rng.random((k, n)) - 0.5).astype(np.float32)
    C0 = (rng.random((m, n)) - 0.5).astype(np.float32)
    c = local_ctx(G)
    hA, hB, hC = mat(c, A), mat(c, B), mat(c, C0)
    try:
        pats = [M.PAT_BLOCK2D, M.PAT_BLOCK2D_T, M.PAT_INOUT_SI]
        moved = M.mapsm_invoke_unmodified(c, m, "sgemm", [hA, hB, hC], pats, (1.5, -0.5))
        C = gather(hC, (m, n))
        within(C, blas.sgemm(A, B, C0, 1.5, -0.5), blas.sgemm_bound(A, B, C0, 1.5, -0.5))
        # Alg 2: every slab but slab 0 (where bind put the data) receives its
        # rows of A and of C, and all of B
        r = rows_of(m, G)
        expect = 4 * ((m - r[0]) * k + (G - 1) * k * n + (m - r[0]) * n)
        assert moved == expect
        # chain: inputs unchanged -> nothing moves; C is an output only
        moved2 = M.mapsm_invoke_unmodified(c, m, "sgemm", [hA, hB, hC], [M.PAT_BLOCK2D, M.PAT_BLOCK2D_T,
                                                                          M.PAT_OUT_SI], (1.0, 0.0))
        assert moved2 == 0
        C2 = gather(hC, (m, n))
        within(C2, blas.sgemm(A, B), blas.sgemm_bound(A, B))
    finally:
        for h in (hA, hB, hC):
            M.mapsm_matrix_destroy(h)


def test_chain_output_feeds_next_task(local_ctx):
    """D = (A B) B2: C's row blocks stay on their slabs (SI output, then
    Block(2D) input of the same partition) — only B2 moves."""
    G, m, k, n, p = 3, 300, 64, 96, 40
    rng = np.random.default_rng(7)
    A = (rng.random((m, k)) - 0.5).astype(np.float32)
    B = (rng.random((k, n)) - 0.5).astype(np.float32)
    B2 = (rng.random((n, p)) - 0.5).astype(np.float32)
    c = local_ctx(G)
    hA, hB, hB2 = mat(c, A), mat(c, B), mat(c, B2)
    hC = M.mapsm_matrix_create(c, m, n)
    hD = M.mapsm_matrix_create(c, m, p)
    try:
        M.mapsm_invoke_unmodified(c, m, "sgemm", [hA, hB, hC], [0, 1, 2], (1.0, 0.0))
        moved = M.mapsm_invoke_unmodified(c, m, "sgemm", [hC, hB2, hD], [0, 1, 2], (1.0, 0.0))
        assert moved == 4 * (G - 1) * n * p
        C = gather(hC, (m, n))
        D = gather(hD, (m, p))
        within(C, blas.sgemm(A, B), blas.sgemm_bound(A, B))
        within(D, blas.sgemm(C, B2), blas.sgemm_bound(C, B2))
    finally:
        for h in (hA, hB, hB2, hC, hD):
            M.mapsm_matrix_destroy(h)


@pytest.mark.parametrize("G", [1, 4])
def test_saxpy_fig5(local_ctx, G):
    n = 100003
    rng = np.random.default_rng(11)
    x = (rng.random((n, 1)) - 0.5).astype(np.float32)
    y = (rng.random((n, 1)) - 0.5).astype(np.float32)
    c = local_ctx(G)
    hx, hy = mat(c, x), mat(c, y)
    try:
        exp = y.astype(np.float64)
        for _ in range(3):
            yprev = exp
            M.mapsm_invoke_unmodified(c, n, "saxpy", [hx, hy], [M.PAT_BLOCK2D, M.PAT_INOUT_SI], (2.5,))
            exp = blas.saxpy(x, yprev, 2.5)
        got = gather(hy, (n, 1))
        within(got, exp, 3 * blas.saxpy_bound(x, np.abs(exp) + 1, 2.5))
    finally:
        M.mapsm_matrix_destroy(hx)
        M.mapsm_matrix_destroy(hy)


def test_user_routine_gets_the_pattern_segments(local_ctx):
    """A Python wrapper (the predetermined prototype) sees, per slab,
    its row block of a Block(2D) parameter and the whole Block(2D-T) one."""
    G, m = 3, 10
    c = local_ctx(G)
    hA = mat(c, np.ones((m, 4), np.float32))
    hB = mat(c, np.ones((6, 4), np.float32))
    seen = []

    @M.ROUTINE
    def rt(ctxp, slab, device, stream, segs, nsegs, scalars, nscalars):
        seen.append((slab, [(segs[i].row0, segs[i].rows, segs[i].cols) for i in range(nsegs)], scalars[0]))
        return 0

    try:
        M.mapsm_invoke_unmodified(c, m, rt, [hA, hB], [M.PAT_BLOCK2D, M.PAT_BLOCK2D_T], (7.0,))
        assert [s[0] for s in seen] == [0, 1, 2]
        assert [s[1][0] for s in seen] == [(0, 4, 4), (4, 3, 4), (7, 3, 4)]
        assert all(s[1][1] == (0, 6, 4) and s[2] == 7.0 for s in seen)

        @M.ROUTINE
        def bad(*a):
            return 5
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_invoke_unmodified(c, m, bad, [hA], [M.PAT_BLOCK2D])
        assert e.value.status == M.ECUDA
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_invoke_unmodified(c, m + 1, "saxpy", [hA, hA], [M.PAT_BLOCK2D, M.PAT_INOUT_SI], (1.0,))
        assert e.value.status == M.EINVAL
        hN = M.mapsm_matrix_create(c, m, 4)
        with pytest.raises(M.MapsmError) as e:
            M.mapsm_invoke_unmodified(c, m, "saxpy", [hN, hA], [M.PAT_BLOCK2D, M.PAT_INOUT_SI], (1.0,))
        assert e.value.status == M.ESTATE
        M.mapsm_matrix_destroy(hN)
    finally:
        M.mapsm_matrix_destroy(hA)
        M.mapsm_matrix_destroy(hB)


def test_sgemm_8k_sampled(ctx):
    """The bench size (8192^2, the paper's 8K matrices) on sampled
    rows and columns against the fp64 oracle and its bound."""
    n = 8192
    rng = np.random.default_rng(5)
    A = (rng.random((n, n), dtype=np.float32) - 0.5)
    B = (rng.random((n, n), dtype=np.float32) - 0.5)
    hA, hB = mat(ctx, A), mat(ctx, B)
    hC = M.mapsm_matrix_create(ctx, n, n)
    try:
        M.mapsm_invoke_unmodified(ctx, n, "sgemm", [hA, hB, hC], [0, 1, 2], (1.0, 0.0))
        C = gather(hC, (n, n))
        ri = rng.choice(n, 16, replace=False)
        ci = rng.choice(n, 16, replace=False)
        sub = blas.sgemm(A[ri], B[:, ci])
        within(C[np.ix_(ri, ci)], sub, blas.sgemm_bound(A[ri], B[:, ci]))
    finally:
        for h in (hA, hB, hC):
            M.mapsm_matrix_destroy(h)
