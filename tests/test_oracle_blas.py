"""Pins for the unmodified-routine oracle (oracle/blas.py; SURVEY §8(f)
NEXT-4, Fig 5): exact small-integer products (a plain
triple loop in Python integers), identity / permutation closed forms, and the
forward-error bound checked against exact rational arithmetic of an fp32
evaluation (np.float32 sequential sums) and against numpy's float32 matmul.
CPU only."""
from fractions import Fraction

import numpy as np

from oracle import blas


def test_integer_product_exact():
    rng = np.random.default_rng(1)
    A = rng.integers(-9, 10, (7, 5))
    B = rng.integers(-9, 10, (5, 4))
    C = rng.integers(-9, 10, (7, 4))
    ref = [[3 * sum(int(A[i, t]) * int(B[t, j]) for t in range(5)) - 2 * int(C[i, j]) for j in range(4)]
           for i in range(7)]
    assert np.array_equal(blas.sgemm(A, B, C, 3.0, -2.0), np.array(ref, np.float64))


def test_identity_and_permutation():
    rng = np.random.default_rng(2)
    A = rng.random((6, 6)).astype(np.float32)
    I = np.eye(6, dtype=np.float32)
    P = I[[3, 0, 5, 1, 4, 2]]
    assert np.array_equal(blas.sgemm(A, I), A.astype(np.float64))
    assert np.array_equal(blas.sgemm(P, A), A[[3, 0, 5, 1, 4, 2]].astype(np.float64))
    assert np.array_equal(blas.saxpy(A[0], A[1], 0.0), A[1].astype(np.float64))


def test_bound_holds_for_sequential_fp32_and_numpy():
    rng = np.random.default_rng(3)
    A = (rng.random((9, 33)) - 0.3).astype(np.float32)
    B = (rng.random((33, 5)) - 0.6).astype(np.float32)
    exact = np.array([[float(sum(Fraction(float(A[i, t])) * Fraction(float(B[t, j])) for t in range(33)))
                       for j in range(5)] for i in range(9)])
    seq = np.zeros((9, 5), np.float32)
    for t in range(33):
        seq = (seq + A[:, t:t + 1] * B[t:t + 1, :]).astype(np.float32)
    bound = blas.sgemm_bound(A, B)
    assert np.all(np.abs(seq - exact) <= bound)
    assert np.all(np.abs((A @ B).astype(np.float64) - exact) <= bound)
    assert np.max(np.abs(blas.sgemm(A, B) - exact)) <= 1e-12 * np.max(np.abs(exact))
    assert np.any(np.abs(seq - exact) > 0)   # fp32 really rounds


def test_saxpy_bound():
    rng = np.random.default_rng(4)
    x = (rng.random(1000) - 0.5).astype(np.float32)
    y = (rng.random(1000) - 0.5).astype(np.float32)
    a = np.float32(1.7)
    got = (a * x + y).astype(np.float32)
    assert np.all(np.abs(got - blas.saxpy(x, y, a)) <= blas.saxpy_bound(x, y, a))
