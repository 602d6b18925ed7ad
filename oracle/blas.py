"""Dense linear algebra for the unmodified-routine tasks — TEST INFRASTRUCTURE ONLY.

The unmodified routines of SURVEY §8(f) NEXT-4 (§4.6, Fig 5; the
8K matrix-multiplication chain of P:L491-508 §5.4) compute plain BLAS
operations, so the oracle is their definition in float64 (numpy's matmul is
the library step), plus the textbook forward-error bound any fp32
evaluation order satisfies (Higham, Accuracy and Stability, Thm 3.5 with
gamma_n = n u / (1 - n u), u = 2^-24), which is what the fp32 GPU results are
checked against (reading u1 in DESIGN.md).  Only tests/ and bench.py's
cpu_baseline leg may import this module.
"""
from __future__ import annotations

import numpy as np

U32 = 2.0 ** -24


def gamma(n: int, u: float = U32) -> float:
    return n * u / (1 - n * u)


def sgemm(A, B, C=None, alpha=1.0, beta=0.0) -> np.ndarray:
    """alpha * A @ B + beta * C in float64 (C may be None when beta == 0)."""
    out = float(alpha) * (np.asarray(A, np.float64) @ np.asarray(B, np.float64))
    if beta != 0.0:
        out += float(beta) * np.asarray(C, np.float64)
    return out


def sgemm_bound(A, B, C=None, alpha=1.0, beta=0.0) -> np.ndarray:
    """Elementwise bound on |fl32(alpha A B + beta C) - exact| for any order of
    the k products (fp32 inputs, fp32 accumulation, FMA or not)."""
    k = np.asarray(A).shape[1]
    mag = abs(float(alpha)) * (np.abs(np.asarray(A, np.float64)) @ np.abs(np.asarray(B, np.float64)))
    if beta != 0.0:
        mag += abs(float(beta)) * np.abs(np.asarray(C, np.float64))
    return gamma(k + 2) * mag


def saxpy(x, y, alpha) -> np.ndarray:
    """alpha * x + y in float64."""
    return float(alpha) * np.asarray(x, np.float64) + np.asarray(y, np.float64)


def saxpy_bound(x, y, alpha) -> np.ndarray:
    return gamma(2) * (abs(float(alpha)) * np.abs(np.asarray(x, np.float64)) + np.abs(np.asarray(y, np.float64)))
