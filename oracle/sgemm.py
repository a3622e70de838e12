"""fp64 SGEMM oracle.  TEST INFRASTRUCTURE ONLY.

C*_ij = alpha * sum_k (double)A_ik (double)B_kj + beta * (double)C0_ij — the
Parboil sgemm the paper profiles (§4.3; work-assignment factor
16x between its two GPU versions).  Row-major, no transposes
(reading A-17 in DESIGN.md).  The matmul is a library primitive (numpy fp64).

Pinned by tests/test_oracle_sgemm.py: triple loop on small shapes, B = I closed
form, small-integer exactness; sgemm_abs by tests/test_oracle_denominators.py
(explicit triple loop of |A||B| + |beta||C0|, non-square, negative scalars,
hand example).
"""
from __future__ import annotations

import numpy as np


def sgemm(A, B, C0, alpha, beta) -> np.ndarray:
    A64 = np.asarray(A, np.float64)
    B64 = np.asarray(B, np.float64)
    return float(alpha) * (A64 @ B64) + float(beta) * np.asarray(C0, np.float64)


def sgemm_abs(A, B, C0, alpha, beta) -> np.ndarray:
    """d_ij = |alpha| sum_k |A_ik||B_kj| + |beta||C0_ij| (c-2 denominator)."""
    return (abs(float(alpha)) * (np.abs(np.asarray(A, np.float64)) @ np.abs(np.asarray(B, np.float64)))
            + abs(float(beta)) * np.abs(np.asarray(C0, np.float64)))


def sgemm_entries(A, B, C0, alpha, beta, idx):
    """(C*, d) at sampled (i, j) pairs, each as its own dot product."""
    y = np.empty(len(idx))
    d = np.empty(len(idx))
    for t, (i, j) in enumerate(idx):
        a = np.asarray(A[i, :], np.float64)
        b = np.asarray(B[:, j], np.float64)
        c0 = float(C0[i, j])
        y[t] = float(alpha) * float(np.dot(a, b)) + float(beta) * c0
        d[t] = abs(float(alpha)) * float(np.dot(np.abs(a), np.abs(b))) + abs(float(beta)) * abs(c0)
    return y, d


SGEMM_TOL = 1e-4  # north_star: "1e-4 for SGEMM variants"
