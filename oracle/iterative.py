"""fp64 power-iteration oracle for the iterative driver.
TEST INFRASTRUCTURE ONLY (tests/, __graft_entry__.smoke(), bench.py's CPU leg).

The paper's iterative usage: an iterative kernel is micro-profiled on its first
invocation and the selection reused while the profiling activation flag is off
(§3.1); §5.2 studies the per-iteration overhead of profiling every
iteration.  The loop computed around the DySel SpMV is the plain
power iteration, written out step by step:

    y_k     = A x_k                 (oracle.spmv.spmv, fp64, CSR order)
    x_{k+1} = y_k / ||y_k||_2       (x_{k+1} = 0 when y_k = 0)

Pinned by tests/test_oracle_iterative.py: for the 2-D Dirichlet Laplacian the
norms converge to the closed-form largest eigenvalue
4 + 4 cos(pi / (N + 1)); for small symmetric matrices they converge to the
largest-magnitude eigenvalue of numpy.linalg.eigvalsh; one step equals
A x / ||A x|| computed densely.
"""
from __future__ import annotations

import numpy as np

from . import spmv as ospmv


def power_iteration(row_ptr, col, val, x0, n_iter):
    """Returns (x_n, y_{n-1}, norms[k] = ||y_k||_2) in fp64."""
    x = np.asarray(x0, np.float64).copy()
    y = np.zeros_like(x)
    norms = np.zeros(n_iter, np.float64)
    for k in range(n_iter):
        y = ospmv.spmv(row_ptr, col, val, x)
        nr = float(np.sqrt(np.dot(y, y)))
        norms[k] = nr
        x = y / nr if nr > 0.0 else np.zeros_like(y)
    return x, y, norms


def laplacian_2d_lambda_max(grid: int) -> float:
    """Closed form: eigenvalues of the 5-point Dirichlet Laplacian are
    4 - 2 cos(p pi/(N+1)) - 2 cos(q pi/(N+1)), p, q = 1..N; the largest is at
    p = q = N: 4 + 4 cos(pi/(N+1))."""
    return 4.0 + 4.0 * np.cos(np.pi / (grid + 1))
