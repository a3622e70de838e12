"""Pins of the power-iteration oracle against closed forms
and library eigen-solvers, independent of the oracle's own code."""
import numpy as np

from oracle import iterative
from workloads import laplacian_2d, uniform_f32, CSR


def test_laplacian_closed_form_eigenvalue():
    N = 6
    A = laplacian_2d(N)
    x0 = uniform_f32(5, A.n_cols, 0.5, 1.0)      # positive start: overlaps the top eigenvector
    _, _, norms = iterative.power_iteration(A.row_ptr, A.col, A.val, x0, 600)
    assert abs(norms[-1] - iterative.laplacian_2d_lambda_max(N)) < 1e-6


def test_laplacian_matrix_matches_definition():
    N = 5
    A = laplacian_2d(N)
    dense = np.zeros((N * N, N * N))
    for r in range(N * N):
        dense[r, A.col[A.row_ptr[r]:A.row_ptr[r + 1]]] = A.val[A.row_ptr[r]:A.row_ptr[r + 1]]
    T = 2 * np.eye(N) - np.eye(N, k=1) - np.eye(N, k=-1)
    assert np.array_equal(dense, np.kron(T, np.eye(N)) + np.kron(np.eye(N), T))   # textbook Kronecker form
    ev = np.linalg.eigvalsh(dense)
    assert abs(ev.max() - iterative.laplacian_2d_lambda_max(N)) < 1e-12


def test_symmetric_matrix_vs_eigvalsh():
    g = np.random.default_rng(3)
    n = 40
    B = g.uniform(-1, 1, (n, n))
    S = (B + B.T) / 2 + np.diag(np.arange(n) * 0.5)      # well separated top eigenvalue
    rp = np.arange(0, n * n + 1, n, dtype=np.int32)
    col = np.tile(np.arange(n, dtype=np.int32), n)
    val = S.astype(np.float32).ravel()
    Sf = val.astype(np.float64).reshape(n, n)
    _, _, norms = iterative.power_iteration(rp, col, val, np.ones(n), 400)
    assert abs(norms[-1] - np.abs(np.linalg.eigvalsh(Sf)).max()) < 1e-8


def test_one_step_is_normalised_product():
    A = laplacian_2d(4)
    x0 = uniform_f32(9, A.n_cols)
    x1, y0, norms = iterative.power_iteration(A.row_ptr, A.col, A.val, x0, 1)
    dense = np.zeros((16, 16))
    for r in range(16):
        dense[r, A.col[A.row_ptr[r]:A.row_ptr[r + 1]]] = A.val[A.row_ptr[r]:A.row_ptr[r + 1]]
    ref = dense @ x0.astype(np.float64)
    assert np.allclose(y0, ref, rtol=0, atol=1e-14)
    assert np.allclose(x1, ref / np.linalg.norm(ref), rtol=0, atol=1e-15)
    assert abs(norms[0] - np.linalg.norm(ref)) < 1e-13


def test_zero_matrix_gives_zero_vector():
    A = CSR(3, 3, np.zeros(4, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    x, y, norms = iterative.power_iteration(A.row_ptr, A.col, A.val, np.ones(3), 2)
    assert not x.any() and not y.any() and not norms.any()
