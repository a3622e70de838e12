"""Pins for oracle/sgemm.py and oracle/c/oracle_ref.c (SURVEY c-2)."""
import numpy as np
import pytest

from oracle import ref_c, sgemm, spmv
from workloads import random_lengths_csr, sgemm_inputs, small_int_gemm, uniform_f32


def triple_loop(A, B, C0, alpha, beta):
    M, K = A.shape
    N = B.shape[1]
    C = np.zeros((M, N))
    for i in range(M):
        for j in range(N):
            s = 0.0
            for k in range(K):
                s += float(A[i, k]) * float(B[k, j])
            C[i, j] = alpha * s + beta * float(C0[i, j])
    return C


def test_triple_loop_non_square():
    A, B, C0 = sgemm_inputs(13, 7, 9, 1, 2, 3)      # M != K != N: a transpose shows
    C = sgemm.sgemm(A, B, C0, 1.5, -0.5)
    assert np.allclose(C, triple_loop(A, B, C0, 1.5, -0.5), rtol=1e-13, atol=1e-13)


def test_identity_closed_form():
    A, _, C0 = sgemm_inputs(40, 24, 24, 4, 5, 6)
    I = np.eye(24, dtype=np.float32)
    C = sgemm.sgemm(A, I, C0, 1.5, -0.5)
    assert np.array_equal(C, 1.5 * A.astype(np.float64) - 0.5 * C0.astype(np.float64))


def test_small_integer_exact():
    A, B, C0 = small_int_gemm(64, 1024, 48, 9)
    C = sgemm.sgemm(A, B, C0, 1.0, 1.0)
    Ci = A.astype(np.int64) @ B.astype(np.int64) + C0.astype(np.int64)   # exact integer arithmetic
    assert np.array_equal(C, Ci.astype(np.float64))
    assert np.abs(Ci).max() < 2 ** 24


def test_abs_and_entries():
    A, B, C0 = sgemm_inputs(20, 30, 10, 7, 8, 9)
    d = sgemm.sgemm_abs(A, B, C0, 1.5, -0.5)
    C = sgemm.sgemm(A, B, C0, 1.5, -0.5)
    idx = [(0, 0), (19, 9), (7, 3)]
    ys, ds = sgemm.sgemm_entries(A, B, C0, 1.5, -0.5, idx)
    for t, (i, j) in enumerate(idx):
        assert abs(ys[t] - C[i, j]) <= 1e-13 and abs(ds[t] - d[i, j]) <= 1e-13
        assert ds[t] >= abs(ys[t]) - 1e-12


# ------------------------------------------------ C oracle (CPU baseline copy)
@pytest.mark.parametrize("threads", [1, 4])
def test_c_oracle_spmv(threads):
    A = random_lengths_csr(3000, 2500, 50, 31, empty_frac=0.1)
    x = uniform_f32(32, A.n_cols)
    yc = ref_c.spmv_f64(A.row_ptr, A.col, A.val, x, threads)
    yn = spmv.spmv(A.row_ptr, A.col, A.val, x)
    assert np.array_equal(yc, yn)        # same order, same fp64 ops


@pytest.mark.parametrize("threads", [1, 3])
def test_c_oracle_gemm(threads):
    A, B, C0 = sgemm_inputs(33, 21, 17, 41, 42, 43)
    Cc = ref_c.gemm_f64(A, B, C0, 1.5, -0.5, threads)
    assert np.allclose(Cc, triple_loop(A, B, C0, 1.5, -0.5), rtol=1e-13, atol=1e-13)
