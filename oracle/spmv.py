"""fp64 SpMV oracle.  TEST INFRASTRUCTURE ONLY.

y*_i = sum_{k in row i} (double)val_k * (double)x[col_k], accumulated in CSR
order — the plain definition of y = A x for the SHOC spmv-csr kernels the paper
selects between ("spmv with scalar dot products on a CSR format matrix without
padding", §4.2; scalar vs vector versions, §4.4).
DySel changes only *which variant computes each row*, never *what* is computed
(productive profiling, §2.2), so this is the oracle for every variant
and every profiling mode.

Pinned by tests/test_oracle_spmv.py: small-integer exactness, identity /
diagonal closed forms, dense brute force, scipy.sparse; spmtv by dense
brute force (explicit loops), scipy's A.T @ x and the duality u.(A^T x) =
(A u).x against spmv; the denominators spmv_abs / spmtv_abs by
tests/test_oracle_denominators.py (explicit loops, sign cancellation, a
y0-dominated empty column).
"""
from __future__ import annotations

import numpy as np


def _rows_of(row_ptr: np.ndarray) -> np.ndarray:
    rp = np.asarray(row_ptr, np.int64)
    return np.repeat(np.arange(rp.shape[0] - 1), np.diff(rp))


def spmv(row_ptr, col, val, x) -> np.ndarray:
    """y = A x in fp64, per-row sums accumulated in CSR order (np.add.at is
    unbuffered and applies the products in index order)."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    prod = np.asarray(val, np.float64) * np.asarray(x, np.float64)[np.asarray(col, np.int64)]
    y = np.zeros(n, np.float64)
    np.add.at(y, _rows_of(rp), prod)
    return y


def spmv_abs(row_ptr, col, val, x) -> np.ndarray:
    """d_i = sum |val_k| * |x[col_k]| — the error denominator of c-1."""
    return spmv(row_ptr, col, np.abs(np.asarray(val, np.float64)), np.abs(np.asarray(x, np.float64)))


def spmv_rows(row_ptr, col, val, x, rows):
    """(y*, d) for a sample of rows, each computed on its own (full-size parity)."""
    rp = np.asarray(row_ptr, np.int64)
    xs = np.asarray(x, np.float64)
    y = np.empty(len(rows), np.float64)
    d = np.empty(len(rows), np.float64)
    for j, r in enumerate(rows):
        b, e = rp[r], rp[r + 1]
        v = np.asarray(val[b:e], np.float64)
        xv = xs[np.asarray(col[b:e], np.int64)]
        s = 0.0
        a = 0.0
        for p, q in zip(v, xv):   # CSR order, one term at a time
            s += p * q
            a += abs(p) * abs(q)
        y[j] = s
        d[j] = a
    return y, d


def spmtv(row_ptr, col, val, x, y0=None) -> np.ndarray:
    """y = y0 + A^T x in fp64: y_j = y0_j + sum over nonzeros (i, j) of
    val_ij * x_i — the plain definition of the transposed product that the
    atomic scatter pool (dysel_spmtv, the swap-mode case of P:L453-464 §2.2 /
    P:L977-992 §3.3) computes.  Products applied in CSR order (np.add.at)."""
    rp = np.asarray(row_ptr, np.int64)
    c = np.asarray(col, np.int64)
    n_cols = int(c.max()) + 1 if c.size else 0
    prod = np.asarray(val, np.float64) * np.asarray(x, np.float64)[_rows_of(rp)]
    if y0 is not None:
        y = np.array(y0, np.float64)
    else:
        y = np.zeros(n_cols, np.float64)
    np.add.at(y, c, prod)
    return y


def spmtv_abs(row_ptr, col, val, x, y0) -> np.ndarray:
    """d_j = |y0_j| + sum |val_ij| * |x_i| — the error denominator for y0 + A^T x."""
    return spmtv(row_ptr, col, np.abs(np.asarray(val, np.float64)), np.abs(np.asarray(x, np.float64)),
                 np.abs(np.asarray(y0, np.float64)))


def rel_error(y_hat, y_star, denom) -> float:
    """max_i |y_hat_i - y*_i| / d_i with 0/0 := 0 (c-1).  Non-finite values in
    y_hat where y* is finite count as +inf error."""
    y_hat = np.asarray(y_hat, np.float64)
    diff = np.abs(y_hat - y_star)
    denom = np.asarray(denom, np.float64)
    with np.errstate(invalid="ignore", divide="ignore"):
        e = np.where(diff == 0, 0.0, diff / denom)
    e = np.where(np.isnan(e), np.inf, e)
    return float(e.max()) if e.size else 0.0


SPMV_TOL = 1e-5   # north_star: "max relative error 1e-5 of the fp64 oracle for fp32 SpMV"
