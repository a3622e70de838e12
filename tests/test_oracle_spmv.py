"""Pins for oracle/spmv.py and oracle/formats.py (SURVEY c-1, c-3, c-4)."""
import os

import numpy as np
import pytest
import scipy.sparse as sp

from oracle import formats, spmv
from workloads import (CSR, d1_bus, d3_fem, d4_powerlaw, d6_diag, identity,
                       random_lengths_csr, small_int_csr, small_int_vector, uniform_f32)

GOLD = os.path.join(os.path.dirname(__file__), "golden", "small_formats.txt")


def load_golden():
    d = {}
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        k, *v = line.split()
        d[k] = np.array([float(t) for t in v])
    return d


def scipy_ref(A: CSR, x):
    m = sp.csr_matrix((A.val.astype(np.float64), A.col, A.row_ptr), shape=(A.n_rows, A.n_cols))
    return m @ x.astype(np.float64)


def test_golden_small_matrix():
    g = load_golden()
    y = spmv.spmv(g["row_ptr"].astype(np.int32), g["col"].astype(np.int32),
                  g["val"].astype(np.float32), g["x"].astype(np.float32))
    assert np.array_equal(y, g["y"])


@pytest.mark.parametrize("maker", [lambda: d1_bus(), lambda: random_lengths_csr(700, 513, 40, 7, empty_frac=0.1),
                                   lambda: d4_powerlaw(n=5000, lmax=600)])
def test_matches_scipy(maker):
    A = maker()
    x = uniform_f32(5, A.n_cols)
    y = spmv.spmv(A.row_ptr, A.col, A.val, x)
    ref = scipy_ref(A, x)
    assert np.allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_dense_brute_force():
    A = random_lengths_csr(300, 200, 60, 11, empty_frac=0.05)   # non-square: transposition shows
    x = uniform_f32(12, A.n_cols)
    D = np.zeros((A.n_rows, A.n_cols))
    for i in range(A.n_rows):
        for k in range(A.row_ptr[i], A.row_ptr[i + 1]):
            D[i, A.col[k]] += A.val[k]
    assert np.allclose(spmv.spmv(A.row_ptr, A.col, A.val, x), D @ x.astype(np.float64), rtol=1e-13, atol=1e-13)


def test_small_integer_exact():
    A = small_int_csr(d1_bus(), 3)
    x = small_int_vector(A.n_cols, 4)
    y = spmv.spmv(A.row_ptr, A.col, A.val, x)
    ref = scipy_ref(A, x)
    assert np.array_equal(y, ref)              # exact in fp64 (and fp32)
    assert np.array_equal(y, np.rint(y))


def test_identity_and_diagonal_closed_forms():
    n = 1000
    x = uniform_f32(1, n)
    I = identity(n)
    assert np.array_equal(spmv.spmv(I.row_ptr, I.col, I.val, x), x.astype(np.float64))
    D = d6_diag(n=4096)
    x = uniform_f32(2, 4096)
    y = spmv.spmv(D.row_ptr, D.col, D.val, x)
    assert np.array_equal(y, D.val.astype(np.float64) * x.astype(np.float64))


def test_abs_denominator_and_rows():
    A = random_lengths_csr(200, 200, 30, 21, empty_frac=0.2)
    x = uniform_f32(22, 200)
    d = spmv.spmv_abs(A.row_ptr, A.col, A.val, x)
    m = sp.csr_matrix((np.abs(A.val.astype(np.float64)), A.col, A.row_ptr), shape=(200, 200))
    assert np.allclose(d, m @ np.abs(x.astype(np.float64)), rtol=1e-13)
    rows = [0, 5, 17, 199]
    y_s, d_s = spmv.spmv_rows(A.row_ptr, A.col, A.val, x, rows)
    y = spmv.spmv(A.row_ptr, A.col, A.val, x)
    assert np.allclose(y_s, y[rows], rtol=1e-14, atol=0) and np.allclose(d_s, d[rows], rtol=1e-14)


def test_rel_error_semantics():
    assert spmv.rel_error([0.0, 1.0], np.array([0.0, 1.0]), np.array([0.0, 1.0])) == 0.0
    assert spmv.rel_error([np.nan], np.array([1.0]), np.array([1.0])) == np.inf
    assert spmv.rel_error([1.5], np.array([1.0]), np.array([2.0])) == 0.25


# ----------------------------------------------------------------- formats
def test_golden_formats():
    g = load_golden()
    rp, c, v = g["row_ptr"].astype(np.int32), g["col"].astype(np.int32), g["val"].astype(np.float32)
    W, npad, ec, ev = formats.csr_to_ell(rp, c, v, unit=4)
    assert W == g["ell_W"][0] and npad == g["ell_npad"][0]
    assert np.array_equal(ec, g["ell_col"]) and np.array_equal(ev, g["ell_val"])
    j = formats.csr_to_block_jds(rp, c, v, unit=4)
    assert np.array_equal(j["perm"], g["jds_perm"])
    assert np.array_equal(j["blk_off"], g["jds_blk_off"])
    assert np.array_equal(j["jd_off"], g["jds_jd_off"])
    assert np.array_equal(j["jd_ptr"], g["jds_jd_ptr"])
    assert np.array_equal(j["jds_col"], g["jds_col"]) and np.array_equal(j["jds_val"], g["jds_val"])


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_ell_roundtrip_and_fast(seed):
    A = random_lengths_csr(777, 300, 25, seed, empty_frac=0.1)
    W, npad, ec, ev = formats.csr_to_ell(A.row_ptr, A.col, A.val)
    assert npad % 256 == 0 and npad >= A.n_rows
    assert int((ec >= 0).sum()) == A.nnz
    rp, c, v = formats.ell_to_csr(W, npad, ec, ev, A.n_rows)
    assert np.array_equal(rp, A.row_ptr) and np.array_equal(c, A.col) and np.array_equal(v, A.val)
    W2, npad2, ec2, ev2 = formats.csr_to_ell_fast(A.row_ptr, A.col, A.val)
    assert (W2, npad2) == (W, npad) and np.array_equal(ec, ec2) and np.array_equal(ev, ev2)


@pytest.mark.parametrize("seed", [4, 5])
def test_jds_invariants_roundtrip_fast(seed):
    A = random_lengths_csr(900, 400, 30, seed, empty_frac=0.15)
    j = formats.csr_to_block_jds(A.row_ptr, A.col, A.val)
    n = A.n_rows
    lens = A.lengths()
    nb = -(-n // 256)
    for b in range(nb):
        r0, r1 = b * 256, min(n, (b + 1) * 256)
        p = j["perm"][r0:r1]
        assert sorted(p.tolist()) == list(range(r0, r1))              # bijection in block
        L = lens[p]
        assert np.all(np.diff(L) <= 0)                                # non-increasing
        jp = j["jd_ptr"][j["jd_off"][b]:j["jd_off"][b + 1]]
        inc = np.diff(jp)
        assert np.all(inc >= 0) and np.all(np.diff(inc) <= 0)
        assert jp[-1] == j["blk_off"][b + 1] - j["blk_off"][b]
    assert j["blk_off"][-1] == A.nnz
    rp, c, v = formats.block_jds_to_csr(j, n)
    assert np.array_equal(rp, A.row_ptr) and np.array_equal(c, A.col) and np.array_equal(v, A.val)
    f = formats.csr_to_block_jds_fast(A.row_ptr, A.col, A.val)
    for k in j:
        assert np.array_equal(np.asarray(j[k]), np.asarray(f[k])), k


def test_applicability_and_uniformity_readings():
    assert formats.uniform_rows(d3_fem(grid=40).row_ptr)
    assert formats.ell_applicable(d3_fem(grid=40).row_ptr)
    P = d4_powerlaw(n=20000, lmax=4096)
    assert not formats.uniform_rows(P.row_ptr)
    assert not formats.ell_applicable(P.row_ptr)
    assert formats.ell_applicable(d1_bus().row_ptr)


def test_spmtv_dense_brute_force_and_scipy():
    """y0 + A^T x: explicit-loop dense transpose and scipy's A.T @ x (non-square)."""
    A = random_lengths_csr(300, 200, 60, 13, empty_frac=0.05)
    x = uniform_f32(14, A.n_rows)
    y0 = uniform_f32(15, A.n_cols)
    D = np.zeros((A.n_cols, A.n_rows))
    for i in range(A.n_rows):
        for k in range(A.row_ptr[i], A.row_ptr[i + 1]):
            D[A.col[k], i] += A.val[k]   # D = A^T
    y = spmv.spmtv(A.row_ptr, A.col, A.val, x, y0)
    assert y.shape == (A.n_cols,)
    assert np.allclose(y, y0.astype(np.float64) + D @ x.astype(np.float64), rtol=1e-13, atol=1e-13)
    m = sp.csr_matrix((A.val.astype(np.float64), A.col, A.row_ptr), shape=(A.n_rows, A.n_cols))
    assert np.allclose(y, y0 + m.T @ x.astype(np.float64), rtol=1e-12, atol=1e-12)


def test_spmtv_duality_and_small_int():
    """u.(A^T x) = (A u).x against the (separately pinned) spmv oracle; small
    integers are exact; all-zero x leaves y0 unchanged."""
    A = d4_powerlaw(n=3000, lmax=400)
    x = uniform_f32(21, A.n_rows)
    u = uniform_f32(22, A.n_cols).astype(np.float64)
    z = np.zeros(A.n_cols)
    lhs = u @ spmv.spmtv(A.row_ptr, A.col, A.val, x, z)
    rhs = spmv.spmv(A.row_ptr, A.col, A.val, u) @ x.astype(np.float64)
    assert abs(lhs - rhs) <= 1e-10 * max(1.0, abs(rhs))
    B = small_int_csr(d1_bus(), 3)
    xi = small_int_vector(B.n_rows, 4)
    yi = spmv.spmtv(B.row_ptr, B.col, B.val, xi, np.zeros(B.n_cols))
    assert np.array_equal(yi, np.round(yi))
    y0 = uniform_f32(23, B.n_cols)
    assert np.array_equal(spmv.spmtv(B.row_ptr, B.col, B.val, np.zeros(B.n_rows, np.float32), y0),
                          y0.astype(np.float64))
    d = spmv.spmtv_abs(B.row_ptr, B.col, B.val, xi, y0)
    assert np.all(d >= np.abs(spmv.spmtv(B.row_ptr, B.col, B.val, xi, y0)) - 1e-12)
