"""Pins of the oracle's error DENOMINATORS and error functions (SURVEY §8c
c-1 / c-2, §8f f-1 / f-4).  Each denominator sets the pass line of every parity
test in its family, so each is checked here against a pure-Python loop written
from its definition (not a re-call of the oracle's vectorised formula), on
inputs chosen so that a dropped term, a wrong sign or a transposed operand
fails:

  * spmv_abs   d_i  = sum_k |val_k| |x[col_k]|                      (c-1)
  * spmtv_abs  d_j  = |y0_j| + sum_{(i,j)} |val_ij| |x_i|            (f-1, y0 + A^T x)
  * sgemm_abs  d_ij = |alpha| sum_k |A_ik| |B_kj| + |beta| |C0_ij|   (c-2)
  * stencil_abs d   = |c1| sum_6 |nb| + |c0| |centre| (interior), |in| (boundary)  (A-37)
  * rel_error  max |out - ref| / d  with the 0/0 convention of each module.
"""
import numpy as np

from oracle import sgemm as osg
from oracle import spmv as osp
from oracle import stencil as ost
from workloads import random_lengths_csr, sgemm_inputs, uniform_f32


# ------------------------------------------------------------------ SpMV
def test_spmv_abs_loop_with_sign_cancellation():
    # row 0: +2*3 + (-2)*3 = 0 but d = 12 (a dropped abs() on val gives 0)
    # row 1: val > 0, x < 0 (a dropped abs() on x gives a negative d)
    rp = np.array([0, 2, 3, 3], np.int32)
    col = np.array([0, 1, 2], np.int32)
    val = np.array([2.0, -2.0, 5.0], np.float32)
    x = np.array([3.0, -3.0, -0.5], np.float32)
    d = osp.spmv_abs(rp, col, val, x)
    assert d.tolist() == [12.0, 2.5, 0.0]
    A = random_lengths_csr(300, 180, 40, 3, empty_frac=0.1)
    xr = uniform_f32(4, A.n_cols)
    dl = np.zeros(A.n_rows)
    for i in range(A.n_rows):
        s = 0.0
        for k in range(int(A.row_ptr[i]), int(A.row_ptr[i + 1])):
            s += abs(float(A.val[k])) * abs(float(xr[int(A.col[k])]))
        dl[i] = s
    assert np.allclose(osp.spmv_abs(A.row_ptr, A.col, A.val, xr), dl, rtol=1e-14, atol=0)


# ----------------------------------------------------------------- SpMTV
def _spmtv_abs_loop(rp, col, val, x, y0):
    d = [abs(float(v)) for v in y0]
    for i in range(len(rp) - 1):
        for k in range(int(rp[i]), int(rp[i + 1])):
            d[int(col[k])] += abs(float(val[k])) * abs(float(x[i]))
    return np.array(d)


def test_spmtv_abs_y0_dominated_and_empty_column():
    # 3 x 4 matrix; column 3 is empty, so its denominator is |y0_3| alone
    # (a missing |y0| term gives 0 there); column 0 mixes signs.
    rp = np.array([0, 2, 3, 4], np.int32)
    col = np.array([0, 2, 0, 1], np.int32)
    val = np.array([1.0, -2.0, -4.0, 0.5], np.float32)
    x = np.array([-1.0, 0.25, 2.0], np.float32)
    y0 = np.array([-8.0, 0.0, 3.0, -7.5], np.float32)
    d = osp.spmtv_abs(rp, col, val, x, y0)
    # col 0: |-8| + |1||-1| + |-4||0.25| = 10 ; col 1: 0 + |0.5||2| = 1
    # col 2: |3| + |-2||-1| = 5 ; col 3: |-7.5| = 7.5
    assert d.tolist() == [10.0, 1.0, 5.0, 7.5]
    assert np.array_equal(d, _spmtv_abs_loop(rp, col, val, x, y0))
    # the value itself: y0 + A^T x
    y = osp.spmtv(rp, col, val, x, y0)
    assert y.tolist() == [-8.0 - 1.0 - 1.0, 1.0, 3.0 + 2.0, -7.5]


def test_spmtv_abs_random_loop():
    A = random_lengths_csr(120, 90, 30, 8, empty_frac=0.2)
    x = uniform_f32(9, A.n_rows)
    y0 = uniform_f32(10, A.n_cols) * 4
    assert np.allclose(osp.spmtv_abs(A.row_ptr, A.col, A.val, x, y0),
                       _spmtv_abs_loop(A.row_ptr, A.col, A.val, x, y0), rtol=1e-14, atol=0)


# ----------------------------------------------------------------- SGEMM
def _sgemm_abs_loop(A, B, C0, alpha, beta):
    M, K = A.shape
    N = B.shape[1]
    d = np.zeros((M, N))
    for i in range(M):
        for j in range(N):
            s = 0.0
            for k in range(K):
                s += abs(float(A[i, k])) * abs(float(B[k, j]))
            d[i, j] = abs(alpha) * s + abs(beta) * abs(float(C0[i, j]))
    return d


def test_sgemm_abs_loop_non_square_negative_scalars():
    # M != K != N (a transposed operand cannot broadcast), alpha < 0 and
    # beta < 0 (a dropped abs() on a scalar makes d negative)
    A, B, C0 = sgemm_inputs(7, 5, 3, 21, 22, 23)
    for alpha, beta in ((-1.5, -0.5), (2.0, 0.0), (0.0, -3.0)):
        d = osg.sgemm_abs(A, B, C0, alpha, beta)
        assert d.shape == (7, 3)
        assert np.allclose(d, _sgemm_abs_loop(A, B, C0, alpha, beta), rtol=1e-14, atol=0)
        assert np.all(d >= np.abs(osg.sgemm(A, B, C0, alpha, beta)) - 1e-12)


def test_sgemm_abs_hand_example():
    # A = [1 -2]  B = [ 3  0]   |A||B| = [1 2][3 0] = [3+4  0+2]
    #     [0  4]      [-2  1]            [0 4][2 1]   [0+8  0+4]
    # alpha = -1, beta = -2: + |beta||C0| = [2 2; 1 0]
    A = np.array([[1, -2], [0, 4]], np.float32)
    B = np.array([[3, 0], [-2, 1]], np.float32)
    C0 = np.array([[1, -1], [0.5, 0]], np.float32)
    d = osg.sgemm_abs(A, B, C0, -1.0, -2.0)
    assert d.tolist() == [[7.0 + 2.0, 2.0 + 2.0], [8.0 + 1.0, 4.0 + 0.0]]
    C = osg.sgemm(A, B, C0, -1.0, -2.0)
    # A B = [[7, -2], [-8, 4]]
    assert C.tolist() == [[-7.0 - 2.0, 2.0 + 2.0], [8.0 - 1.0, -4.0 - 0.0]]


# --------------------------------------------------------------- stencil
NBRS = ((-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1))


def _stencil_abs_loop(a, c0, c1):
    nz, ny, nx = a.shape
    d = np.abs(np.array(a, np.float64))
    for z in range(1, nz - 1):
        for y in range(1, ny - 1):
            for x in range(1, nx - 1):
                s = 0.0
                for dz, dy, dx in NBRS:
                    s += abs(float(a[z + dz, y + dy, x + dx]))
                d[z, y, x] = abs(c1) * s + abs(c0) * abs(float(a[z, y, x]))
    return d


def test_stencil_abs_loop_signs_and_boundary():
    g = np.random.default_rng(11)
    a = g.uniform(-1, 1, (4, 5, 6))
    # both coefficient signs: d must not depend on them
    for c0, c1 in ((0.8125, 0.15625), (-0.8125, 0.15625), (0.5, -1.25)):
        d = ost.stencil_abs(a, c0, c1)
        assert np.allclose(d, _stencil_abs_loop(a, c0, c1), rtol=1e-14, atol=0)
        # boundary denominator is |in| (out = in there)
        assert np.array_equal(d[0], np.abs(a[0])) and np.array_equal(d[:, :, -1], np.abs(a[:, :, -1]))
        assert np.all(d >= np.abs(ost.stencil(a, c0, c1)) - 1e-12)


def test_stencil_abs_closed_form_constant_field():
    # constant field v < 0: interior d = (6|c1| + |c0|)|v| (a dropped |c0| term
    # or a sign slip in it changes this), boundary d = |v|
    a = np.full((3, 4, 5), -2.0)
    d = ost.stencil_abs(a, -0.75, 0.5)
    assert np.all(d[1:-1, 1:-1, 1:-1] == (6 * 0.5 + 0.75) * 2.0)
    assert d[0, 0, 0] == 2.0 and d[2, 3, 4] == 2.0


def test_stencil_rel_error_semantics():
    ref = np.array([1.0, -2.0, 0.0, 5.0])
    den = np.array([2.0, 4.0, 0.0, 10.0])
    out = np.array([1.5, -2.0, 0.0, 4.0])
    # |0.5|/2, 0, 0/0 := 0 (den 0 counts as 1), |1|/10
    assert ost.rel_error(out, ref, den) == 0.25
    assert ost.rel_error(np.array([0.0, 0.0]), np.zeros(2), np.zeros(2)) == 0.0
    # den == 0 but out != ref: the absolute difference counts (not hidden)
    assert ost.rel_error(np.array([3e-3]), np.zeros(1), np.zeros(1)) == 3e-3
    assert ost.rel_error(np.zeros(0), np.zeros(0), np.zeros(0)) == 0.0
    assert ost.rel_error(np.array([np.nan]), np.ones(1), np.ones(1)) == np.inf


def test_tolerances_are_the_stated_ones():
    assert osp.SPMV_TOL == 1e-5 and osg.SGEMM_TOL == 1e-4       # north_star
    # stencil: 8 roundings of relative size 2^-24 bound the fp32 error by 8 * 2^-24 of d
    assert ost.STENCIL_TOL >= 8 * 2.0 ** -24 and ost.STENCIL_TOL <= 1e-5
