"""Pins of the f-2 format oracles: global-sort JDS (Parboil
spmv-jds, P:L1424-1426 / P:L1454-1461) and the per-unit x windows of the
smem-staged placement variant."""
import numpy as np

from oracle import formats, spmv
from workloads import CSR, d3_fem, random_lengths_csr, uniform_f32


def small():
    # rows: 0 -> 2 entries, 1 -> 0, 2 -> 3, 3 -> 2, 4 -> 1
    rp = np.array([0, 2, 2, 5, 7, 8], np.int32)
    col = np.array([1, 4, 0, 2, 3, 0, 4, 2], np.int32)
    val = np.array([10, 11, 20, 21, 22, 30, 31, 40], np.float32)
    return rp, col, val


def test_global_jds_hand_example():
    """Stable sort by length desc: rows (2: 3), (0: 2), (3: 2), (4: 1), (1: 0);
    W = 3; jd_ptr = [0, 4, 7, 8] (4 rows have >0 entries, 3 have >1, 1 has >2)."""
    rp, col, val = small()
    j = formats.csr_to_global_jds(rp, col, val)
    assert j["perm"].tolist() == [2, 0, 3, 4, 1]
    assert j["len"].tolist() == [3, 2, 2, 1, 0]
    assert j["jd_ptr"].tolist() == [0, 4, 7, 8]
    # diagonal 0: first entries of rows 2, 0, 3, 4; diagonal 1: rows 2, 0, 3; diagonal 2: row 2
    assert j["val"].tolist() == [20, 10, 30, 40, 21, 11, 31, 22]
    assert j["col"].tolist() == [0, 1, 0, 2, 2, 4, 4, 3]


def test_global_jds_roundtrip_invariants_and_fast():
    for seed in (1, 2, 3):
        A = random_lengths_csr(700, 500, 40, seed, empty_frac=0.15)
        j = formats.csr_to_global_jds(A.row_ptr, A.col, A.val)
        jf = formats.csr_to_global_jds_fast(A.row_ptr, A.col, A.val)
        for k in ("perm", "len", "jd_ptr", "col"):
            assert np.array_equal(j[k], jf[k]), k
        assert np.array_equal(j["val"].view(np.uint32), jf["val"].view(np.uint32))
        assert sorted(j["perm"].tolist()) == list(range(A.n_rows))          # a permutation
        assert np.all(np.diff(j["len"]) <= 0)                              # lengths non-increasing
        inc = np.diff(j["jd_ptr"])
        assert np.all(inc >= 0) and np.all(np.diff(inc) <= 0)              # non-increasing diagonal sizes
        assert j["jd_ptr"][-1] == A.nnz
        rp, c, v = formats.global_jds_to_csr(j, A.n_rows)
        assert np.array_equal(rp, A.row_ptr) and np.array_equal(c, A.col)
        assert np.array_equal(v.view(np.uint32), A.val.view(np.uint32))


def test_global_jds_spmv_brute_force():
    """y[perm[p]] = sum_k val[jd_ptr[k] + p] * x[col[...]] equals the dense product."""
    A = random_lengths_csr(300, 200, 25, 7, empty_frac=0.1)
    x = uniform_f32(8, A.n_cols).astype(np.float64)
    j = formats.csr_to_global_jds(A.row_ptr, A.col, A.val)
    y = np.zeros(A.n_rows)
    for p in range(A.n_rows):
        s = 0.0
        for k in range(int(j["len"][p])):
            e = j["jd_ptr"][k] + p
            s += float(j["val"][e]) * x[j["col"][e]]
        y[j["perm"][p]] = s
    dense = np.zeros((A.n_rows, A.n_cols))
    for r in range(A.n_rows):
        for e in range(A.row_ptr[r], A.row_ptr[r + 1]):
            dense[r, A.col[e]] += A.val[e]
    assert np.allclose(y, dense @ x, rtol=1e-12, atol=1e-12)
    assert np.allclose(y, spmv.spmv(A.row_ptr, A.col, A.val, x), rtol=0, atol=1e-12)


def test_unit_x_windows():
    rp, col, _ = small()
    assert formats.unit_x_windows(rp, col).tolist() == [[0, 4]]
    # banded FEM matrix: a 256-row unit's window spans at most 256 + 2 * radius * (grid + 1) columns
    A = d3_fem(grid=101)
    w = formats.unit_x_windows(A.row_ptr, A.col)
    assert np.all(w[:, 1] - w[:, 0] + 1 <= 256 + 2 * 2 * (101 + 1))
    empty = CSR(300, 300, np.zeros(301, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    assert formats.unit_x_windows(empty.row_ptr, empty.col).tolist() == [[0, -1], [0, -1]]
