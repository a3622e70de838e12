"""Seeded synthetic workloads shaped like the paper's inputs.

Every generator uses ``numpy.random.Generator(PCG64(seed))``; values are drawn in
fp64 and rounded to fp32.  Sparse matrices come back as :class:`CSR` with int32
``row_ptr``/``col`` (sorted, distinct columns per row) and fp32 ``val``.

Paper anchors (PAPER.md line numbers):
  * SHOC spmv-csr inputs: "16k-by-16k random sparse matrix with 1% probability
    of non-zeros ... and a 2M-by-2M diagonal matrix" (L1136-1139, §4.2).
  * Parboil sgemm / spmv-jds shapes (L1286-1294, §4.3) -> BASELINE.json configs.
The D1/D3/D4 recipes are the SURVEY §8d ones (stated again in DESIGN.md §Inputs).

No DySel arithmetic lives here (see package docstring).
"""
from __future__ import annotations

import heapq
from dataclasses import dataclass

import numpy as np

__all__ = [
    "CSR", "rng", "uniform_f32", "d1_bus", "d3_fem", "d4_powerlaw",
    "powerlaw_alpha", "powerlaw_lengths", "d6_random", "d6_diag", "identity",
    "small_int_csr", "small_int_vector", "sgemm_inputs", "small_int_gemm",
    "random_lengths_csr", "csr_from_lengths", "laplacian_2d",
]


@dataclass
class CSR:
    n_rows: int
    n_cols: int
    row_ptr: np.ndarray  # int32 [n_rows + 1]
    col: np.ndarray      # int32 [nnz]
    val: np.ndarray      # float32 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def lengths(self) -> np.ndarray:
        return np.diff(self.row_ptr.astype(np.int64))


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform_f32(seed: int, size, lo=-1.0, hi=1.0) -> np.ndarray:
    """U[lo, hi) drawn in fp64, rounded to fp32."""
    return rng(seed).uniform(lo, hi, size).astype(np.float32)


def _csr_from_pattern(n_rows, n_cols, rows, cols, val_seed) -> CSR:
    order = np.lexsort((cols, rows))
    rows = rows[order]
    cols = cols[order]
    counts = np.bincount(rows, minlength=n_rows)
    row_ptr = np.zeros(n_rows + 1, np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    val = uniform_f32(val_seed, cols.shape[0])
    return CSR(n_rows, n_cols, row_ptr.astype(np.int32), cols.astype(np.int32), val)


# --------------------------------------------------------------------------- D1
def _prufer_tree(n: int, g: np.random.Generator):
    """Uniform random labelled tree on n nodes from a random Prüfer sequence."""
    seq = g.integers(0, n, n - 2)
    degree = np.ones(n, np.int64)
    for s in seq:
        degree[s] += 1
    leaves = [i for i in range(n) if degree[i] == 1]
    heapq.heapify(leaves)
    edges = []
    for s in seq:
        leaf = heapq.heappop(leaves)
        edges.append((leaf, int(s)))
        degree[s] -= 1
        if degree[s] == 1:
            heapq.heappush(leaves, int(s))
    u = heapq.heappop(leaves)
    v = heapq.heappop(leaves)
    edges.append((u, v))
    return edges


def d1_bus(n=1138, extra_edges=321, pattern_seed=1138, val_seed=1139) -> CSR:
    """1138_bus-shaped symmetric pattern.

    diagonal + random spanning tree (n-1 edges) + `extra_edges` distinct
    off-diagonal edges, mirrored => nnz = n + 2*(n-1+extra) = 4,054 at n=1138.
    """
    g = rng(pattern_seed)
    edges = set()
    for a, b in _prufer_tree(n, g):
        edges.add((min(a, b), max(a, b)))
    while len(edges) < (n - 1) + extra_edges:
        a, b = g.integers(0, n, 2)
        if a != b:
            edges.add((int(min(a, b)), int(max(a, b))))
    e = np.array(sorted(edges), np.int64)
    rows = np.concatenate([np.arange(n), e[:, 0], e[:, 1]])
    cols = np.concatenate([np.arange(n), e[:, 1], e[:, 0]])
    return _csr_from_pattern(n, n, rows, cols, val_seed)


# --------------------------------------------------------------------------- D3
def d3_fem(grid=383, radius=2, val_seed=383) -> CSR:
    """Dubcova3-shaped FEM matrix: grid x grid nodes, (2r+1)^2 box stencil.

    grid=383, r=2 => n = 146,689, nnz = 3,644,281.
    """
    n = grid * grid
    i, j = np.divmod(np.arange(n, dtype=np.int64), grid)
    rows_l, cols_l = [], []
    for di in range(-radius, radius + 1):          # ascending column order
        for dj in range(-radius, radius + 1):
            ii, jj = i + di, j + dj
            ok = (ii >= 0) & (ii < grid) & (jj >= 0) & (jj < grid)
            rows_l.append(np.nonzero(ok)[0])
            cols_l.append((ii * grid + jj)[ok])
    rows = np.concatenate(rows_l)
    cols = np.concatenate(cols_l)
    return _csr_from_pattern(n, n, rows, cols, val_seed)


def laplacian_2d(grid: int) -> CSR:
    """5-point Dirichlet Laplacian on a grid x grid mesh (input for the
    iterative driver's parity tests): 4 on the diagonal, -1 to
    the four neighbours, row-major node order, ascending columns."""
    n = grid * grid
    i, j = np.divmod(np.arange(n, dtype=np.int64), grid)
    rows_l, cols_l, vals_l = [], [], []
    for di, dj, v in ((-1, 0, -1.0), (0, -1, -1.0), (0, 0, 4.0), (0, 1, -1.0), (1, 0, -1.0)):
        ii, jj = i + di, j + dj
        ok = (ii >= 0) & (ii < grid) & (jj >= 0) & (jj < grid)
        rows_l.append(np.nonzero(ok)[0])
        cols_l.append((ii * grid + jj)[ok])
        vals_l.append(np.full(int(ok.sum()), v))
    rows = np.concatenate(rows_l)
    cols = np.concatenate(cols_l)
    vals = np.concatenate(vals_l)
    order = np.lexsort((cols, rows))
    rows, cols, vals = rows[order], cols[order], vals[order]
    row_ptr = np.zeros(n + 1, np.int64)
    np.add.at(row_ptr, rows + 1, 1)
    np.cumsum(row_ptr, out=row_ptr)
    return CSR(n, n, row_ptr.astype(np.int32), cols.astype(np.int32), vals.astype(np.float32))


# --------------------------------------------------------------------------- D4
def powerlaw_alpha(mean=20.0, lmax=16384, lo=1.0001, hi=4.0, iters=200) -> float:
    """alpha such that p(L) ∝ L^-alpha on [1, lmax] has the given mean (bisection)."""
    L = np.arange(1, lmax + 1, dtype=np.float64)

    def m(a):
        w = L ** (-a)
        return float((L * w).sum() / w.sum())

    for _ in range(iters):
        mid = 0.5 * (lo + hi)
        if m(mid) > mean:
            lo = mid
        else:
            hi = mid
    return 0.5 * (lo + hi)


def powerlaw_lengths(n, seed, mean=20.0, lmax=16384) -> np.ndarray:
    a = powerlaw_alpha(mean, lmax)
    L = np.arange(1, lmax + 1, dtype=np.float64)
    w = L ** (-a)
    cdf = np.cumsum(w / w.sum())
    cdf[-1] = 1.0
    u = rng(seed).random(n)
    return (np.searchsorted(cdf, u, side="right") + 1).astype(np.int64)


def csr_from_lengths(lengths, n_cols, col_seed, val_seed, chunk=1 << 20) -> CSR:
    """Sorted distinct uniform columns per row via exponential spacings.

    For a row of length L: E_0..E_L ~ Exp(1), u_k = (E_0+..+E_k)/(E_0+..+E_L) are
    the order statistics of L uniforms; col_k = floor(u_k*(n_cols-L+1)) + k is
    strictly increasing in [0, n_cols).  Vectorised in row chunks, no sort.
    """
    lengths = np.asarray(lengths, np.int64)
    n = lengths.shape[0]
    if n and lengths.max() > n_cols:
        raise ValueError("row longer than n_cols")
    row_ptr = np.zeros(n + 1, np.int64)
    np.cumsum(lengths, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    col = np.empty(nnz, np.int32)
    g = rng(col_seed)
    for r0 in range(0, n, chunk):
        r1 = min(n, r0 + chunk)
        Ls = lengths[r0:r1]
        m = int(Ls.sum())
        if m == 0:
            continue
        E = g.standard_exponential(m + (r1 - r0))
        cs = np.cumsum(E)
        # segment of row r: L+1 spacings; starts at off2[r]
        off2 = np.zeros(r1 - r0 + 1, np.int64)
        np.cumsum(Ls + 1, out=off2[1:])
        base = np.where(off2[:-1] > 0, cs[np.maximum(off2[:-1] - 1, 0)], 0.0)
        total = cs[off2[1:] - 1] - base
        rowid = np.repeat(np.arange(r1 - r0), Ls)
        k = np.arange(m) - np.repeat(row_ptr[r0:r1] - row_ptr[r0], Ls)
        pos = off2[:-1][rowid] + k
        u = (cs[pos] - base[rowid]) / total[rowid]
        span = (n_cols - Ls + 1)[rowid]
        c = np.floor(u * span).astype(np.int64)
        c = np.minimum(c, span - 1) + k
        col[row_ptr[r0]:row_ptr[r1]] = c.astype(np.int32)
    val = uniform_f32(val_seed, nnz)
    return CSR(n, n_cols, row_ptr.astype(np.int32) if nnz < 2**31 else row_ptr,
               col, val)


def d4_powerlaw(n=10_000_000, len_seed=10007, col_seed=10008, val_seed=10009,
                mean=20.0, lmax=16384) -> CSR:
    """Power-law rows: p(L) ∝ L^-alpha, L in [1, lmax], mean 20.

    Row order is i.i.d. (already a uniform shuffle); columns uniform distinct
    sorted in [0, n).  `n` and `lmax` may be reduced for small parity cases.
    """
    lmax = min(lmax, n)
    L = powerlaw_lengths(n, len_seed, mean, lmax)
    return csr_from_lengths(L, n, col_seed, val_seed)


def random_lengths_csr(n_rows, n_cols, max_len, seed, val_seed=None, empty_frac=0.0):
    """Ragged test matrix: uniform lengths in [0, max_len], some forced empty."""
    g = rng(seed)
    L = g.integers(0, max_len + 1, n_rows)
    if empty_frac > 0:
        L[g.random(n_rows) < empty_frac] = 0
    return csr_from_lengths(np.minimum(L, n_cols), n_cols, seed + 1,
                            seed + 2 if val_seed is None else val_seed)


# --------------------------------------------------------------------------- D6
def d6_random(n=16384, p=0.01, seed=16384) -> CSR:
    """SHOC default: each entry nonzero independently with probability p (L1136-1138)."""
    g = rng(seed)
    L = g.binomial(n, p, n).astype(np.int64)
    return csr_from_lengths(L, n, seed + 1, seed + 2)


def d6_diag(n=2 ** 21, seed=2097152) -> CSR:
    """n x n diagonal (identity pattern), val ~ U[-1,1) (L1139)."""
    row_ptr = np.arange(n + 1, dtype=np.int32)
    col = np.arange(n, dtype=np.int32)
    return CSR(n, n, row_ptr, col, uniform_f32(seed, n))


def identity(n) -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int32), np.arange(n, dtype=np.int32),
               np.ones(n, np.float32))


# ------------------------------------------------------------------ integer pins
def small_int_csr(csr: CSR, seed: int) -> CSR:
    """Same pattern, values in {-3..3} (exactly representable; SURVEY c-1 pin)."""
    v = rng(seed).integers(-3, 4, csr.nnz).astype(np.float32)
    return CSR(csr.n_rows, csr.n_cols, csr.row_ptr, csr.col, v)


def small_int_vector(n, seed) -> np.ndarray:
    return rng(seed).integers(-4, 5, n).astype(np.float32)


# ------------------------------------------------------------------------ SGEMM
def sgemm_inputs(M, K, N, seed_a=992, seed_b=993, seed_c=None):
    """Parboil-sgemm-shaped fp32 operands, row-major A[M,K], B[K,N], C0[M,N]."""
    A = uniform_f32(seed_a, (M, K))
    B = uniform_f32(seed_b, (K, N))
    C0 = np.zeros((M, N), np.float32) if seed_c is None else uniform_f32(seed_c, (M, N))
    return A, B, C0


def small_int_gemm(M, K, N, seed):
    g = rng(seed)
    A = g.integers(-4, 5, (M, K)).astype(np.float32)
    B = g.integers(-4, 5, (K, N)).astype(np.float32)
    C0 = g.integers(-4, 5, (M, N)).astype(np.float32)
    return A, B, C0
