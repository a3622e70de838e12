"""Format preparation oracle: CSR -> ELL, CSR -> block-local JDS (SURVEY §8a a-1,
§8c c-3/c-4).  TEST INFRASTRUCTURE ONLY.

The paper lists "input format transformation [4]" among the optimisations
DySel selects between and notes it "may require duplication of inputs"
(§2.3); spmv-jds is Parboil's JDS kernel (P:L1128,
P:L1424-1426 §4.3).  Layouts (bit-exact contract with the CUDA path, see
DESIGN.md §Data layout):

ELL  (Bell & Garland [4]): n_pad = ceil(n/256)*256, W = max row
     length; slot (k, i) at k*n_pad + i holds the k-th CSR entry of row i, else
     col = -1, val = 0.

Block-local JDS (reading A-14): per 256-row block b, order = stable argsort of
     -len over the block's rows; perm[b*256+p] = b*256 + order[p];
     W_b = len(order[0]); jd_ptr_b[0] = 0, jd_ptr_b[k+1] = jd_ptr_b[k] +
     #{p : len(order[p]) > k}; entry (p, k) sits at blk_off[b] + jd_ptr_b[k] + p
     where blk_off[b] = row_ptr[b*256].  jd_ptr of all blocks is concatenated;
     block b's W_b+1 entries start at jd_off[b] = sum_{b'<b} (W_b'+1).

Global-sort JDS (Parboil spmv-jds as the paper profiles it, P:L1424-1426,
P:L1454-1461; SURVEY §8f f-2 "global-sort JDS", a standalone pool since its
units are permuted rows): perm = stable argsort of -len over ALL rows
(position p holds row perm[p]); W = len(perm[0]); jd_ptr[0] = 0, jd_ptr[k+1]
= jd_ptr[k] + #{p : len(perm[p]) > k}; entry (p, k) sits at jd_ptr[k] + p and
holds the k-th CSR entry of row perm[p].

Pinned by tests/test_oracle_spmv.py / tests/test_oracle_f2.py: hand-computed
fixtures, CSR round trips (bit-exact), invariants, brute force.
"""
from __future__ import annotations

import numpy as np

UNIT_ROWS = 256


def csr_to_ell(row_ptr, col, val, unit=UNIT_ROWS):
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    W = int(lens.max()) if n else 0
    n_pad = -(-n // unit) * unit
    ell_col = np.full(W * n_pad, -1, np.int32)
    ell_val = np.zeros(W * n_pad, np.float32)
    for i in range(n):                      # plain loop over rows and slots
        for k in range(int(lens[i])):
            ell_col[k * n_pad + i] = col[rp[i] + k]
            ell_val[k * n_pad + i] = val[rp[i] + k]
    return W, n_pad, ell_col, ell_val


def csr_to_ell_fast(row_ptr, col, val, unit=UNIT_ROWS):
    """Vectorised form of csr_to_ell (same definition), for large inputs."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    W = int(lens.max()) if n else 0
    n_pad = -(-n // unit) * unit
    ell_col = np.full(W * n_pad, -1, np.int32)
    ell_val = np.zeros(W * n_pad, np.float32)
    rows = np.repeat(np.arange(n), lens)
    k = np.arange(rp[-1]) - np.repeat(rp[:-1], lens)
    ell_col[k * n_pad + rows] = col
    ell_val[k * n_pad + rows] = val
    return W, n_pad, ell_col, ell_val


def ell_to_csr(W, n_pad, ell_col, ell_val, n):
    row_ptr = [0]
    cols, vals = [], []
    for i in range(n):
        for k in range(W):
            c = ell_col[k * n_pad + i]
            if c < 0:
                break
            cols.append(c)
            vals.append(ell_val[k * n_pad + i])
        row_ptr.append(len(cols))
    return (np.array(row_ptr, np.int32), np.array(cols, np.int32),
            np.array(vals, np.float32))


def csr_to_block_jds(row_ptr, col, val, unit=UNIT_ROWS):
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    nb = -(-n // unit)
    perm = np.empty(n, np.int32)
    blk_off = np.zeros(nb + 1, np.int64)
    jd_off = np.zeros(nb + 1, np.int64)
    jd_ptr_parts = []
    jds_col = np.empty(rp[-1], np.int32)
    jds_val = np.empty(rp[-1], np.float32)
    for b in range(nb):
        r0, r1 = b * unit, min(n, (b + 1) * unit)
        order = np.argsort(-lens[r0:r1], kind="stable")   # ties: lower row first
        perm[r0:r1] = r0 + order
        blk_off[b] = rp[r0]
        W_b = int(lens[r0 + order[0]])
        jp = np.zeros(W_b + 1, np.int64)
        for k in range(W_b):
            jp[k + 1] = jp[k] + int((lens[r0 + order] > k).sum())
        jd_ptr_parts.append(jp)
        jd_off[b + 1] = jd_off[b] + W_b + 1
        for p, o in enumerate(order):
            g = r0 + o
            for k in range(int(lens[g])):
                jds_col[blk_off[b] + jp[k] + p] = col[rp[g] + k]
                jds_val[blk_off[b] + jp[k] + p] = val[rp[g] + k]
    blk_off[nb] = rp[-1]
    jd_ptr = (np.concatenate(jd_ptr_parts) if jd_ptr_parts else np.zeros(0)).astype(np.int32)
    return dict(perm=perm, blk_off=blk_off, jd_off=jd_off, jd_ptr=jd_ptr,
                jds_col=jds_col, jds_val=jds_val)


def csr_to_block_jds_fast(row_ptr, col, val, unit=UNIT_ROWS):
    """Vectorised form of csr_to_block_jds (same definition), for large inputs."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    nb = -(-n // unit)
    blk = np.arange(n) // unit
    # stable sort by (block asc, len desc, row asc)
    order = np.lexsort((np.arange(n), -lens, blk))
    perm = order.astype(np.int32)
    p_of_row = np.empty(n, np.int64)
    p_of_row[order] = np.arange(n) - blk[order] * unit
    W = np.zeros(nb, np.int64)
    np.maximum.at(W, blk, lens)
    jd_off = np.zeros(nb + 1, np.int64)
    np.cumsum(W + 1, out=jd_off[1:])
    # count_b[k] = #{rows in b with len > k}; via per-block histogram of lens
    jd_ptr = np.zeros(int(jd_off[-1]), np.int64)
    # histogram of (block, len)
    hist_idx = jd_off[blk] + lens          # position len within block's W+1 slots
    cnt = np.zeros(int(jd_off[-1]), np.int64)
    np.add.at(cnt, hist_idx, 1)
    # rows with len > k = total_rows_b - #{len <= k}
    for b in range(nb):
        s, e = jd_off[b], jd_off[b + 1]
        nrows_b = min(n, (b + 1) * unit) - b * unit
        le = np.cumsum(cnt[s:e])            # #{len <= k} for k = 0..W_b
        gt = nrows_b - le[:-1]              # #{len > k} for k = 0..W_b-1
        jd_ptr[s + 1:e] = np.cumsum(gt)
    blk_off = np.zeros(nb + 1, np.int64)
    blk_off[:nb] = rp[np.arange(nb) * unit]
    blk_off[nb] = rp[-1]
    rows = np.repeat(np.arange(n), lens)
    k = np.arange(rp[-1]) - np.repeat(rp[:-1], lens)
    b_e = blk[rows]
    dest = blk_off[b_e] + jd_ptr[jd_off[b_e] + k] + p_of_row[rows]
    jds_col = np.empty(rp[-1], np.int32)
    jds_val = np.empty(rp[-1], np.float32)
    jds_col[dest] = col
    jds_val[dest] = val
    return dict(perm=perm, blk_off=blk_off, jd_off=jd_off, jd_ptr=jd_ptr.astype(np.int32),
                jds_col=jds_col, jds_val=jds_val)


def block_jds_to_csr(j, n, unit=UNIT_ROWS):
    """Inverse of csr_to_block_jds (c-4 round-trip pin)."""
    lens = np.zeros(n, np.int64)
    nb = -(-n // unit)
    rows_cols = [[] for _ in range(n)]
    rows_vals = [[] for _ in range(n)]
    for b in range(nb):
        r0, r1 = b * unit, min(n, (b + 1) * unit)
        jp = j["jd_ptr"][j["jd_off"][b]:j["jd_off"][b + 1]]
        W_b = len(jp) - 1
        for p in range(r1 - r0):
            g = int(j["perm"][r0 + p])
            for k in range(W_b):
                if p >= jp[k + 1] - jp[k]:
                    break
                idx = j["blk_off"][b] + jp[k] + p
                rows_cols[g].append(j["jds_col"][idx])
                rows_vals[g].append(j["jds_val"][idx])
    for g in range(n):
        lens[g] = len(rows_cols[g])
    row_ptr = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    col = np.array([c for r in rows_cols for c in r], np.int32)
    val = np.array([v for r in rows_vals for v in r], np.float32)
    return row_ptr.astype(np.int32), col, val


def ell_applicable(row_ptr, cap=4.0, unit=UNIT_ROWS) -> bool:
    """Reading A-15: ELL is dropped when W * n > cap * nnz."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    nnz = int(rp[-1])
    if n == 0:
        return True
    W = int(np.diff(rp).max())
    return W * n <= cap * max(nnz, 1)


def uniform_rows(row_ptr) -> bool:
    """Reading A-13: uniform workload <=> max row length <= 2 * mean."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    if n == 0 or rp[-1] == 0:
        return True
    lens = np.diff(rp)
    return int(lens.max()) * n <= 2 * int(rp[-1])


def csr_to_global_jds(row_ptr, col, val):
    """Global-sort JDS (definition in the module docstring), plain loops."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    perm = np.array(sorted(range(n), key=lambda r: (-int(lens[r]), r)), np.int64)   # stable by row id
    W = int(lens[perm[0]]) if n else 0
    jd_ptr = np.zeros(W + 1, np.int64)
    for k in range(W):
        jd_ptr[k + 1] = jd_ptr[k] + int(np.sum(lens[perm] > k))
    nnz = int(rp[-1])
    jc = np.zeros(nnz, np.int32)
    jv = np.zeros(nnz, np.float32)
    for p in range(n):
        r = perm[p]
        for k in range(int(lens[r])):
            jc[jd_ptr[k] + p] = col[rp[r] + k]
            jv[jd_ptr[k] + p] = val[rp[r] + k]
    return {"perm": perm.astype(np.int32), "len": lens[perm].astype(np.int32), "jd_ptr": jd_ptr.astype(np.int32),
            "col": jc, "val": jv, "W": W}


def csr_to_global_jds_fast(row_ptr, col, val):
    """Vectorised form of csr_to_global_jds (same definition), for large inputs."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    lens = np.diff(rp)
    perm = np.argsort(-lens, kind="stable")
    sl = lens[perm]
    W = int(sl[0]) if n else 0
    # #{p : len_p > k} for k < W: rows sorted descending -> searchsorted on -sl
    cnt = np.searchsorted(-sl, -np.arange(W), side="left") if W else np.zeros(0, np.int64)
    jd_ptr = np.zeros(W + 1, np.int64)
    np.cumsum(cnt, out=jd_ptr[1:])
    nnz = int(rp[-1])
    rows = np.repeat(np.arange(n), sl)                 # permuted position of each entry (position-major)
    k = np.arange(nnz) - np.repeat(np.concatenate([[0], np.cumsum(sl)[:-1]]) if n else np.zeros(0, np.int64), sl)
    src = rp[perm[rows]] + k
    dst = jd_ptr[k] + rows
    jc = np.zeros(nnz, np.int32)
    jv = np.zeros(nnz, np.float32)
    jc[dst] = np.asarray(col)[src]
    jv[dst] = np.asarray(val)[src]
    return {"perm": perm.astype(np.int32), "len": sl.astype(np.int32), "jd_ptr": jd_ptr.astype(np.int32),
            "col": jc, "val": jv, "W": W}


def global_jds_to_csr(j, n):
    """Inverse of csr_to_global_jds (round-trip pin)."""
    perm, lens, jd_ptr = j["perm"], j["len"], np.asarray(j["jd_ptr"], np.int64)
    row_len = np.zeros(n, np.int64)
    row_len[perm] = lens
    rp = np.zeros(n + 1, np.int64)
    np.cumsum(row_len, out=rp[1:])
    col = np.zeros(int(rp[-1]), np.int32)
    val = np.zeros(int(rp[-1]), np.float32)
    for p in range(n):
        r = int(perm[p])
        for k in range(int(lens[p])):
            col[rp[r] + k] = j["col"][jd_ptr[k] + p]
            val[rp[r] + k] = j["val"][jd_ptr[k] + p]
    return rp, col, val


def unit_x_windows(row_ptr, col, unit=UNIT_ROWS):
    """Per 256-row unit: (min col, max col) over its entries, (0, -1) when the
    unit has none — the x window the smem-staged placement variant copies
    (integer, bit-exact contract)."""
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    nu = (n + unit - 1) // unit
    out = np.zeros((nu, 2), np.int32)
    c = np.asarray(col, np.int64)
    for u in range(nu):
        a, b = rp[u * unit], rp[min((u + 1) * unit, n)]
        out[u] = (int(c[a:b].min()), int(c[a:b].max())) if b > a else (0, -1)
    return out
