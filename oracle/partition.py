"""Multi-GPU row partition oracle.  TEST INFRASTRUCTURE ONLY.

Contiguous row ranges with equal nnz: r_g = the smallest r with
row_ptr[r] >= g * nnz / G (exact integer comparison row_ptr[r] * G >= g * nnz),
snapped down to a multiple of 256 rows (one SpMV unit), monotone, r_0 = 0,
r_G = n.  The paper is single-GPU; this is the build's own
exchange-free sharding, so the oracle is its plain definition (linear scan).
Pinned by tests/test_oracle_plan.py::test_partition_*.
"""
from __future__ import annotations

import numpy as np


def partition_rows(row_ptr, world):
    rp = np.asarray(row_ptr, np.int64)
    n = rp.shape[0] - 1
    nnz = int(rp[-1])
    bounds = [0]
    for g in range(1, world):
        r = 0
        while r < n and rp[r] * world < g * nnz:     # plain linear scan
            r += 1
        bounds.append(max(bounds[-1], (r // 256) * 256))
    bounds.append(n)
    return bounds
