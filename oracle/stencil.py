"""fp64 stencil oracle.  TEST INFRASTRUCTURE ONLY
(tests/, __graft_entry__.smoke(), bench.py's CPU leg).

The paper's stencil case (Parboil stencil: "three versions and work assignment
factors relative to the base version are 64x and 128x", §4.3,
optimisations "tiling, coarsening, and data placement using scratchpad",
P:L1298-1305) does not restate the operator; reading A-37 takes the
3-D 7-point Jacobi step, written out here as its plain definition:

    out[z,y,x] = c1 * (in[z-1,y,x] + in[z+1,y,x] + in[z,y-1,x] + in[z,y+1,x]
                       + in[z,y,x-1] + in[z,y,x+1]) - c0 * in[z,y,x]

for interior points, and out = in on the boundary (any coordinate 0 or n-1).
DySel only changes which variant computes each 32x4x1 block of points
(P:L355-363), so this is the oracle for every variant and mode.

Pinned by tests/test_oracle_stencil.py: constant and linear fields (the
6-neighbour sum of a linear field is 6 * its centre value), a pure-Python
triple loop on tiny grids, boundary copy; the denominator stencil_abs and
rel_error by tests/test_oracle_denominators.py (pure-Python loop of
|c1| sum |nb| + |c0| |c|, constant-field closed form, hand-computed errors).
"""
from __future__ import annotations

import numpy as np


def stencil(inp, c0: float, c1: float) -> np.ndarray:
    """One step in fp64; inp is [nz, ny, nx]."""
    a = np.asarray(inp, np.float64)
    out = a.copy()
    if min(a.shape) >= 3:
        nb = (a[:-2, 1:-1, 1:-1] + a[2:, 1:-1, 1:-1] + a[1:-1, :-2, 1:-1] + a[1:-1, 2:, 1:-1]
              + a[1:-1, 1:-1, :-2] + a[1:-1, 1:-1, 2:])
        out[1:-1, 1:-1, 1:-1] = float(c1) * nb - float(c0) * a[1:-1, 1:-1, 1:-1]
    return out


def stencil_abs(inp, c0: float, c1: float) -> np.ndarray:
    """Error denominator: |c1| * sum |neighbours| + |c0| * |centre| (interior), |in| (boundary)."""
    return stencil(np.abs(np.asarray(inp, np.float64)), -abs(float(c0)), abs(float(c1)))


STENCIL_TOL = 1e-6   # fp32: 5 adds + 2 products + 1 subtraction, |rel| <= 8 * 2^-24 ~ 4.8e-7 of the denominator


def rel_error(out, ref, den) -> float:
    """max |out - ref| / den, den = 0 counted as 1 (the absolute difference);
    a non-finite out where ref is finite counts as +inf (as spmv.rel_error)."""
    out = np.asarray(out, np.float64)
    den = np.where(np.asarray(den) == 0, 1.0, den)
    e = np.abs(out - ref) / den
    e = np.where(np.isnan(e), np.inf, e)
    return float(np.max(e)) if out.size else 0.0
