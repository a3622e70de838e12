"""compute-sanitizer target: every SpMV variant and the DySel device path on
ragged matrices whose nnz is not a multiple of 4 (exact-size allocations:
run with PYTORCH_NO_CUDA_MEMORY_CACHING=1), checked against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from oracle import spmv as ospmv
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, random_lengths_csr, uniform_f32
ctx = D.Context(0)
bad = 0
for A in (random_lengths_csr(3001, 2000, 700, 31, empty_frac=0.2), d4_powerlaw(n=160_000, lmax=16384)):
    for cut in (0, 1, 2, 3):   # drop entries of the last row: nnz mod 4 takes every value
        rp = A.row_ptr.copy()
        last = max(int(rp[-2]), int(rp[-1]) - cut)
        rp[-1] = last
        col, val = A.col[:last].copy(), A.val[:last].copy()
        x = uniform_f32(3, A.n_cols)
        d = [torch.from_numpy(a).cuda() for a in (rp, col, val)]
        plan = ctx.spmv_prepare(*d, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ALL)
        xd = torch.from_numpy(x).cuda()
        ys = ospmv.spmv(rp, col, val, x)
        dd = ospmv.spmv_abs(rp, col, val, x)
        runs = [("pure", v) for v in plan.variant_ids] + [("dysel", m) for m in
                (D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.FULLY | D.FORCE_PROFILE, D.HYBRID | D.ASYNC | D.FORCE_PROFILE)]
        for kind, a in runs:
            y = torch.full((A.n_rows,), float("nan"), device="cuda")
            if kind == "pure":
                ctx.spmv_variant(plan, a, xd, y)
            else:
                ctx.spmv(plan, xd, y, f=0.05, mode=a)
            torch.cuda.synchronize()
            e = ospmv.rel_error(y.cpu().numpy(), ys, dd)
            if not e <= ospmv.SPMV_TOL:
                bad += 1
                print("FAIL", A.n_rows, last % 4, kind, a, e, flush=True)
        plan.destroy()
print("memcheck target done, failures:", bad, flush=True)
