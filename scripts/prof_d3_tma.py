"""D3 pure runs of CSR-T (bulk-staged) and ELL for ncu --set full (A/B of the staging)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
A = d3_fem()
x = torch.from_numpy(uniform_f32(384, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL, default=D.SPMV_DEFAULT_AUTO)
for v in (D.SPMV_CSR_TMA, D.SPMV_ELL):
    for _ in range(3):
        ctx.spmv_variant(plan, v, x, y)
torch.cuda.synchronize()
