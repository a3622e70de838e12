"""D3x with ELL as the initial version and CSR-T winning (SYNC): the switch
kernel device-launches CSR-T's claim kernel.  For ncu on that child launch vs
the host-launched pure CSR-T claim kernel."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
A = d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_ELL, formats=D.FMT_ALL)
for _ in range(2):
    ctx.spmv_variant(plan, D.SPMV_CSR_TMA, x, y)
    r = ctx.spmv(plan, x, y, f=0.02, mode=D.FULLY | D.FORCE_PROFILE, report=True)
torch.cuda.synchronize()
print(r["selected_name"])
