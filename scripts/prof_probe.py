"""ncu target: D4 gather probe (flavour 0 / 1) and the pure CSR-W claim kernel, one launch each."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw()
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=4)
torch.cuda.synchronize()
ctx.spmv_gather_probe(plan, 0, x, y)
ctx.spmv_gather_probe(plan, 1, x, y)
ctx.spmv_variant(plan, 4, x, y)
torch.cuda.synchronize()
print("done")
