"""ncu target: the pure CSR-W claim kernel on D4 (one launch after a warm-up)."""
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
ctx.spmv_variant(plan, 4, x, y)
ctx.spmv_variant(plan, 4, x, y)
torch.cuda.synchronize()
print("done")
