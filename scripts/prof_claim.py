"""One plain CSR-W grid and one claim-kernel run on D4 (for ncu)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000")))
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
v = int(os.environ.get("V", "4"))
for how in (0, 3):
    ctx.debug_spmv_device_launch(plan, v, x, y, how)
torch.cuda.synchronize()
