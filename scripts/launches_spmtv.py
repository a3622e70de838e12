"""Launch list of one SpMTV swap call (for ncu --metrics gpu__time_duration.sum)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d4_powerlaw, uniform_f32  # noqa: E402

ctx = D.Context(0)
A = d4_powerlaw(n=2_000_000, lmax=4096)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
x = torch.from_numpy(uniform_f32(61, A.n_rows)).cuda()
y = torch.zeros(A.n_cols, device="cuda")
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("swap")
ctx.spmtv(plan, x, y, f=0.01, mode=D.AUTO)
torch.cuda.synchronize()
