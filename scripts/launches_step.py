"""Kernel launch list of the headline DySel step (bench.py's timed region:
D4 10M rows, AUTO|ASYNC, f = 0.001) for ncu:
  ncu --nvtx --nvtx-include "step/" --metrics gpu__time_duration.sum --clock-control none \
      --csv --log-file profiles/launches_r2.csv python scripts/launches_step.py
Three steps after five warm-up steps, each inside an NVTX range "step"."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
A, x = bench.make_d4(10_000_000)
ctx = D.Context(0)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
xd = torch.from_numpy(x).cuda()
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
step = lambda: ctx.spmv(plan, xd, y, f=0.001, mode=D.AUTO | D.ASYNC)
for _ in range(5):
    step()
torch.cuda.synchronize()
for _ in range(3):
    torch.cuda.nvtx.range_push("step")
    step()
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
print("done")
