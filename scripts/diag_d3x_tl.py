"""D3x (FEM 1500^2, all formats) single shot with the report timeline, per mode."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
A = d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ALL)
print("default", D.SPMV_NAMES[plan.info.default_variant])
for mname, mode in (("fully_async", D.FULLY | D.ASYNC), ("fully_sync", D.FULLY), ("hybrid_async", D.HYBRID | D.ASYNC)):
    for _ in range(3):
        r = ctx.spmv(plan, x, y, f=0.02, mode=mode, report=True)
    print(mname, r["selected_name"], "eager", r["eager_units"], "tail", r["tail_units"],
          "tl_us", [None if t is None else round(t / 1e3, 1) for t in r["timeline_ns"]], flush=True)
