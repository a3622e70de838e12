"""D3x (FEM 1500^2, all formats): DySel single shot by initial version, with timeline."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
A = d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
s = torch.cuda.current_stream()
for dname in ("ell", "csr_tma", "csr_scalar"):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_NAMES.index(dname), formats=D.FMT_ALL)
    tp = bench.time_b2b(lambda: ctx.spmv_variant(plan, D.SPMV_CSR_TMA, x, y), 20, s)
    for mname, mode in (("fully_async", D.FULLY | D.ASYNC), ("fully_sync", D.FULLY)):
        t = bench.time_b2b(lambda: ctx.spmv(plan, x, y, f=0.02, mode=mode | D.FORCE_PROFILE), 20, s)
        r = ctx.spmv(plan, x, y, f=0.02, mode=mode | D.FORCE_PROFILE, report=True)
        print(dname, mname, f"{t*1e6:.1f} us vs csr_tma pure {tp*1e6:.1f} ({100*(t/tp-1):.1f}%)", r["selected_name"],
              "eager", r["eager_units"], "tl_us", [None if v is None else round(v / 1e3, 1) for v in r["timeline_ns"]], flush=True)
    plan.destroy()
