"""D3x (2.25M-row FEM, every format): per-call report timeline (publish vs the
last profiling CTA's end) and per-variant profiling makespans, sync / async."""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch  # noqa: E402

from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d3_fem, uniform_f32  # noqa: E402

ctx = D.Context(0)
A = d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ALL)
for mode, nm in ((D.AUTO, "sync"), (D.AUTO | D.ASYNC, "async")):
    for _ in range(3):
        r = ctx.spmv(plan, x, y, f=0.02, mode=mode, report=True)
        tl = [None if t is None else round(t / 1e3, 1) for t in r["timeline_ns"]]
        print(nm, "sel", r["selected_name"], "publish", tl[1], "last profiling CTA end", tl[2], "tl", tl)
        print("   makespan us", [round(m / 1e3, 1) for m in r["makespan_ns"][:r["n_variants"]]])
