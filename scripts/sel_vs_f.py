"""Selection vs profile fraction f on regular FEM matrices (default pool and
all formats): how often DySel picks the pure-best variant, 10 calls per f."""
import os, sys, collections
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from bench import time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0); s = torch.cuda.current_stream()
for grid in [int(g) for g in os.environ.get("GRIDS", "1500,3000").split(",")]:
    A = d3_fem(grid=grid)
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda(); y = torch.empty(A.n_rows, device="cuda")
    for pool, kw in ((("default", {}), ("all", {"formats": D.FMT_ALL})) if not os.environ.get("ONLY_DEFAULT") else (("default", {}),)):
        plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, **kw)
        T = {D.SPMV_NAMES[v]: time_b2b(lambda: ctx.spmv_variant(plan, v, x, y), 10, s) for v in plan.variant_ids}
        best = min(T, key=T.get)
        for f in [float(v) for v in os.environ.get("FS", "0.001,0.002,0.005,0.01,0.02").split(",")]:
            c = collections.Counter()
            for _ in range(10):
                r = ctx.spmv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC, report=True)
                c[r["selected_name"]] += 1
            print(grid, pool, "f", f, "c", r["c"], "best", best, {k: round(v * 1e6) for k, v in T.items()}, dict(c), flush=True)
        plan.destroy()
