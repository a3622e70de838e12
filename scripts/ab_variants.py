"""A/B of pure variant times between library builds (DYSEL_LIB=<alt .so>):
D4 (10M power-law), D3x (FEM 1500^2) and D1-like uniform; cold-L2 b2b medians.
python scripts/ab_variants.py  (prints one JSON line per matrix)"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
mats = [("d4", lambda: bench.make_d4(10_000_000)[0]), ("d3x", lambda: d3_fem(grid=1500))]
for name, mk in mats:
    A = mk()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ALL)
    out = {"lib": os.path.basename(D.LIB_PATH), "mat": name}
    for v in plan.variant_ids:
        out[D.SPMV_NAMES[v]] = round(bench.time_b2b(lambda: ctx.spmv_variant(plan, v, x, y), 20, s) * 1e6, 1)
    out["auto"] = round(bench.time_b2b(lambda: ctx.spmv(plan, x, y, f=0.001, mode=D.AUTO | D.ASYNC), 20, s) * 1e6, 1)
    print(json.dumps(out), flush=True)
    plan.destroy()
    del rp, col, val
