"""D3 / D3x (5x5 FEM stencil, all formats): pure variants vs DySel single shot per mode, cold L2."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0); s = torch.cuda.current_stream()
flush = torch.empty(256 * 1024 * 1024 // 4, device="cuda")
def cold(fn, reps=20):
    ts = []
    for _ in range(reps + 3):
        flush.fill_(1.0); a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    return float(np.median(ts[3:])) * 1e3
for grid in [int(g) for g in os.environ.get("GRIDS", "383,1500").split(",")]:
    A = d3_fem(grid=grid)
    x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, **({} if os.environ.get("DEFAULT_POOL") else {"formats": D.FMT_ALL}))
    res = {D.SPMV_NAMES[v]: cold(lambda: ctx.spmv_variant(plan, v, x, y)) for v in plan.variant_ids}
    best = min(res.values())
    for name, mode in (("auto_async", D.AUTO | D.ASYNC), ("auto_sync", D.AUTO), ("forced_async", D.AUTO | D.ASYNC | D.FORCE_PROFILE)):
        td = cold(lambda: ctx.spmv(plan, x, y, f=0.02, mode=mode))
        r = ctx.spmv(plan, x, y, f=0.02, mode=mode, report=True)
        print(grid, D.SPMV_NAMES[plan.info.default_variant], name, {k: round(v, 1) for k, v in res.items()}, "dysel", round(td, 1),
              "ovh%", round((td / best - 1) * 100, 1), "sel", r["selected_name"], "prof", r["profiled"],
              "tl", [None if t is None else round(t / 1e3, 1) for t in r["timeline_ns"]], flush=True)
    plan.destroy()
