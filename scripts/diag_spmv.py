"""Diagnostics: per-variant times and DySel reports (scores) on D4 / D3."""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, d3_fem, uniform_f32

def ev_time(fn, reps=10):
    s = torch.cuda.current_stream(); out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s); torch.cuda.synchronize(); out.append(a.elapsed_time(b))
    return float(np.median(out))

ctx = D.Context(0)
print("tick_ns", ctx.globaltimer_tick_ns, "n_sm", ctx.n_sm, "calib", ctx.timer_calibrate())
which = sys.argv[1] if len(sys.argv) > 1 else "d4"
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000"))) if which == "d4" else d3_fem()
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
y = torch.empty(A.n_rows, device="cuda")
for v in plan.variant_ids:
    ctx.spmv_variant(plan, v, x, y)
    print("variant", D.SPMV_NAMES[v], "ms", ev_time(lambda: ctx.spmv_variant(plan, v, x, y)))
for name, mode in [("auto_async", D.AUTO|D.ASYNC), ("auto_sync", D.AUTO), ("fully_async", D.FULLY|D.ASYNC),
                   ("hybrid_async_cycles", D.HYBRID|D.ASYNC|D.SCORE_CYCLES), ("fully_async_cycles", D.FULLY|D.ASYNC|D.SCORE_CYCLES),
                   ("hybrid_sync_host", D.HYBRID|D.HOST_ORCH)]:
    t = ev_time(lambda: ctx.spmv(plan, x, y, f=0.02, mode=mode))
    r = ctx.spmv(plan, x, y, f=0.02, mode=mode, report=True)
    ids = plan.variant_ids
    print(name, "ms", round(t, 4), "sel", r["selected_name"], "c", r["c"], "eager", r["eager_units"],
          "makespan_us", [round(r["makespan_ns"][i]/1e3, 1) for i in ids],
          "cyc_per_unit", [r["cycles"][i] // max(1, r["units"][i]) for i in ids], "units", [r["units"][i] for i in ids])
