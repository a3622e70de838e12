"""Selection on a regular multi-wave FEM matrix (2.25M rows, 5x5 stencil):
pure variant times (cold L2) vs the DySel selection and scores per scoring
mode.  python scripts/diag_d3x.py [grid]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
grid = int(sys.argv[1]) if len(sys.argv) > 1 else 1500
FS = [float(v) for v in sys.argv[2].split(",")] if len(sys.argv) > 2 else (0.02, 0.05)
ctx = D.Context(0)
A = d3_fem(grid=grid)
x = torch.from_numpy(uniform_f32(385, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
def cold(fn, reps=10):
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return float(np.median(ts))
for fm, name in ((D.FMT_ALL, "all"), (D.FMT_DEFAULT, "default")):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=fm)
    T = {D.SPMV_NAMES[v]: cold(lambda: ctx.spmv_variant(plan, v, x, y)) for v in plan.variant_ids}
    print(name, "pure us (cold)", {k: round(v, 1) for k, v in T.items()}, flush=True)
    for mname, mode in (("fully_async", D.FULLY | D.ASYNC), ("fully_sync", D.FULLY), ("makespan", D.FULLY | D.ASYNC |
                         D.SCORE_MAKESPAN), ("cycles", D.FULLY | D.ASYNC | D.SCORE_CYCLES),
                        ("seq", D.FULLY | D.SEQUENTIAL), ("hybrid_async", D.HYBRID | D.ASYNC)):
        for f in FS:
            t = cold(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
            sels = [ctx.spmv(plan, x, y, f=f, mode=mode, report=True) for _ in range(5)]
            r = sels[-1]
            ids = plan.variant_ids
            print(f"  {mname:12s} f={f} us {t:7.1f} sel {[q['selected_name'] for q in sels]} c {r['c']} "
                  f"score {[r['score'][i] for i in ids]} busy/unit {[round(r['busy_ns'][i] / max(1, r['units'][i]) / 1e3, 2) for i in ids]} "
                  f"makespan {[round(r['makespan_ns'][i] / 1e3, 1) for i in ids]}", flush=True)
    plan.destroy()
