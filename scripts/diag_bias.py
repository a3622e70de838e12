"""D4 hybrid/fully with NO_ABORT: per-variant busy time per unit by role (default vs sandbox)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=10_000_000)
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
for default in (D.SPMV_CSR_VECTOR, D.SPMV_CSR_STREAM, D.SPMV_CSR_SCALAR):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL, default=default)
    ids = plan.variant_ids
    print("default", D.SPMV_NAMES[default])
    for f in (0.005, 0.02):
        for mode, mn in ((D.HYBRID | D.NO_ABORT, "hybrid_sync"), (D.HYBRID | D.ASYNC | D.NO_ABORT, "hybrid_async"),
                         (D.FULLY | D.NO_ABORT, "fully_sync"), (D.HYBRID | D.NO_ABORT | D.SEQUENTIAL, "hybrid_seq"),
                         (D.HYBRID | D.NO_ABORT | D.SCORE_MAKESPAN, "hybrid_mksp")):
            for _ in range(2): ctx.spmv(plan, x, y, f=f, mode=mode | D.FORCE_PROFILE)
            r = ctx.spmv(plan, x, y, f=f, mode=mode | D.FORCE_PROFILE, report=True)
            print(f"  f={f} {mn:13s} sel {r['selected_name']:10s} c {r['c']} pred_ms", [round(r["score"][v] / 1e6, 3) for v in ids],
                  "busy/unit", [round(r["busy_ns"][v] / max(1, r["units"][v]) / 1e3, 1) for v in ids],
                  "mksp_ms", [round(r["makespan_ns"][v] / 1e6, 3) for v in ids])
    plan.destroy()
