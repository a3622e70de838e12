"""D4 with the full pool (CSR-W included): does profiling rank CSR-W first?"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=10_000_000)
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
s = torch.cuda.current_stream()
def b2b(fn, reps=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(reps): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps
y = torch.empty(A.n_rows, device="cuda")
for default in (D.SPMV_CSR_VECTOR, D.SPMV_CSR_STREAM):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL, default=default)
    ids = plan.variant_ids
    print("default", D.SPMV_NAMES[default], "variants", {D.SPMV_NAMES[v]: round(b2b(lambda: ctx.spmv_variant(plan, v, x, y)), 4) for v in ids})
    for f in (0.005, 0.02):
        for mode, mn in ((D.AUTO | D.ASYNC, "auto_async"), (D.FULLY | D.ASYNC, "fully_async")):
            t = b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
            sels = [ctx.spmv(plan, x, y, f=f, mode=mode, report=True) for _ in range(5)]
            r = sels[-1]
            print(f"  f={f} {mn}: {t:.4f} ms sel {[q['selected_name'] for q in sels]} score",
                  [r["score"][v] for v in ids], "busy/unit", [round(r["busy_ns"][v] / max(1, r["units"][v]) / 1e3, 1) for v in ids])
    plan.destroy()
