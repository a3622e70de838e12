"""Diagnostics: per-variant times and DySel reports (scores) on D4 / D3."""
import os, sys
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
which = sys.argv[1] if len(sys.argv) > 1 else "d4"
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000"))) if which == "d4" else d3_fem()
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
y = torch.empty(A.n_rows, device="cuda")
only = os.environ.get("ONLY")
for v in plan.variant_ids:
    if only and D.SPMV_NAMES[v] != only: continue
    ctx.spmv_variant(plan, v, x, y)
    print("variant", D.SPMV_NAMES[v], "ms", round(ev_time(lambda: ctx.spmv_variant(plan, v, x, y)), 4))
if only: sys.exit(0)
ids = plan.variant_ids
F = float(os.environ.get("F", "0.02"))
MODES = [(f"auto_async_f{f}", D.AUTO|D.ASYNC, f) for f in (0.002, 0.005, 0.01, 0.02, 0.05)] + [("auto_async", D.AUTO|D.ASYNC, F), ("auto_sync", D.AUTO, F), ("fully_async", D.FULLY|D.ASYNC, F),
                   ("hybrid_async_f.005", D.HYBRID|D.ASYNC, 0.005), ("hybrid_seq_f.1", D.HYBRID|D.SEQUENTIAL, 0.1),
                   ("hybrid_seq_f.05", D.HYBRID|D.SEQUENTIAL, 0.05), ("fully_seq_f.1", D.FULLY|D.SEQUENTIAL, 0.1),
                   ("hybrid_sync_host", D.HYBRID|D.HOST_ORCH, F), ("no_profile", D.NO_PROFILE, F)]
for name, mode, f in MODES:
    t = ev_time(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
    r = ctx.spmv(plan, x, y, f=f, mode=mode, report=True)
    print(f"{name:22s} ms {t:8.4f} sel {r['selected_name']:10s} c {r['c']} eager {r['eager_units']} tail {r['tail_units']}",
          "score", [r["score"][i] for i in ids], "busy_us/unit", [round(r["busy_ns"][i]/max(1,r["units"][i])/1e3,1) for i in ids],
          "aborted", [r["aborted"][i] for i in ids])
