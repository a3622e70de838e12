"""Cost of the sandbox dominance poll: default = JDS (slowest, completes last),
so sandboxes poll but are never dominated before they finish."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=10_000_000)
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL, default=D.SPMV_JDS)
ids = plan.variant_ids
for f in (0.005, 0.02):
    for mode, mn in ((D.HYBRID, "poll"), (D.HYBRID | D.NO_ABORT, "nopoll"), (D.HYBRID | D.SEQUENTIAL, "poll_seq"),
                     (D.HYBRID | D.SEQUENTIAL | D.NO_ABORT, "nopoll_seq")):
        for _ in range(2): ctx.spmv(plan, x, y, f=f, mode=mode | D.FORCE_PROFILE)
        r = ctx.spmv(plan, x, y, f=f, mode=mode | D.FORCE_PROFILE, report=True)
        print(f"f={f} {mn:11s} sel {r['selected_name']:10s}", "busy/unit", [round(r["busy_ns"][v] / max(1, r["units"][v]) / 1e3, 1) for v in ids],
              "aborted", [r["aborted"][v] for v in ids], "max_unit_us", [round(r["score"][v] / 1e3) for v in ids])
