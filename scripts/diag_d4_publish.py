"""D4 headline pool: per-variant profiling makespan / busy / aborted and the
publish time, SYNC and ASYNC (what bounds the selection latency)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
A, x = bench.make_d4(10_000_000)
ctx = D.Context(0)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
xd = torch.from_numpy(x).cuda()
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
ids = plan.variant_ids
for name, mode in (("sync", D.AUTO), ("async", D.AUTO | D.ASYNC)):
    for _ in range(3):
        r = ctx.spmv(plan, xd, y, f=0.001, mode=mode, report=True)
    print(name, "c", r["c"], "tl_us", [None if t is None else round(t / 1e3, 1) for t in r["timeline_ns"]])
    for v in ids:
        print("   ", D.SPMV_NAMES[v], "makespan_us", round(r["makespan_ns"][v] / 1e3, 1), "busy/unit",
              round(r["busy_ns"][v] / max(1, r["units"][v]) / 1e3, 1), "units", r["units"][v], "aborted", r["aborted"][v],
              "score", r["score"][v])
