"""SpMTV swap-mode overhead on the 2M-row power-law matrix (bench secondary
spmtv_powerlaw_2M, standalone): pure variants, AUTO (swap) single shot, host
swap, amortised.  Run with DYSEL_SPMTV_PERSISTENT=1 for the persistent-wave
remainder ablation (removed)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from bench import time_b2b  # noqa: E402
from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d4_powerlaw, uniform_f32  # noqa: E402

ctx = D.Context(0)
stream = torch.cuda.current_stream()
A = d4_powerlaw(n=2_000_000, lmax=4096)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
x = torch.from_numpy(uniform_f32(61, A.n_rows)).cuda()
y = torch.zeros(A.n_cols, device="cuda")
t = {D.SPMTV_NAMES[v]: time_b2b(lambda: ctx.spmtv_variant(plan, v, x, y), 20, stream) for v in range(len(D.SPMTV_NAMES))}
best = min(t.values())
out = {"persistent": bool(os.environ.get("DYSEL_SPMTV_PERSISTENT")), "pure_us": {k: round(v * 1e6, 1) for k, v in t.items()}}
for f in (0.002, 0.005, 0.01, 0.02):
    td = time_b2b(lambda: ctx.spmtv(plan, x, y, f=f, mode=D.AUTO), 20, stream)
    rep = ctx.spmtv(plan, x, y, f=f, mode=D.AUTO, report=True)
    sels = [ctx.spmtv(plan, x, y, f=f, mode=D.AUTO, report=True)["selected_name"] for _ in range(10)]
    out["f=%g" % f] = {"us": round(td * 1e6, 1), "overhead_pct": round((td / best - 1) * 100, 2),
                       "selected": rep["selected_name"], "c": rep["c"], "profiled": rep["profiled"],
                       "selections_10": sels, "score": rep["score"][:3], "aborted": rep["aborted"][:3],
                       "timeline_us": [None if t is None else round(t / 1e3, 1) for t in rep["timeline_ns"]]}
print(json.dumps(out))
for name, m in (("swap_no_abort", D.AUTO | D.NO_ABORT), ("fully", D.FULLY), ("swap_sequential", D.AUTO | D.SEQUENTIAL)
                if hasattr(D, "SEQUENTIAL") else (("swap_no_abort", D.AUTO | D.NO_ABORT), ("fully", D.FULLY))):
    td = time_b2b(lambda: ctx.spmtv(plan, x, y, f=0.01, mode=m), 20, stream)
    rep = ctx.spmtv(plan, x, y, f=0.01, mode=m, report=True)
    print(name, round(td * 1e6, 1), "us", {k: rep.get(k) for k in ("selected_name", "makespan_ns", "score", "aborted",
                                                                  "busy_ns", "host_ns", "mode_used")})
rep = ctx.spmtv(plan, x, y, f=0.01, mode=D.AUTO, report=True)
print("swap", {k: rep.get(k) for k in ("selected_name", "makespan_ns", "score", "aborted", "busy_ns", "host_ns")})
