"""D4 step time vs T* by default variant and mode (back-to-back steps), with
the report's timeline.  python scripts/diag_default.py  (env ROWS, DEFAULTS, F)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32

ctx = D.Context(0)
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000")))
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
s = torch.cuda.current_stream()
F = float(os.environ.get("F", "0.001"))


def b2b(step, n=20):
    for _ in range(5):
        step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n):
        step()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


Ts = None
for dname in os.environ.get("DEFAULTS", "auto,csr_vector,jds").split(","):
    dv = D.SPMV_DEFAULT_AUTO if dname == "auto" else D.SPMV_NAMES.index(dname)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=dv)
    if Ts is None:
        T = {D.SPMV_NAMES[v]: b2b(lambda: ctx.spmv_variant(plan, v, x, y)) for v in plan.variant_ids}
        Ts = min(T.values())
        print("pure ms", {k: round(v, 4) for k, v in T.items()}, "n_light", plan.info.n_light, "n_heavy",
              plan.info.n_heavy, "prep_ms", plan.info.prep_ns / 1e6, flush=True)
        for fl in (0, 1):
            print("  probe", fl, round(b2b(lambda: ctx.spmv_gather_probe(plan, fl, x, y)), 4), flush=True)
    for name, mode, f in [("auto_async", D.AUTO | D.ASYNC, F), ("auto_sync", D.AUTO, F),
                          ("fully_async", D.FULLY | D.ASYNC, F), ("no_profile", D.NO_PROFILE, F)]:
        t = b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
        r = ctx.spmv(plan, x, y, f=f, mode=mode, report=True)
        ids = plan.variant_ids
        print(f"  {D.SPMV_NAMES[plan.info.default_variant]:10s} {name:12s} f={f:<6} ms {t:.4f} ovh "
              f"{100 * (t / Ts - 1):6.1f}% sel {r['selected_name']:10s} c {r['c']} eager {r['eager_units']} "
              f"tail {r['tail_units']} busy_us/unit "
              f"{[round(r['busy_ns'][i] / max(1, r['units'][i]) / 1e3, 1) for i in ids]} "
              f"aborted {[r['aborted'][i] for i in ids]}\n      timeline_us "
              f"{[None if t is None else round(t / 1e3, 1) for t in r['timeline_ns']]}", flush=True)
    plan.destroy()
