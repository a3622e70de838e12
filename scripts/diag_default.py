"""D4 step time vs T* by default variant, mode and f (back-to-back steps).
python scripts/diag_default.py"""
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


for dname in os.environ.get("DEFAULTS", "csr_vector,csr_stream").split(","):
    dv = D.SPMV_NAMES.index(dname)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=dv)
    T = {D.SPMV_NAMES[v]: b2b(lambda: ctx.spmv_variant(plan, v, x, y)) for v in plan.variant_ids}
    Ts = min(T.values())
    print("default", dname, "pure ms", {k: round(v, 4) for k, v in T.items()})
    for name, mode, f in [("auto_async", D.AUTO | D.ASYNC, 0.005), ("auto_async", D.AUTO | D.ASYNC, 0.002),
                          ("auto_async", D.AUTO | D.ASYNC, 0.01), ("auto_sync", D.AUTO, 0.005),
                          ("fully_async", D.FULLY | D.ASYNC, 0.005), ("fully_sync", D.FULLY, 0.005),
                          ("hyb_async_noabort", D.HYBRID | D.ASYNC | D.NO_ABORT, 0.005),
                          ("no_profile", D.NO_PROFILE, 0.005)]:
        t = b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
        r = ctx.spmv(plan, x, y, f=f, mode=mode, report=True)
        ids = plan.variant_ids
        print(f"  {name:18s} f={f:<6} ms {t:.4f} ovh {100 * (t / Ts - 1):6.1f}% sel {r['selected_name']:10s} "
              f"c {r['c']} eager {r['eager_units']} tail {r['tail_units']} busy_us/unit "
              f"{[round(r['busy_ns'][i] / max(1, r['units'][i]) / 1e3, 1) for i in ids]} "
              f"aborted {[r['aborted'][i] for i in ids]}\n      timeline_us "
              f"{[None if t is None else round(t / 1e3, 1) for t in r['timeline_ns']]}", flush=True)
    plan.destroy()
