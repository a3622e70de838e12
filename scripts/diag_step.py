"""D4 DySel step anatomy: b2b times for mode / f / pool variations + report timeline."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
A = d4_powerlaw()
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
for fm, label, dflt in ((D.FMT_DEFAULT, "pool4", D.SPMV_DEFAULT_AUTO), (D.FMT_DEFAULT, "pool4_defV", 1)):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=fm, default=dflt)
    T = b2b(lambda: ctx.spmv_variant(plan, 4, x, y))
    print(os.environ.get("DYSEL_LIB", "default"), label, "pure csr_stream", round(T, 1), "us", flush=True)
    for name, mode, f in [("hyb_async", D.AUTO | D.ASYNC, 0.002), ("hyb_async", D.AUTO | D.ASYNC, 0.001),
                          ("hyb_async", D.AUTO | D.ASYNC, 0.0005), ("no_profile", D.AUTO | D.NO_PROFILE, 0.002),
                          ("fully_async", D.FULLY | D.ASYNC, 0.002), ("hyb_sync", D.AUTO, 0.002),
                          ("hyb_async_solo", D.AUTO | D.ASYNC | D.SOLO, 0.001),
                          ("no_profile_solo", D.AUTO | D.NO_PROFILE | D.SOLO, 0.001),
                          ("hyb_async_allclaims", D.AUTO | D.ASYNC | D.ALL_CLAIMS, 0.001)]:
        t = b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=mode))
        r = ctx.spmv(plan, x, y, f=f, mode=mode, report=True)
        print(f"  {label} {name:18s} f={f:<7} {t:7.1f} us ovh {100*(t/T-1):5.1f}% c={r['c']} eager={r['eager_units']} "
              f"sel={r['selected_name']} tl_us={[None if (v is None or r['timeline_ns'][0] is None) else round((v-r['timeline_ns'][0])/1e3,1) for v in r['timeline_ns']]}", flush=True)
    plan.destroy()
