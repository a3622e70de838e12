"""A-38 A/B: D4 DySel step with a non-best default (the winner's remainder then runs inside the default's claim kernel when solo)."""
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
for dv in (D.SPMV_CSR_STREAM, D.SPMV_CSR_VECTOR, D.SPMV_JDS, D.SPMV_CSR_SCALAR):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=dv)
    T = b2b(lambda: ctx.spmv_variant(plan, D.SPMV_CSR_STREAM, x, y))
    out = []
    for name, md in (("solo", D.AUTO | D.ASYNC | D.SOLO), ("per-variant", D.AUTO | D.ASYNC)):
        t = b2b(lambda: ctx.spmv(plan, x, y, f=0.001, mode=md))
        r = ctx.spmv(plan, x, y, f=0.001, mode=md, report=True)
        out.append(f"{name}: {t:.1f} us ({100 * (t / T - 1):+.1f}%, sel {r['selected_name']}, eager {r['eager_units']})")
    print(f"default {D.SPMV_NAMES[dv]:11s} best-pure {T:.1f} us | " + " | ".join(out), flush=True)
    plan.destroy()
