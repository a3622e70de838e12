"""Pure full-grid SpMV times (back-to-back) for D4 and D3: A/B of library builds (DYSEL_LIB)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, d3_fem, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n
out = []
for name, A in (("d4", d4_powerlaw()), ("d3", d3_fem())):
    x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=4)
    for v in plan.variant_ids:
        out.append(f"{name}:{D.SPMV_NAMES[v]}={b2b(lambda: ctx.spmv_variant(plan, v, x, y), 20 if name == 'd4' else 100) * 1e3:.1f}us")
    if name == "d4":
        t = b2b(lambda: ctx.spmv(plan, x, y, f=0.005, mode=D.AUTO | D.ASYNC))
        out.append(f"d4:dysel={t * 1e3:.1f}us")
    plan.destroy()
print(os.environ.get("DYSEL_LIB", "default"), " ".join(out), flush=True)
