"""ELL chunk / occupancy A/B (DYSEL_LIB builds): pure ELL back to back on D3,
D6 random / diagonal and a 2.25M-row FEM matrix (multi-wave)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, d6_diag, d6_random, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=100):
    for _ in range(5): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
out = []
for name, A in (("d3", d3_fem()), ("d6r", d6_random()), ("d6d", d6_diag()), ("fem1500", d3_fem(grid=1500))):
    x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    for v in (0, 2, 3):
        if v in plan.variant_ids:
            out.append(f"{name}:{D.SPMV_NAMES[v]}={b2b(lambda: ctx.spmv_variant(plan, v, x, y)):.1f}us")
    plan.destroy()
print(os.environ.get("DYSEL_LIB", "default"), " ".join(out), flush=True)
