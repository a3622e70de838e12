"""A/B: D4 DySel hybrid-async step vs pure CSR-W (default = CSR-W), back to back."""
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
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000")))
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=int(os.environ.get("DEF", "4")))
out = []
for rep in range(2):
    T = b2b(lambda: ctx.spmv_variant(plan, 4, x, y))
    out.append(f"pure={T:.1f}")
    for f in (0.005, 0.0005):
        t = b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC))
        out.append(f"f{f}={t:.1f}({100*(t/T-1):.1f}%)")
print(os.environ.get("DYSEL_LIB", "default"), " ".join(out), flush=True)
