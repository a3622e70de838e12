"""Heavy-first claim order (A-40) A/B: pure CSR-W / CSR-V times on power-law
matrices of several sizes (run with and without DYSEL_LIB=exp_libs/noheavy/...)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=50):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n
out = []
for n in (60_000, 300_000, 1_000_000, 3_000_000):
    A = d4_powerlaw(n=n, lmax=16384)
    x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=4)
    for v in (1, 4):
        out.append(f"n{n}(h{plan.info.n_heavy}):{D.SPMV_NAMES[v]}={b2b(lambda: ctx.spmv_variant(plan, v, x, y)) * 1e3:.1f}us")
    plan.destroy()
print(os.environ.get("DYSEL_LIB", "default"), " ".join(out), flush=True)
