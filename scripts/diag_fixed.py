"""Fixed per-call cost of a profiled dysel_spmv on a small matrix (D6 diagonal 2^21)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d6_diag, uniform_f32
ctx = D.Context(0)
A = d6_diag()
x = torch.from_numpy(uniform_f32(6, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
y = torch.empty(A.n_rows, device="cuda")
s = torch.cuda.current_stream()
def b2b(fn, reps=50):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(reps): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e3
F = D.FORCE_PROFILE
print("variant csr_scalar", b2b(lambda: ctx.spmv_variant(plan, 0, x, y)))
for name, m in [("fully_sync", D.FULLY | F), ("fully_sync_notail", D.FULLY | F | D.NO_TAIL), ("fully_async", D.FULLY | D.ASYNC | F),
                ("hybrid_async", D.HYBRID | D.ASYNC | F), ("no_profile", D.NO_PROFILE), ("seq", D.FULLY | F | D.SEQUENTIAL)]:
    for f in (0.001, 0.02):
        print(f"{name:20s} f={f}: {b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=m)):8.1f} us")
# D4 comparison: tail launch vs host switch remainder
from workloads import d4_powerlaw
A4 = d4_powerlaw(n=10_000_000)
x4 = torch.from_numpy(uniform_f32(3, A4.n_cols)).cuda()
rp4, col4, val4 = (torch.from_numpy(a).cuda() for a in (A4.row_ptr, A4.col, A4.val))
plan4 = ctx.spmv_prepare(rp4, col4, val4, A4.n_cols)
y4 = torch.empty(A4.n_rows, device="cuda")
print("D4 csr_vector", b2b(lambda: ctx.spmv_variant(plan4, 1, x4, y4), 20))
for name, m in [("auto_sync_tail", D.AUTO), ("auto_sync_switch", D.AUTO | D.NO_TAIL), ("auto_async", D.AUTO | D.ASYNC)]:
    print(f"D4 {name:20s}: {b2b(lambda: ctx.spmv(plan4, x4, y4, f=0.005, mode=m), 20):8.1f} us")
