"""Back-to-back vs synchronised DySel SpMV steps on D4, per mode."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=10_000_000)
x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
y = torch.empty(A.n_rows, device="cuda")
s = torch.cuda.current_stream()
def measure(name, step):
    for _ in range(5): step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(20): step()
    b.record(s); torch.cuda.synchronize()
    t_b2b = a.elapsed_time(b) / 20
    ts = []
    for _ in range(20):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); step(); b.record(s); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    print(f"{name:28s} back-to-back {t_b2b:.4f} ms/step, synced median {np.median(ts):.4f} ms")
f = 0.005
measure("auto_async", lambda: ctx.spmv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC))
measure("auto_sync", lambda: ctx.spmv(plan, x, y, f=f, mode=D.AUTO))
measure("hybrid_async_notail", lambda: ctx.spmv(plan, x, y, f=f, mode=D.HYBRID | D.ASYNC | D.NO_TAIL))
measure("hybrid_sync_notail", lambda: ctx.spmv(plan, x, y, f=f, mode=D.HYBRID | D.NO_TAIL))
measure("no_profile", lambda: ctx.spmv(plan, x, y, mode=D.NO_PROFILE))
measure("csr_vector", lambda: ctx.spmv_variant(plan, 1, x, y))
