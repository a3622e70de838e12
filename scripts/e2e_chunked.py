"""End-to-end SpMV with host buffers: copy -> dysel_spmv -> copy vs
dysel_spmv_host (y copied out in chunks released by the SpMV's slot counters),
back to back, on a 9M-row FEM matrix (units complete in index order) and D4."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import make_d4, time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
for name, mk in (("fem_9M", lambda: d3_fem(grid=3000)), ("d4", lambda: make_d4(10_000_000)[0])):
    A = mk()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
    hx = torch.from_numpy(uniform_f32(3, A.n_cols)).pin_memory()
    hy = torch.empty(A.n_rows).pin_memory()
    dx = torch.empty(A.n_cols, device="cuda")
    dy = torch.empty(A.n_rows, device="cuda")
    for mn, md in (("auto_async", D.AUTO | D.ASYNC), ("no_profile", D.NO_PROFILE)):
        def plain():
            dx.copy_(hx, non_blocking=True)
            ctx.spmv(plan, dx, dy, f=0.001, mode=md)
            hy.copy_(dy, non_blocking=True)
        tk = time_b2b(lambda: ctx.spmv(plan, dx, dy, f=0.001, mode=md), 10, s)
        tp = time_b2b(plain, 10, s)
        tc = time_b2b(lambda: ctx.spmv_host(plan, hx, hy, dx, dy, f=0.001, mode=md), 10, s)
        print(name, mn, "spmv us", round(tk * 1e6, 1), "copy+spmv+copy us", round(tp * 1e6, 1),
              "spmv_host us", round(tc * 1e6, 1), flush=True)
    plan.destroy()
    del rp, col, val, A
