"""Per-variant SpMV times on the small / regular inputs (D3, D6, D1): cold L2
(flush before each launch) and back-to-back.  python scripts/diag_small.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d1_bus, d3_fem, d6_diag, d6_random, uniform_f32

ctx = D.Context(0)
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def cold(fn, n=20):
    ts = []
    for _ in range(n):
        flush.zero_()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return float(np.median(ts))


def b2b(fn, n=50):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n):
        fn()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / n


for name, A in (("d3", d3_fem()), ("d6_random", d6_random()), ("d6_diag", d6_diag()), ("d1", d1_bus())):
    x = torch.from_numpy(uniform_f32(7, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL | D.FMT_STREAM)
    y = torch.empty(A.n_rows, device="cuda")
    nb = 8 * A.nnz + 4 * (A.n_rows + 1) + 4 * A.n_cols + 4 * A.n_rows
    print(f"{name}: n={A.n_rows} nnz={A.nnz} bytes={nb/1e6:.2f} MB")
    for v in plan.variant_ids:
        fn = lambda: ctx.spmv_variant(plan, v, x, y)
        tc, tb = cold(fn), b2b(fn)
        print(f"  {D.SPMV_NAMES[v]:11s} cold {tc:7.2f} us ({nb/tc/1e3:6.0f} GB/s)  b2b {tb:7.2f} us ({nb/tb/1e3:6.0f} GB/s)")
    plan.destroy()
