"""SpMTV pool on short / uniform row shapes (b2b us): which variant wins where,
and what DySel selects (sync / async, f = 0.02).  Basis of reading A-30d."""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch  # noqa: E402

from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d3_fem, d4_powerlaw, random_lengths_csr, uniform_f32  # noqa: E402

ctx = D.Context(0)
st = torch.cuda.current_stream()
cases = [("len0-2", lambda: random_lengths_csr(1_500_000, 1_200_000, 2, 81)),
         ("len0-8", lambda: random_lengths_csr(2_000_000, 2_000_000, 8, 85)),
         ("len0-16", lambda: random_lengths_csr(1_500_000, 1_200_000, 16, 84)),
         ("len0-32", lambda: random_lengths_csr(1_500_000, 1_500_000, 32, 86)),
         ("len0-48", lambda: random_lengths_csr(1_000_000, 1_000_000, 48, 87)),
         ("fem25_1M", lambda: d3_fem(grid=1000)),
         ("powerlaw_2M", lambda: d4_powerlaw(n=2_000_000, lmax=4096))]


def b2b(fn, n=20):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(n):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1e3


for name, mk in cases:
    A = mk()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    x = torch.from_numpy(uniform_f32(82, A.n_rows)).cuda()
    y = torch.zeros(A.n_cols, device="cuda")
    t = {D.SPMTV_NAMES[v]: round(b2b(lambda: ctx.spmtv_variant(plan, v, x, y)), 1) for v in range(3)}
    out = {}
    for m, nm in ((D.AUTO, "sync"), (D.AUTO | D.ASYNC, "async")):
        out[nm] = round(b2b(lambda: ctx.spmtv(plan, x, y, f=0.02, mode=m)), 1)
        r = ctx.spmtv(plan, x, y, f=0.02, mode=m, report=True)
        out[nm + "_sel"] = r["selected_name"]
        out[nm + "_prof"] = r["profiled"]
    print(name, "rows", A.n_rows, "nnz", A.nnz, "mean", round(A.nnz / A.n_rows, 1), "uniform", plan.info.uniform,
          "pure us", t, out, flush=True)
    plan.destroy()
