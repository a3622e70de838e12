"""compute-sanitizer driver workload (memcheck / racecheck / synccheck):
small instances of every device path -- the SpMV dispatcher (init,
profiling, claim and switch kernels; SYNC / ASYNC, a non-default winner),
the generic launcher (SGEMM, stencil), the SpMTV swap device path and the
f-2 pools -- each checked against the fp64 oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from oracle import spmv as ospmv
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, d4_powerlaw, sgemm_inputs, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=160_000, lmax=3000)        # 625 units: multi-wave, heavy units, light/heavy order
x = uniform_f32(1, A.n_cols)
xd = torch.from_numpy(x).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
ys, den = ospmv.spmv(A.row_ptr, A.col, A.val, x), ospmv.spmv_abs(A.row_ptr, A.col, A.val, x)
errs = {}
for dflt in (D.SPMV_DEFAULT_AUTO, D.SPMV_CSR_VECTOR, D.SPMV_JDS):
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=dflt)
    for mode in (D.AUTO | D.ASYNC, D.AUTO, D.FULLY | D.ASYNC, D.HYBRID | D.NO_ABORT):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv(plan, xd, y, f=0.05, mode=mode | D.FORCE_PROFILE)
        errs[f"spmv d{dflt} m{mode}"] = ospmv.rel_error(y.cpu().numpy(), ys, den)
    plan.destroy()
# every format (CSR-T's grouped profiling kernel, its host-ordered remainder)
F = d3_fem(grid=300)
xf = uniform_f32(5, F.n_cols)
rpf, colf, valf = (torch.from_numpy(a).cuda() for a in (F.row_ptr, F.col, F.val))
yfs, denf = ospmv.spmv(F.row_ptr, F.col, F.val, xf), ospmv.spmv_abs(F.row_ptr, F.col, F.val, xf)
for dflt in (D.SPMV_ELL, D.SPMV_CSR_TMA):
    pf = ctx.spmv_prepare(rpf, colf, valf, F.n_cols, default=dflt, formats=D.FMT_ALL)
    for mode in (D.FULLY | D.ASYNC, D.FULLY):
        y = torch.full((F.n_rows,), float("nan"), device="cuda")
        ctx.spmv(pf, torch.from_numpy(xf).cuda(), y, f=0.05, mode=mode | D.FORCE_PROFILE)
        errs[f"spmv fmt_all d{dflt} m{mode}"] = ospmv.rel_error(y.cpu().numpy(), yfs, denf)
    pf.destroy()
# row-sharded path on a one-rank communicator (overlapped chunked allgather)
ctx.comm_init(0, 1, D.comm_unique_id())
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
y = torch.full((A.n_rows,), float("nan"), device="cuda")
ctx.spmv_sharded(plan, [0, A.n_rows], xd, y, f=0.05, mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
errs["sharded"] = ospmv.rel_error(y.cpu().numpy(), ys, den)
xt, y0 = uniform_f32(2, A.n_rows), uniform_f32(3, A.n_cols)
yt = torch.from_numpy(y0.copy()).cuda()
ctx.spmtv(plan, torch.from_numpy(xt).cuda(), yt, f=0.05, mode=D.AUTO | D.FORCE_PROFILE)
errs["spmtv swap"] = ospmv.rel_error(yt.cpu().numpy(), ospmv.spmtv(A.row_ptr, A.col, A.val, xt, y0),
                                     ospmv.spmtv_abs(A.row_ptr, A.col, A.val, xt, y0))
y = torch.empty(A.n_rows, device="cuda")
ctx.spmv_placement(plan, xd, y, f=0.1, mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
errs["placement"] = ospmv.rel_error(y.cpu().numpy(), ys, den)
jp = ctx.spmv_jds_prepare(rp, col, val, A.n_cols)
ctx.spmv_jds(jp, xd, y, f=0.1, mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
errs["global jds"] = ospmv.rel_error(y.cpu().numpy(), ys, den)
if not os.environ.get("SANITIZE_SKIP_SGEMM"):   # synccheck: see scripts/mbar_synccheck.cu
    Ah, Bh, C0 = sgemm_inputs(256, 128, 384, 1, 2, 3)
    C = torch.from_numpy(C0.copy()).cuda()
    ctx.sgemm(torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda(), C, f=0.5,
              mode=D.FULLY | D.ASYNC | D.FORCE_PROFILE)
a3 = torch.from_numpy(uniform_f32(4, (66, 12, 96))).cuda()
o3 = torch.empty_like(a3)
ctx.stencil(a3, o3, 0.8, 0.15, f=0.5, mode=D.FULLY | D.ASYNC | D.FORCE_PROFILE)
torch.cuda.synchronize()
print("sanitize workload ok; max err", max(errs.values()), errs)
