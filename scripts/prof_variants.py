"""ncu target (SURVEY §8d "one profiled rep per variant per config"): every
pool variant's pure full-grid kernel once on D3, D4, D6-random, D6-diagonal,
and every SGEMM tiling once on D2m and 4096^3.  Markers (stdout) give the order."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, d4_powerlaw, d6_diag, d6_random, sgemm_inputs, uniform_f32
ctx = D.Context(0)
for name, A in (("D3", d3_fem()), ("D4", d4_powerlaw()), ("D6r", d6_random()), ("D6d", d6_diag())):
    x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL)
    torch.cuda.synchronize()
    for v in plan.variant_ids:
        ctx.spmv_variant(plan, v, x, y)
        torch.cuda.synchronize()
        print("launch", name, D.SPMV_NAMES[v], flush=True)
    plan.destroy()
for (M, K, N) in ((1024, 992, 1056), (4096, 4096, 4096)):
    Ah, Bh, _ = sgemm_inputs(M, K, N, 5, 6)
    Ad, Bd = torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()
    C = torch.empty((M, N), device="cuda")
    for v in range(4):
        ctx.sgemm_variant(v, Ad, Bd, C)
        torch.cuda.synchronize()
        print("launch", f"{M}x{K}x{N}", D.SGEMM_NAMES[v], flush=True)
