"""Pure full-grid runs of one SpMV pool variant for timing or an ncu capture.
env: MATRIX=d4|d3x (default d4), VARIANT=<DYSEL_SPMV_* id> (default: CSR-W
for d4, ELL for d3x), PROF=1 (3 launches, no timing), DYSEL_LIB (A/B build)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, d4_powerlaw, uniform_f32
m = os.environ.get("MATRIX", "d4")
ctx = D.Context(0)
A = d4_powerlaw() if m == "d4" else d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
s = torch.cuda.current_stream()
v = int(os.environ.get("VARIANT", str(D.SPMV_CSR_STREAM if m == "d4" else D.SPMV_ELL)))
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
if os.environ.get("PROF"):
    for _ in range(3):
        flush.zero_()
        ctx.spmv_variant(plan, v, x, y)
    torch.cuda.synchronize()
    sys.exit(0)
ts = []
for _ in range(20):
    flush.zero_()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s); ctx.spmv_variant(plan, v, x, y); b.record(s)
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
nb = 8 * A.nnz + 4 * (A.n_rows + 1) + 4 * A.n_cols + 4 * A.n_rows
t = float(np.median(ts))
print(os.environ.get("DYSEL_LIB", "main"), m, D.SPMV_NAMES[v], round(t, 4), "ms cold", round(nb / t / 1e6, 1), "GB/s",
      flush=True)
