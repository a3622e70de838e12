"""Pure CSR-W (the D4 winner) full-grid runs on D4: b2b timing, or a few
launches for an ncu capture (PROF=1).  Library from DYSEL_LIB (A/B builds)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw(n=int(os.environ.get("ROWS", "10000000")))
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
s = torch.cuda.current_stream()
v = int(os.environ.get("VARIANT", str(D.SPMV_CSR_STREAM)))
if os.environ.get("PROF"):
    for _ in range(3):
        ctx.spmv_variant(plan, v, x, y)
    torch.cuda.synchronize()
    sys.exit(0)
for _ in range(5):
    ctx.spmv_variant(plan, v, x, y)
torch.cuda.synchronize()
a, b = torch.cuda.Event(True), torch.cuda.Event(True)
a.record(s)
for _ in range(30):
    ctx.spmv_variant(plan, v, x, y)
b.record(s)
torch.cuda.synchronize()
print(os.environ.get("DYSEL_LIB", "main"), D.SPMV_NAMES[v], round(a.elapsed_time(b) / 30, 4), "ms", flush=True)
