"""TMA gather4 probe (flavour 2/3) vs the LSU gather probe (flavour 0) on D4:
verify the gathered values (flavour 3), then time each flavour with events
around single launches (the flavour-2 call synchronises internally)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, uniform_f32
ctx = D.Context(0)
A = d4_powerlaw()
x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=4)
s = torch.cuda.current_stream()
try:
    ctx.spmv_gather_probe(plan, 3, x, y)
    print("verify flavour 3: OK", flush=True)
except Exception as e:
    print("verify flavour 3 FAILED:", e, flush=True)
def one(fl):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize()
    a.record(s)
    ctx.spmv_gather_probe(plan, fl, x, y)
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3
for fl in (0, 2, 4, 0, 2, 4, 1):
    try:
        ts = sorted(one(fl) for _ in range(7))
        print(f"flavour {fl}: median {ts[3]:.1f} us (min {ts[0]:.1f})", flush=True)
    except Exception as e:
        print(f"flavour {fl} failed: {e}", flush=True)
a, b = torch.cuda.Event(True), torch.cuda.Event(True)
a.record(s); ctx.spmv_variant(plan, 4, x, y); b.record(s); torch.cuda.synchronize()
print(f"csr_stream single launch {a.elapsed_time(b)*1e3:.1f} us", flush=True)
