"""Plain grid vs claim kernel paths (pure / remainder preset / all-eager) on D4, back to back."""
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
def b2b(fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
for rep in range(2):
    for v in (4, 1):
        r = [f"pure={b2b(lambda: ctx.spmv_variant(plan, v, x, y)):.1f}"]
        for how in (0, 3, 4):
            r.append(f"{['plain', 'ff', 'tail', 'claim_rem', 'claim_eager'][how]}={b2b(lambda: ctx.debug_spmv_device_launch(plan, v, x, y, how)):.1f}")
        print(D.SPMV_NAMES[v], " ".join(r), flush=True)
