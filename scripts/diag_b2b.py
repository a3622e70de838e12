"""Why b2b step time != per-step events: the bench preamble, then repeated
b2b regions with / without the nvidia-smi clock sampler, and per-step events."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
A, x = bench.make_d4(10_000_000)
ctx = D.Context(0)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
xd = torch.from_numpy(x).cuda()
y = torch.empty(A.n_rows, device="cuda")
plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
s = torch.cuda.current_stream()
step = lambda: ctx.spmv(plan, xd, y, f=0.001, mode=D.AUTO | D.ASYNC)
for v in plan.variant_ids:
    print("pure", D.SPMV_NAMES[v], round(bench.time_b2b(lambda: ctx.spmv_variant(plan, v, xd, y), 15, s) * 1e3, 4))
for _ in range(5):
    step()
torch.cuda.synchronize()
def region(n=20):
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n):
        step()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n
for i in range(3):
    with bench.ClockSampler(0):
        torch.cuda.synchronize()
        t1 = region()
    t2 = region()
    pe = bench.time_events(step, 20, s)
    print(f"round {i}: b2b+sampler {t1:.4f} b2b {t2:.4f} per-step mean {np.mean(pe)*1e3:.4f} max {np.max(pe)*1e3:.4f}",
          flush=True)
