"""Host vs device (fire-and-forget / tail) launch of a full SpMV grid on D4."""
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
def b2b(step, n=20):
    for _ in range(3): step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): step()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n
ref = None
for v in (1, 4):
    for how in (0, 1, 2):
        t = b2b(lambda: ctx.debug_spmv_device_launch(plan, v, x, y, how))
        yy = y.clone()
        if how == 0: ref = yy
        print(D.SPMV_NAMES[v], ["host", "device_ff", "device_tail"][how], f"{t:.4f} ms", "same" if torch.equal(ref, yy) else "DIFF", flush=True)
import collections
for v in (1, 4):
    for how in (0, 1):
        r = ctx.debug_spmv_device_launch(plan, v, x, y, how, resident=True)
        print(D.SPMV_NAMES[v], ["host", "device_ff"][how], "max resident CTAs/SM histogram", dict(collections.Counter(r)))
