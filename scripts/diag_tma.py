"""Per-variant pure SpMV times (back-to-back warm, and cold-L2 single) on D3 / D4 / D6: CSR-T A/B."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d4_powerlaw, d3_fem, d6_random, d6_diag, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
def b2b(fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
def cold(fn, n=20):
    ts = []
    for _ in range(n):
        flush.zero_()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    ts.sort(); return ts[len(ts) // 2]
mats = [("d3", d3_fem), ("d6r", d6_random), ("d6d", d6_diag), ("d4", d4_powerlaw)]
if len(sys.argv) > 1: mats = [m for m in mats if m[0] in sys.argv[1:]]
for name, gen in mats:
    A = gen()
    x = torch.from_numpy(uniform_f32(10010, A.n_cols)).cuda()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    y = torch.empty(A.n_rows, device="cuda")
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    out = []
    for v in plan.variant_ids:
        f = lambda: ctx.spmv_variant(plan, v, x, y)
        out.append(f"{D.SPMV_NAMES[v]}: warm {b2b(f, 20 if name == 'd4' else 200):.1f} cold {cold(f, 5 if name == 'd4' else 20):.1f}")
    print(name, A.n_rows, int(A.row_ptr[-1]), "| " + " | ".join(out), flush=True)
    plan.destroy()
