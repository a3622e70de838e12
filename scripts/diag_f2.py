"""f-2 x-placement pool on D3x: pure variants vs DySel single shot per mode (b2b),
the report timeline, and the default's plain full grid through the same call
(NO_PROFILE) -- where the single-shot time goes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from bench import time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
A = d3_fem(grid=1500)
x = torch.from_numpy(uniform_f32(7, A.n_cols)).cuda()
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
y = torch.empty(A.n_rows, device="cuda")
pl = ctx.spmv_prepare(rp, col, val, A.n_cols)
T = {D.PLACE_NAMES[v]: time_b2b(lambda: ctx.spmv_placement_variant(pl, v, x, y), 10, s) for v in range(4)}
print("pure us", {k: round(v * 1e6, 1) for k, v in T.items()}, flush=True)
for mn, md in (("no_profile", D.NO_PROFILE), ("fully_async", D.FULLY | D.ASYNC), ("fully_sync", D.FULLY),
               ("hybrid_async", D.HYBRID | D.ASYNC), ("auto_async", D.AUTO | D.ASYNC)):
    t = time_b2b(lambda: ctx.spmv_placement(pl, x, y, f=0.02, mode=md), 10, s)
    r = ctx.spmv_placement(pl, x, y, f=0.02, mode=md, report=True)
    print(f"{mn:13s} {t*1e6:8.1f} us sel {r['selected_name']} c {r['c']} eager {r['eager_units']} "
          f"tl_us {[None if v is None else round(v/1e3,1) for v in r['timeline_ns']]}", flush=True)
    print("   pure x_ldg after:", round(time_b2b(lambda: ctx.spmv_placement_variant(pl, 0, x, y), 10, s) * 1e6, 1), flush=True)
