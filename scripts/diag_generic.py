"""Single-shot anatomy of the generic launcher's device path (SGEMM, stencil,
f-2 pools): pure times vs DySel single shot per mode, with the report's
publish time, scores, aborted CTAs and host time."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from bench import time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import d3_fem, sgemm_inputs, uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def show(name, T, run, modes):
    best = min(T.values())
    print(name, "pure us", {k: round(v * 1e6, 1) for k, v in T.items()}, flush=True)
    for mn, md in modes:
        t = time_b2b(lambda: run(md, False), 10, s)
        r = run(md, True)
        print(f"  {mn:14s} {t*1e6:8.1f} us ovh {100*(t/best-1):6.1f}% sel {r['selected_name']} c {r['c']} "
              f"publish_us {None if r['timeline_ns'][1] is None else round(r['timeline_ns'][1]/1e3,1)} "
              f"aborted {r['aborted'][:r['n_variants']]} units {r['units'][:r['n_variants']]} "
              f"eager {r['eager_units']} tl_us {[None if v is None else round(v/1e3,1) for v in r['timeline_ns']]}", flush=True)
modes = [("fully_sync", D.FULLY | D.FORCE_PROFILE), ("fully_async", D.FULLY | D.ASYNC | D.FORCE_PROFILE),
         ("hybrid_async", D.HYBRID | D.ASYNC | D.FORCE_PROFILE), ("no_abort", D.FULLY | D.NO_ABORT | D.FORCE_PROFILE)]
ONLY = sys.argv[1] if len(sys.argv) > 1 else None   # stencil | f2 | sgemm
for nz in (64, 256):
    if ONLY not in (None, "stencil"):
        break
    a3 = torch.from_numpy(uniform_f32(64, (nz, 512, 512))).cuda(); o3 = torch.empty_like(a3)
    T = {D.STENCIL_NAMES[v]: time_b2b(lambda: ctx.stencil_variant(v, a3, o3, 0.8, 0.15), 10, s) for v in range(3)}
    show(f"stencil 512x512x{nz}", T, lambda md, rep: ctx.stencil(a3, o3, 0.8, 0.15, f=0.02, mode=md, report=rep),
         modes)
    del a3, o3
if ONLY == "stencil":
    sys.exit(0)
if ONLY != "sgemm":
  A = d3_fem(grid=1500)
  x = torch.from_numpy(uniform_f32(7, A.n_cols)).cuda()
  rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
  y = torch.empty(A.n_rows, device="cuda")
  pl = ctx.spmv_prepare(rp, col, val, A.n_cols)
  T = {D.PLACE_NAMES[v]: time_b2b(lambda: ctx.spmv_placement_variant(pl, v, x, y), 10, s) for v in range(4)}
  show("placement d3x", T, lambda md, rep: ctx.spmv_placement(pl, x, y, f=0.02, mode=md, report=rep), modes)
  jp = ctx.spmv_jds_prepare(rp, col, val, A.n_cols)
  T = {D.JDSG_NAMES[v]: time_b2b(lambda: ctx.spmv_jds_variant(jp, v, x, y), 10, s) for v in range(4)}
  show("global jds d3x", T, lambda md, rep: ctx.spmv_jds(jp, x, y, f=0.02, mode=md, report=rep), modes)
M = K = N = 4096
Ah, Bh, _ = sgemm_inputs(M, K, N, 5, 6)
Ad, Bd = torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()
C = torch.empty((M, N), device="cuda")
T = {D.SGEMM_NAMES[v]: time_b2b(lambda: ctx.sgemm_variant(v, Ad, Bd, C), 5, s) for v in (1, 2, 3)}
show("sgemm 4096", T, lambda md, rep: ctx.sgemm(Ad, Bd, C, f=0.01, mode=md, report=rep), modes)
