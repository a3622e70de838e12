"""SGEMM 4096^3 single shot: per-variant profiling makespan / score / aborted
and the timeline, per mode (what bounds the generic launcher's selection)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import sgemm_inputs
M = K = N = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
Ah, Bh, _ = sgemm_inputs(M, K, N, 5, 6)
A, B = torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()
C = torch.empty((M, N), device="cuda")
ctx = D.Context(0)
s = torch.cuda.current_stream()
tp = time_b2b(lambda: ctx.sgemm_variant(3, A, B, C), 5, s)
print("pure tc128", round(tp * 1e6, 1))
for name, mode in (("fully_sync", D.FULLY), ("fully_async", D.FULLY | D.ASYNC), ("hybrid_async", D.HYBRID | D.ASYNC)):
    t = time_b2b(lambda: ctx.sgemm(A, B, C, f=0.01, mode=mode | D.FORCE_PROFILE), 5, s)
    r = ctx.sgemm(A, B, C, f=0.01, mode=mode | D.FORCE_PROFILE, report=True)
    print(name, round(t * 1e6, 1), f"({100 * (t / tp - 1):.1f}%)", r["selected_name"], "c", r["c"], "eager", r["eager_units"],
          "tl_us", [None if v is None else round(v / 1e3, 1) for v in r["timeline_ns"]])
    for v in range(r["n_variants"]):
        print("   ", D.SGEMM_NAMES[v], "makespan_us", round(r["makespan_ns"][v] / 1e3, 1), "units", r["units"][v],
              "aborted", r["aborted"][v], "score", r["score"][v])
