import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import sgemm_inputs
ctx = D.Context(0)
M = K = N = 4096
A, B, _ = sgemm_inputs(M, K, N, 5, 6)
Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
C = torch.empty((M, N), device="cuda")
for mode in (D.FULLY, D.FULLY | D.SCORE_MAKESPAN, D.HYBRID):
    r = ctx.sgemm(Ad, Bd, C, f=0.02, mode=mode, report=True)
    print(mode, r["selected_name"], "c", r["c"], "score", r["score"][:4], "units", r["units"][:4],
          "cycles", r["cycles"][:4], "makespan_us", [m / 1e3 for m in r["makespan_ns"][:4]])
