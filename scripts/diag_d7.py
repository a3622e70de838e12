"""D7 (8192^3 SGEMM): pure winner vs the cached-selection (NO_PROFILE) call vs
a profiled FULLY call, interleaved, with the SM clock and throttle reasons
sampled around each group (power capping during long tensor-core runs)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import sgemm_inputs
M = K = N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
Ah, Bh, _ = sgemm_inputs(M, K, N, 8192, 8193)
A, B = torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()
C = torch.empty((M, N), device="cuda")
ctx = D.Context(0)
s = torch.cuda.current_stream()
ctx.sgemm(A, B, C, f=0.005, mode=D.FULLY | D.FORCE_PROFILE)
torch.cuda.synchronize()
fns = {"pure128": lambda: ctx.sgemm_variant(D.SGEMM_T128x128, A, B, C),
       "cached": lambda: ctx.sgemm(A, B, C, mode=D.NO_PROFILE),
       "fully": lambda: ctx.sgemm(A, B, C, f=0.005, mode=D.FULLY),
       "forced": lambda: ctx.sgemm(A, B, C, f=0.005, mode=D.FULLY | D.FORCE_PROFILE)}
print({k: v for k, v in ctx.sgemm(A, B, C, mode=D.NO_PROFILE, report=True).items()
       if k in ("selected_name", "profiled", "mode_used")})
for rnd in range(3):
    for k, fn in fns.items():
        with bench.ClockSampler(0) as cs:
            t = bench.time_b2b(fn, 5, s)
        print(rnd, k, round(t * 1e6, 1), "us", cs.summary(), flush=True)
