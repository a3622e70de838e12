"""SGEMM variant timings + parity spot check on D2m / D7-like shapes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from oracle import sgemm as osg
from workloads import sgemm_inputs
ctx = D.Context(0)
s = torch.cuda.current_stream()
def ev(fn, reps=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(s); fn(); b.record(s); torch.cuda.synchronize(); out.append(a.elapsed_time(b))
    return float(np.median(out)) * 1e-3
for (M, K, N) in [(1024, 992, 1056), (4096, 4096, 4096)]:
    A, B, C0 = sgemm_inputs(M, K, N, 1, 2, 3)
    Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    C = torch.empty((M, N), device="cuda")
    fl = 2.0 * M * N * K
    for v in range(4):
        t = ev(lambda: ctx.sgemm_variant(v, Ad, Bd, C))
        line = f"{M}x{K}x{N} {D.SGEMM_NAMES[v]:18s} {t*1e6:9.1f} us {fl/t/1e12:7.1f} TFLOP/s"
        if M <= 1024:
            ref = osg.sgemm(A, B, C0, 1.0, 0.0); d = osg.sgemm_abs(A, B, C0, 1.0, 0.0)
            line += f"  err {float((np.abs(C.cpu().numpy() - ref) / d).max()):.2e}"
        print(line, flush=True)
