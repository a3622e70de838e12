"""SGEMM DySel single-shot per mode (A-32 dominance, A-33 eager wave): 4096^3, D2m, 8192^3."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import sgemm_inputs
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=10):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
sizes = [(4096, 4096, 4096)]
for (M, K, N) in sizes:
    A, B, _ = sgemm_inputs(M, K, N, 5, 6)
    Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    C = torch.empty((M, N), device="cuda")
    pure = {D.SGEMM_NAMES[v]: b2b(lambda: ctx.sgemm_variant(v, Ad, Bd, C), 5) for v in range(4)}
    best = min(pure.values())
    print(f"{M}x{K}x{N} pure_us", {k: round(v, 1) for k, v in pure.items()}, flush=True)
    for name, mode in (("fully_async", D.FULLY | D.ASYNC), ("hybrid_async", D.HYBRID | D.ASYNC)):
        for f in (0.003, 0.005, 0.008, 0.01, 0.02):
            ctx.reset_selection_all() if hasattr(ctx, "reset_selection_all") else None
            t = b2b(lambda: ctx.sgemm(Ad, Bd, C, f=f, mode=mode | D.FORCE_PROFILE), 5)
            r = ctx.sgemm(Ad, Bd, C, f=f, mode=mode | D.FORCE_PROFILE, report=True)
            print(f"  {name:22s} f={f}: {t:8.1f} us  ovh {100 * (t / best - 1):6.1f}%  sel {r['selected_name']:18s} "
                  f"c {r['c']} eager {r['eager_units']} score {[x if x < 2**50 else -1 for x in r['score'][:4]]}", flush=True)
    # parity of the last hybrid async run vs fp64
    ctx.sgemm(Ad, Bd, C, f=0.03, mode=D.HYBRID | D.ASYNC | D.FORCE_PROFILE)
    idx = np.random.default_rng(0).integers(0, M, 64)
    ref = A[idx].astype(np.float64) @ B.astype(np.float64)
    den = np.abs(A[idx]).astype(np.float64) @ np.abs(B).astype(np.float64)
    err = float((np.abs(C.cpu().numpy()[idx] - ref) / den).max())
    print("  sampled-row rel err", err, flush=True)
