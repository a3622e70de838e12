"""Stencil pool pure times (b2b) on 512x512x64 and 256x256x256."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
def b2b(fn, n=50):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record(s)
    for _ in range(n): fn()
    b.record(s); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3
for shape in ((64, 512, 512), (256, 512, 512)):
    a = torch.from_numpy(uniform_f32(1, shape)).cuda(); o = torch.empty_like(a)
    nb = 8 * a.numel()
    r = {D.STENCIL_NAMES[v]: b2b(lambda: ctx.stencil_variant(v, a, o, 0.8, 0.15)) for v in range(3)}
    t = b2b(lambda: ctx.stencil(a, o, 0.8, 0.15, f=0.02, mode=D.FULLY | D.ASYNC))
    print(shape, {k: f"{v:.1f}us {nb / v / 1e3:.0f}GB/s" for k, v in r.items()}, f"dysel {t:.1f}us", flush=True)
    for m, mn in ((D.FULLY, "fully"), (D.FULLY | D.ASYNC, "fully_async")):
        rep = ctx.stencil(a, o, 0.8, 0.15, f=0.02, mode=m | D.FORCE_PROFILE, report=True)
        print("  ", mn, rep["selected_name"], "c", rep["c"], "score", rep["score"][:3], "units", rep["units"][:3],
              "busy_us", [round(b / 1e3, 1) for b in rep["busy_ns"][:3]], flush=True)
