"""Interleaved A/B of generic-launcher single shots (stencil 512^2 x {64,256},
SGEMM 4096^3) across library builds: DYSEL_LIBS=a.so,b.so; each round times
every lib's pure best variant and DySel modes back to back (fresh process per
lib is not needed: each lib gets its own ctypes handle)."""
import ctypes, importlib, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import time_b2b
from workloads import sgemm_inputs, uniform_f32
libs = os.environ.get("DYSEL_LIBS", "").split(",")
mods = []
for l in libs:
    os.environ["DYSEL_LIB"] = l
    import paper_conf_asplos_changkh16_b200.dysel as D
    D = importlib.reload(D)
    mods.append((os.path.basename(l) or "main", D, D.Context(0)))
s = torch.cuda.current_stream()
cases = []
for nz in (64, 256):
    a = torch.from_numpy(uniform_f32(64, (nz, 512, 512))).cuda(); o = torch.empty_like(a)
    cases.append((f"stencil{nz}", lambda D, c, md, a=a, o=o: c.stencil(a, o, 0.8, 0.15, f=0.02, mode=md),
                  lambda D, c, a=a, o=o: c.stencil_variant(2, a, o, 0.8, 0.15)))
Ah, Bh, _ = sgemm_inputs(4096, 4096, 4096, 5, 6)
A, B = torch.from_numpy(Ah).cuda(), torch.from_numpy(Bh).cuda()
C = torch.empty((4096, 4096), device="cuda")
cases.append(("sgemm4096", lambda D, c, md: c.sgemm(A, B, C, f=0.01, mode=md), lambda D, c: c.sgemm_variant(3, A, B, C)))
for rnd in range(2):
    for name, run, pure in cases:
        for tag, D, c in mods:
            modes = {"fully_async": D.FULLY | D.ASYNC | D.FORCE_PROFILE, "hybrid_async": D.HYBRID | D.ASYNC | D.FORCE_PROFILE,
                     "fully_sync": D.FULLY | D.FORCE_PROFILE}
            tp = time_b2b(lambda: pure(D, c), 5 if "sgemm" in name else 10, s)
            r = {m: round((time_b2b(lambda: run(D, c, md), 5 if "sgemm" in name else 10, s) / tp - 1) * 100, 1)
                 for m, md in modes.items()}
            print(rnd, name, tag, "pure_us", round(tp * 1e6, 1), "ovh%", r, flush=True)
