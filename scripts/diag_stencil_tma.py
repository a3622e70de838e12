"""V2 (TMA tile) pure b2b times on 512x512x{64,256}, 3 repeats each, plus the
pool's other variants once (A/B across builds via DYSEL_LIB)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import uniform_f32
ctx = D.Context(0)
s = torch.cuda.current_stream()
out = []
for nz in (64, 256, 512):
    a = torch.from_numpy(uniform_f32(1, (nz, 512, 512))).cuda()
    o = torch.empty_like(a)
    t = [bench.time_b2b(lambda: ctx.stencil_variant(2, a, o, 0.8, 0.15), 30, s) * 1e6 for _ in range(3)]
    out.append(f"nz={nz}: " + " ".join(f"{x:.1f}" for x in t) + f" us ({8 * a.numel() / min(t) / 1e3:.0f} GB/s)")
    del a, o
print(os.path.basename(D.LIB_PATH), " | ".join(out), flush=True)
