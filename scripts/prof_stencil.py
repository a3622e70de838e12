"""One full-grid launch of each stencil variant on 512x512x256 (for ncu:
ncu -k regex:stencil --set full ... python scripts/prof_stencil.py [variant])."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import uniform_f32
ctx = D.Context(0)
nz = int(os.environ.get("NZ", "256"))
a = torch.from_numpy(uniform_f32(1, (nz, 512, 512))).cuda()
o = torch.empty_like(a)
vs = [int(sys.argv[1])] if len(sys.argv) > 1 else range(3)
for v in vs:
    ctx.stencil_variant(v, a, o, 0.8, 0.15)
torch.cuda.synchronize()
print("done")
