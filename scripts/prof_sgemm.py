"""Run one SGEMM variant a few times (for ncu)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import sgemm_inputs
ctx = D.Context(0)
M, K, N = [int(v) for v in os.environ.get("SHAPE", "1024,992,1056").split(",")]
v = int(os.environ.get("V", "2"))
A, B, _ = sgemm_inputs(M, K, N, 1, 2)
Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
C = torch.empty((M, N), device="cuda")
for _ in range(3):
    ctx.sgemm_variant(v, Ad, Bd, C)
torch.cuda.synchronize()
