import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
ctx = D.Context(0)
np.set_printoptions(linewidth=200, precision=2, suppress=True)
M, K, N = 128, 32, 64
rng = np.random.default_rng(0)
def run(A, B, v=2):
    C = torch.zeros((M, N), device="cuda")
    ctx.sgemm_variant(v, torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda(), C)
    return C.cpu().numpy()
# (a) A = identity on the first 32 rows -> C[:32] = B
A = np.zeros((M, K), np.float32); A[np.arange(32), np.arange(32)] = 1
B = (np.arange(K * N).reshape(K, N) % 97).astype(np.float32)
C = run(A, B); ref = A @ B
print("a: ok", np.array_equal(C, ref))
if not np.array_equal(C, ref):
    bad = np.argwhere(C != ref); print("a bad count", len(bad), "first", bad[:10])
    for r in range(4): print("row", r, "got", C[r, :16], "\n      want", ref[r, :16])
    # which B element landed where: find positions of C values in B
    for (i, j) in bad[:6]:
        w = np.argwhere(B == C[i, j]); print((i, j), "got B at", w[:3])
# (b) B = identity on the first 32 cols -> C[:, :32] = A
A = (np.arange(M * K).reshape(M, K) % 89).astype(np.float32)
B = np.zeros((K, N), np.float32); B[np.arange(32), np.arange(32)] = 1
C = run(A, B); ref = A @ B
print("b: ok", np.array_equal(C, ref))
if not np.array_equal(C, ref):
    bad = np.argwhere(C != ref); print("b bad count", len(bad), "first", bad[:10])
    for r in range(3): print("row", r, "got", C[r, :16], "\n      want", ref[r, :16])
    for (i, j) in bad[:6]:
        w = np.argwhere(A == C[i, j]); print((i, j), "got A at", w[:3])
