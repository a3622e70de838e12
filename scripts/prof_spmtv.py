"""One full-grid launch of each SpMTV variant on the 2M-row power-law matrix
(for ncu: `ncu --set full -k regex:spmtv_kernel python scripts/prof_spmtv.py`)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d4_powerlaw, uniform_f32  # noqa: E402

ctx = D.Context(0)
A = d4_powerlaw(n=2_000_000, lmax=4096)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
x = torch.from_numpy(uniform_f32(61, A.n_rows)).cuda()
y = torch.zeros(A.n_cols, device="cuda")
for v in range(len(D.SPMTV_NAMES)):
    ctx.spmtv_variant(plan, v, x, y)
torch.cuda.synchronize()
print("nnz", A.nnz, "algorithmic bytes", 8 * A.nnz + 4 * (A.n_rows + 1) + 4 * A.n_rows + 8 * A.n_cols)
