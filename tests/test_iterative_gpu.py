"""GPU parity of the iterative driver (dysel_spmv_power) vs the
fp64 power-iteration oracle, through the C ABI."""
import numpy as np
import pytest

from oracle import iterative
from workloads import d4_powerlaw, laplacian_2d, random_lengths_csr, uniform_f32

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx(gpu):
    from paper_conf_asplos_changkh16_b200 import dysel
    c = dysel.Context(0)
    yield c
    c.close()


def _dev(A):
    import torch
    return (torch.from_numpy(A.row_ptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda())


@pytest.mark.parametrize("profile_every", [0, 1, 7])
def test_power_iteration_parity(ctx, profile_every):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    N, iters = 96, 40                       # 9216 rows = 36 units: profiling forced on
    A = laplacian_2d(N)
    x0 = uniform_f32(11, A.n_cols, 0.0, 1.0)
    rp, col, val = _dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, formats=D.FMT_ALL, default=D.SPMV_CSR_VECTOR)
    x = torch.from_numpy(x0.copy()).cuda()
    y = torch.empty_like(x)
    norms = torch.zeros(iters, dtype=torch.float64, device="cuda")
    rep = ctx.spmv_power(plan, x, y, iters, profile_every=profile_every, f=0.5,
                         mode=D.FULLY | D.ASYNC | D.FORCE_PROFILE, norms=norms, report=True)
    torch.cuda.synchronize()
    assert rep["profiled"]
    xo, yo, no = iterative.power_iteration(A.row_ptr, A.col, A.val, x0, iters)
    ng = norms.cpu().numpy()
    assert np.max(np.abs(ng - no) / no) <= 1e-5
    assert np.max(np.abs(x.cpu().numpy() - xo)) <= 3e-5 * np.abs(xo).max()
    assert np.max(np.abs(y.cpu().numpy() - yo)) <= 3e-5 * np.abs(yo).max()
    plan.destroy()


def test_profile_every_controls_profiling(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = d4_powerlaw(n=200_000, lmax=4096)
    rp, col, val = _dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
    x = torch.from_numpy(uniform_f32(12, A.n_cols)).cuda()
    y = torch.empty_like(x)
    counts = {}
    for pe in (0, 1):
        n0 = ctx.kernel_launches()
        ctx.spmv_power(plan, x, y, 10, profile_every=pe, f=0.05, mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
        torch.cuda.synchronize()
        counts[pe] = ctx.kernel_launches() - n0
    # profiling iterations launch the init + profiling + K claim kernels; the
    # activation-flag-off iterations one plain kernel (+2 norm kernels each)
    assert counts[1] > counts[0]
    assert np.isfinite(x.cpu().numpy()).all()
    plan.destroy()


def test_power_iteration_rejects_rectangular(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = random_lengths_csr(300, 500, 20, 3)
    rp, col, val = _dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    x = torch.zeros(500, device="cuda")
    y = torch.zeros(300, device="cuda")
    with pytest.raises(Exception):
        ctx.spmv_power(plan, x, y, 3)
    plan.destroy()
