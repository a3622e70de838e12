"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (task rule ③): D4 10^7-row power law (sampled rows + bitwise
composition), D3 and D2m in full, SGEMM 4096^3 on sampled rows, the stencil
pool on the 512 x 512 x 64 grid in full."""
import numpy as np
import pytest

from gpu_helpers import to_dev, vec
from oracle import sgemm as osg
from oracle import spmv as ospmv
from oracle import stencil as ost
from workloads import d3_fem, d4_powerlaw, sgemm_inputs, uniform_f32

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx(gpu):
    from paper_conf_asplos_changkh16_b200 import dysel
    c = dysel.Context(0)
    yield c
    c.close()


def test_d4_full_size_sampled_and_composition(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = d4_powerlaw()
    x = uniform_f32(10010, A.n_cols)
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)   # bench.py's pool
    xd = vec(x)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    rep = ctx.spmv(plan, xd, y, f=0.001, mode=D.AUTO | D.ASYNC, report=True, unit_map=True)   # bench.py's step
    torch.cuda.synchronize()
    assert rep["profiled"]
    yh = y.cpu().numpy()
    assert np.isfinite(yh).all()
    lens = np.diff(A.row_ptr.astype(np.int64))
    g = np.random.default_rng(0)
    rows = np.unique(np.concatenate([g.integers(0, A.n_rows, 20000), np.argsort(lens)[-40:],
                                     [0, A.n_rows - 1]]))
    ys, d = ospmv.spmv_rows(A.row_ptr, A.col, A.val, x, rows)
    assert ospmv.rel_error(yh[rows], ys, d) <= ospmv.SPMV_TOL
    # c-6 at full size: every unit equals, bitwise, the full-grid run of the
    # variant that produced it
    uv = np.frombuffer(rep["unit_variant"], np.uint8)[:plan.n_units]
    unit_of_row = np.arange(A.n_rows) // 256
    for v in set(uv.tolist()):
        yv = torch.empty_like(y)
        ctx.spmv_variant(plan, v, xd, yv)
        m = uv[unit_of_row] == v
        assert np.array_equal(yh[m].view(np.uint32), yv.cpu().numpy()[m].view(np.uint32)), D.SPMV_NAMES[v]
    plan.destroy()


def test_d3_full_size(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = d3_fem()
    x = uniform_f32(384, A.n_cols)
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ALL)
    ys, d = ospmv.spmv(A.row_ptr, A.col, A.val, x), ospmv.spmv_abs(A.row_ptr, A.col, A.val, x)
    for mode in (D.AUTO | D.ASYNC, D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.FULLY | D.FORCE_PROFILE):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv(plan, vec(x), y, f=0.02, mode=mode)
        assert ospmv.rel_error(y.cpu().numpy(), ys, d) <= ospmv.SPMV_TOL, mode
    plan.destroy()


def test_d2m_full_size(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    M, K, N = 1024, 992, 1056
    A, B, C0 = sgemm_inputs(M, K, N, 992, 993, 994)
    ref = osg.sgemm(A, B, C0, 1.5, -0.5)
    den = osg.sgemm_abs(A, B, C0, 1.5, -0.5)
    for mode in (D.FULLY, D.FULLY | D.FORCE_PROFILE, D.HYBRID | D.ASYNC | D.FORCE_PROFILE):
        C = torch.from_numpy(C0.copy()).cuda()
        ctx.sgemm(torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda(), C, 1.5, -0.5, f=0.06, mode=mode)
        assert float((np.abs(C.cpu().numpy() - ref) / den).max()) <= osg.SGEMM_TOL, mode


def test_sgemm_4096_sampled(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    M = K = N = 4096
    A, B, _ = sgemm_inputs(M, K, N, 5, 6)
    C = torch.empty((M, N), device="cuda")
    ctx.sgemm(torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda(), C, f=0.02, mode=D.FULLY)
    rows = np.random.default_rng(1).integers(0, M, 48)
    A64, B64 = A[rows].astype(np.float64), B.astype(np.float64)
    ref = A64 @ B64
    den = np.abs(A64) @ np.abs(B64)
    assert float((np.abs(C.cpu().numpy()[rows] - ref) / den).max()) <= osg.SGEMM_TOL


def test_stencil_full_size(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    shape = (64, 512, 512)
    a = uniform_f32(64, shape)
    ref, den = ost.stencil(a, 0.8125, 0.15625), ost.stencil_abs(a, 0.8125, 0.15625)
    inp = torch.from_numpy(a).cuda()
    for mode in (D.FULLY | D.ASYNC, D.FULLY | D.ASYNC | D.FORCE_PROFILE):
        out = torch.full_like(inp, float("nan"))
        ctx.stencil(inp, out, 0.8125, 0.15625, f=0.02, mode=mode)
        assert ost.rel_error(out.cpu().numpy(), ref, den) <= ost.STENCIL_TOL, mode
