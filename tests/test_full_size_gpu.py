"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (task rule ③): D4 10^7-row power law (sampled rows + bitwise
composition), D3 and D2m in full, SGEMM 4096^3 on sampled rows, the stencil
pool on the 512 x 512 x 64 grid in full and on 512 x 512 x 256 sampled, and the
2.25M-row FEM matrix (D3x, every format) sampled + bitwise composition."""
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


@pytest.mark.parametrize("default", ["ell", "csr_tma"])
def test_d3x_fmt_all_sampled_and_composition(ctx, default):
    """bench.py's 70%-of-HBM config (D3x, 2.25M rows, every format) in its
    launch configuration: grouped profiling (A-49), the switch margin (A-50)
    and — with ELL as the initial version — the host-ordered CSR-T remainder
    (A-42).  Sampled rows vs the oracle and, per unit, bitwise equality with
    the full-grid run of the variant that produced it (c-6)."""
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = d3_fem(grid=1500)
    x = uniform_f32(385, A.n_cols)
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_NAMES.index(default), formats=D.FMT_ALL)
    xd = vec(x)
    rows = np.unique(np.concatenate([np.random.default_rng(2).integers(0, A.n_rows, 20000), [0, A.n_rows - 1]]))
    ys, d = ospmv.spmv_rows(A.row_ptr, A.col, A.val, x, rows)
    unit_of_row = np.arange(A.n_rows) // 256
    pure = {}
    for mode in (D.FULLY | D.ASYNC | D.FORCE_PROFILE, D.FULLY | D.FORCE_PROFILE):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        rep = ctx.spmv(plan, xd, y, f=0.02, mode=mode, report=True, unit_map=True)
        torch.cuda.synchronize()
        assert rep["profiled"]
        yh = y.cpu().numpy()
        assert np.isfinite(yh).all()
        assert ospmv.rel_error(yh[rows], ys, d) <= ospmv.SPMV_TOL
        uv = np.frombuffer(rep["unit_variant"], np.uint8)[:plan.n_units]
        for v in set(uv.tolist()):
            if v not in pure:
                yv = torch.empty_like(y)
                ctx.spmv_variant(plan, v, xd, yv)
                pure[v] = yv.cpu().numpy()
            m = uv[unit_of_row] == v
            assert np.array_equal(yh[m].view(np.uint32), pure[v][m].view(np.uint32)), D.SPMV_NAMES[v]
    plan.destroy()


def test_stencil_512x512x256_sampled(ctx):
    """The bench's ≥ 2 x L2 stencil grid, DySel async (the TMA tile as
    initial version), checked on sampled z-planes against the oracle."""
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    shape = (256, 512, 512)
    a = uniform_f32(64, shape)
    inp = torch.from_numpy(a).cuda()
    out = torch.full_like(inp, float("nan"))
    ctx.stencil(inp, out, 0.8125, 0.15625, f=0.02, mode=D.FULLY | D.ASYNC | D.FORCE_PROFILE)
    o = out.cpu().numpy()
    assert np.isfinite(o).all()
    for z in (0, 1, 15, 16, 17, 63, 64, 127, 128, 200, 254, 255):
        lo, hi = max(0, z - 1), min(shape[0], z + 2)
        sub = a[lo:hi]
        ref = ost.stencil(sub, 0.8125, 0.15625)[z - lo]
        den = ost.stencil_abs(sub, 0.8125, 0.15625)[z - lo]
        if 0 < z < shape[0] - 1:
            assert ost.rel_error(o[z], ref, den) <= ost.STENCIL_TOL, z
        else:
            assert np.array_equal(o[z], a[z]), z
