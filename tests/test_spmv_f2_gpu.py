"""GPU parity of the f-2 pools through the C ABI:
Case II x data placement and Case III global-sort JDS
versions.  Every variant of both pools sums
each row in CSR order with fmaf from +0, so all are bit-identical to the main
pool's CSR-S; DySel launches compose bitwise (c-6) and match the fp64 oracle."""
import numpy as np
import pytest

from gpu_helpers import spmv_err, to_dev, vec
from oracle import formats
from oracle.spmv import SPMV_TOL
from workloads import CSR, d3_fem, d4_powerlaw, d6_diag, random_lengths_csr, small_int_csr, small_int_vector, uniform_f32

pytestmark = pytest.mark.gpu

MATS = {
    "d3small": lambda: d3_fem(grid=160),             # banded: x windows fit shared memory
    "ragged": lambda: random_lengths_csr(7001, 5000, 120, 4, empty_frac=0.1),
    "powerlaw": lambda: d4_powerlaw(n=80_000, lmax=3000),
    "diag": lambda: d6_diag(n=100_000),
}


@pytest.fixture(scope="module")
def D():
    from paper_conf_asplos_changkh16_b200 import dysel
    return dysel


@pytest.fixture(scope="module")
def ctx(gpu, D):
    c = D.Context(0)
    yield c
    c.close()


def csr_s(ctx, A, xd):
    import torch
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=0)
    y = torch.empty(A.n_rows, device="cuda")
    ctx.spmv_variant(plan, 0, xd, y)
    return plan, y.cpu().numpy().view(np.uint32), (rp, col, val)


@pytest.mark.parametrize("name", list(MATS))
def test_placement_variants_bit_identical(ctx, D, name):
    import torch
    A = MATS[name]()
    x = uniform_f32(21, A.n_cols)
    xd = vec(x)
    plan, ref, _ = csr_s(ctx, A, xd)
    for v in range(4):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv_placement_variant(plan, v, xd, y)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().view(np.uint32), ref), D.PLACE_NAMES[v]
    assert spmv_err(A, x, y) <= SPMV_TOL
    # per-unit x windows: bit-exact vs the oracle's definition
    assert np.array_equal(ctx.spmv_placement_windows(plan), formats.unit_x_windows(A.row_ptr, A.col))
    plan.destroy()


@pytest.mark.parametrize("mode_name", ["fully_sync", "fully_async", "hybrid_async", "auto_async", "fully_host"])
def test_placement_dysel_composition(ctx, D, mode_name):
    import torch
    A = MATS["d3small"]() if "auto" not in mode_name else MATS["ragged"]()
    mode = {"fully_sync": D.FULLY, "fully_async": D.FULLY | D.ASYNC, "hybrid_async": D.HYBRID | D.ASYNC,
            "auto_async": D.AUTO | D.ASYNC, "fully_host": D.FULLY | D.HOST_ORCH}[mode_name] | D.FORCE_PROFILE
    x = uniform_f32(22, A.n_cols)
    xd = vec(x)
    plan, ref, _ = csr_s(ctx, A, xd)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    rep = ctx.spmv_placement(plan, xd, y, f=0.1, mode=mode, report=True)
    torch.cuda.synchronize()
    assert rep["profiled"] and 0 <= rep["selected"] < 4
    assert np.array_equal(y.cpu().numpy().view(np.uint32), ref)
    plan.destroy()


def test_placement_small_integer_and_unaligned_x(ctx, D):
    import torch
    A = small_int_csr(MATS["d3small"](), 5)
    x = small_int_vector(A.n_cols, 6)
    xs = torch.empty(A.n_cols + 1, device="cuda")[1:]     # x not 16-byte aligned: the bulk copy must not need it
    xs.copy_(vec(x))
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    from oracle import spmv as ospmv
    ys = ospmv.spmv(A.row_ptr, A.col, A.val, x)
    for v in range(4):
        y = torch.empty(A.n_rows, device="cuda")
        ctx.spmv_placement_variant(plan, v, xs, y)
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ys), v
    plan.destroy()


def jds_plan(ctx, A):
    rp, col, val = to_dev(A)
    return ctx.spmv_jds_prepare(rp, col, val, A.n_cols), (rp, col, val)


@pytest.mark.parametrize("name", list(MATS) + ["empty_rows"])
def test_global_jds_format_bit_exact_and_variants(ctx, D, name):
    import torch
    if name == "empty_rows":
        A = random_lengths_csr(3000, 900, 10, 9, empty_frac=0.5)
    else:
        A = MATS[name]()
    jp, keep = jds_plan(ctx, A)
    j = formats.csr_to_global_jds_fast(A.row_ptr, A.col, A.val)
    for k in ("perm", "len", "jd_ptr", "col"):
        assert np.array_equal(jp.array(k), j[k]), k
    assert np.array_equal(jp.array("val").view(np.uint32), j["val"].view(np.uint32))
    x = uniform_f32(23, A.n_cols)
    xd = vec(x)
    _, ref, _ = csr_s(ctx, A, xd)
    for v in range(4):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv_jds_variant(jp, v, xd, y)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().view(np.uint32), ref), D.JDSG_NAMES[v]
    assert spmv_err(A, x, y) <= SPMV_TOL
    jp.destroy()


@pytest.mark.parametrize("mode_name", ["auto_sync", "auto_async", "fully_async", "hybrid_host"])
def test_global_jds_dysel_composition(ctx, D, mode_name):
    import torch
    A = MATS["powerlaw"]()
    mode = {"auto_sync": D.AUTO, "auto_async": D.AUTO | D.ASYNC, "fully_async": D.FULLY | D.ASYNC,
            "hybrid_host": D.HYBRID | D.HOST_ORCH}[mode_name] | D.FORCE_PROFILE
    jp, keep = jds_plan(ctx, A)
    x = uniform_f32(24, A.n_cols)
    xd = vec(x)
    _, ref, _ = csr_s(ctx, A, xd)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    rep = ctx.spmv_jds(jp, xd, y, f=0.1, mode=mode, report=True)
    torch.cuda.synchronize()
    assert rep["profiled"] and 0 <= rep["selected"] < 4
    assert np.array_equal(y.cpu().numpy().view(np.uint32), ref)
    jp.destroy()


def test_global_jds_edge_cases(ctx, D):
    import torch
    E = CSR(500, 500, np.zeros(501, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    jp, keep = jds_plan(ctx, E)
    y = torch.full((500,), 3.0, device="cuda")
    ctx.spmv_jds(jp, vec(np.ones(500)), y, f=0.5, mode=D.FULLY | D.FORCE_PROFILE)
    assert torch.count_nonzero(y).item() == 0
    jp.destroy()
