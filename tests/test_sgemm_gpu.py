"""GPU parity of the SGEMM variants and DySel SGEMM vs the fp64 oracle (c-2, c-6)."""
import numpy as np
import pytest

from oracle import sgemm as osg
from workloads import sgemm_inputs, small_int_gemm

pytestmark = pytest.mark.gpu

SHAPES = [(128, 96, 160), (200, 77, 131), (1, 1, 1), (130, 1024, 70), (1024, 992, 1056)]


@pytest.fixture(scope="module")
def ctx(gpu):
    from paper_conf_asplos_changkh16_b200 import dysel
    c = dysel.Context(0)
    yield c
    c.close()


@pytest.fixture(scope="module")
def D():
    from paper_conf_asplos_changkh16_b200 import dysel
    return dysel


def dev(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def err(A, B, C0, alpha, beta, C):
    ref = osg.sgemm(A, B, C0, alpha, beta)
    d = osg.sgemm_abs(A, B, C0, alpha, beta)
    diff = np.abs(C.astype(np.float64) - ref)
    with np.errstate(invalid="ignore", divide="ignore"):
        e = np.where(diff == 0, 0.0, diff / d)
    return float(np.nan_to_num(e, nan=np.inf).max())


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("v", range(4))
def test_variant_parity(ctx, D, shape, v):
    M, K, N = shape
    A, B, C0 = sgemm_inputs(M, K, N, 1, 2, 3)
    C = dev(C0.copy())
    ctx.sgemm_variant(v, dev(A), dev(B), C, alpha=1.5, beta=-0.5)
    assert err(A, B, C0, 1.5, -0.5, C.cpu().numpy()) <= osg.SGEMM_TOL, D.SGEMM_NAMES[v]


@pytest.mark.parametrize("v", range(4))
def test_small_integer_bit_exact(ctx, v):
    A, B, C0 = small_int_gemm(192, 1024, 160, 4)     # |sums| < 2^24, exact in tf32 (hi = a, lo = 0)
    C = dev(C0.copy())
    ctx.sgemm_variant(v, dev(A), dev(B), C, alpha=1.0, beta=1.0)
    ref = A.astype(np.int64) @ B.astype(np.int64) + C0.astype(np.int64)
    assert np.array_equal(C.cpu().numpy().astype(np.int64), ref)


def test_beta_zero_ignores_c(ctx):
    A, B, _ = sgemm_inputs(64, 32, 64, 5, 6)
    for v in range(4):
        C = dev(np.full((64, 64), np.nan, np.float32))
        ctx.sgemm_variant(v, dev(A), dev(B), C, alpha=1.0, beta=0.0)
        assert np.isfinite(C.cpu().numpy()).all()


def test_k_zero(ctx):
    import torch
    A = torch.zeros((40, 0), device="cuda")
    B = torch.zeros((0, 50), device="cuda")
    C0 = np.random.default_rng(0).standard_normal((40, 50)).astype(np.float32)
    for v in range(4):
        C = dev(C0.copy())
        ctx.sgemm_variant(v, A, B, C, alpha=1.0, beta=2.0)
        assert np.allclose(C.cpu().numpy(), 2.0 * C0)


@pytest.mark.parametrize("mode_name", ["fully_sync", "fully_host_sync", "fully_host_async", "hybrid_sync",
                                       "fully_async", "hybrid_async", "fully_sync_noabort"])
def test_dysel_sgemm_composition(ctx, D, mode_name):
    M, K, N = 1024, 992, 1056
    A, B, C0 = sgemm_inputs(M, K, N, 992, 993, 994)
    Ad, Bd = dev(A), dev(B)
    full = {}
    for v in range(4):
        C = dev(C0.copy())
        ctx.sgemm_variant(v, Ad, Bd, C, alpha=1.5, beta=-0.5)
        full[v] = C.cpu().numpy().view(np.uint32)
    mode = D.FORCE_PROFILE | (D.HYBRID if "hybrid" in mode_name else D.FULLY)
    mode |= D.HOST_ORCH if "host" in mode_name else 0
    mode |= D.ASYNC if "async" in mode_name else 0
    mode |= D.NO_ABORT if "noabort" in mode_name else 0
    C = dev(C0.copy())
    rep = ctx.sgemm(Ad, Bd, C, alpha=1.5, beta=-0.5, f=0.3, mode=mode, report=True, unit_map=True)
    Ch = C.cpu().numpy()
    assert rep["profiled"] and rep["selected"] in range(4)
    assert err(A, B, C0, 1.5, -0.5, Ch) <= osg.SGEMM_TOL
    uv = rep["unit_variant"]
    Gx = (N + 127) // 128
    Cu = Ch.view(np.uint32)
    for j in range(rep["n_granules"]):
        gy, gx = divmod(j, Gx)
        blk = (slice(gy * 128, min(M, gy * 128 + 128)), slice(gx * 128, min(N, gx * 128 + 128)))
        assert np.array_equal(Cu[blk], full[uv[j]][blk]), (j, uv[j])


def test_dysel_sgemm_deactivated_small(ctx, D):
    M, K, N = 128, 96, 160      # Parboil small: 6 CTAs < 128
    A, B, C0 = sgemm_inputs(M, K, N, 96, 97)
    C = dev(C0.copy())
    rep = ctx.sgemm(dev(A), dev(B), C, f=0.02, report=True)
    assert not rep["profiled"]
    assert err(A, B, C0, 1.0, 0.0, C.cpu().numpy()) <= osg.SGEMM_TOL


def test_tf32_operand_rounding_probe(ctx):
    """Informational: 3xTF32 pre-rounds both halves, so the tensor core's own
    fp32->tf32 handling (truncate vs round) cannot change the result."""
    a = np.float32(1 + 2 ** -11 + 2 ** -12)
    A = np.full((128, 8), 0, np.float32)
    A[0, 0] = a
    B = np.zeros((8, 64), np.float32)
    B[0, 0] = 1.0
    C = dev(np.zeros((128, 64), np.float32))
    ctx.sgemm_variant(2, dev(A), dev(B), C)
    assert C.cpu().numpy()[0, 0] == a
