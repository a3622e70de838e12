"""The NCCL path of the multi-GPU calls on one GPU: a one-rank
communicator runs the real grouped-broadcast allgatherv / broadcast code;
results checked against the fp64 oracles.  (N > 1 needs more GPUs than
gpurun provides; the partition / assembly host logic is covered by the gloo
world-2 tests.)"""
import numpy as np
import pytest

from gpu_helpers import spmv_err, to_dev, vec
from oracle import iterative, sgemm as osg
from workloads import d4_powerlaw, laplacian_2d, sgemm_inputs, uniform_f32

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cctx(gpu):
    from paper_conf_asplos_changkh16_b200 import dysel as D
    c = D.Context(0)
    c.comm_init(0, 1, D.comm_unique_id())
    yield c
    c.close()


def test_spmv_sharded_one_rank(cctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    A = d4_powerlaw(n=300_000, lmax=4096)
    bounds = D.partition_rows(A.row_ptr, 1)
    assert list(bounds) == [0, A.n_rows]
    rp, col, val = to_dev(A)
    plan = cctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
    x = uniform_f32(21, A.n_cols)
    xd = vec(x)
    cctx.comm_broadcast(xd, 0)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    cctx.spmv_sharded(plan, list(bounds), xd, y, f=0.01, mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
    torch.cuda.synchronize()
    assert spmv_err(A, x, y) <= 1e-5
    plan.destroy()


@pytest.mark.parametrize("mode_name", ["auto_async", "auto_sync", "fully_async", "fully_sync", "no_profile", "host"])
def test_spmv_sharded_overlapped_allgather_modes(cctx, mode_name):
    """The chunked allgather overlapped with the SpMV (comm.cu): every mode
    of the device path counts each 32-row slot exactly once, so every chunk's
    waiter is released (no timeout) and y is right; the host path falls back
    to the plain allgather after the SpMV.  Two calls in a row (the counters
    and the timeout flag are reset per call), a multi-wave matrix with heavy
    units (the remainder finishes chunks out of order)."""
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    mode = {"auto_async": D.AUTO | D.ASYNC | D.FORCE_PROFILE, "auto_sync": D.AUTO | D.FORCE_PROFILE,
            "fully_async": D.FULLY | D.ASYNC | D.FORCE_PROFILE, "fully_sync": D.FULLY | D.FORCE_PROFILE,
            "no_profile": D.NO_PROFILE, "host": D.AUTO | D.HOST_ORCH | D.FORCE_PROFILE}[mode_name]
    A = d4_powerlaw(n=400_000, lmax=8192)
    bounds = D.partition_rows(A.row_ptr, 1)
    rp, col, val = to_dev(A)
    plan = cctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
    x = uniform_f32(22, A.n_cols)
    xd = vec(x)
    for _ in range(2):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        cctx.spmv_sharded(plan, list(bounds), xd, y, f=0.01, mode=mode)
        torch.cuda.synchronize()
        assert spmv_err(A, x, y) <= 1e-5, mode_name
    cctx.spmv_sharded(plan, list(bounds), xd, y, f=0.01, mode=mode)   # raises if a chunk wait had timed out
    torch.cuda.synchronize()
    plan.destroy()


def test_power_sharded_one_rank(cctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    L = laplacian_2d(80)
    x0 = uniform_f32(3, L.n_cols, 0.0, 1.0)
    rp, col, val = to_dev(L)
    plan = cctx.spmv_prepare(rp, col, val, L.n_cols, default=D.SPMV_CSR_VECTOR)
    x = vec(x0)
    y = torch.empty_like(x)
    norms = torch.zeros(12, dtype=torch.float64, device="cuda")
    cctx.spmv_power_sharded(plan, [0, L.n_rows], x, y, 12, profile_every=4, f=0.5,
                            mode=D.FULLY | D.ASYNC | D.FORCE_PROFILE, norms=norms)
    torch.cuda.synchronize()
    _, _, no = iterative.power_iteration(L.row_ptr, L.col, L.val, x0, 12)
    assert np.max(np.abs(norms.cpu().numpy() - no) / no) <= 1e-5
    plan.destroy()


def test_sgemm_sharded_one_rank(cctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    M, K, N = 1024, 992, 1056
    A, B, C0 = sgemm_inputs(M, K, N, 992, 993, 994)
    C = torch.from_numpy(C0.copy()).cuda()
    m0, m1 = D.sgemm_shard_rows(M, 1, 0)
    assert (m0, m1) == (0, M)
    cctx.sgemm_sharded(torch.from_numpy(A[m0:m1].copy()).cuda(), torch.from_numpy(B).cuda(), C, 1.5, -0.5,
                       f=0.06, mode=D.FULLY | D.FORCE_PROFILE)
    torch.cuda.synchronize()
    ref, den = osg.sgemm(A, B, C0, 1.5, -0.5), osg.sgemm_abs(A, B, C0, 1.5, -0.5)
    assert float((np.abs(C.cpu().numpy() - ref) / den).max()) <= osg.SGEMM_TOL


@pytest.mark.parametrize("mode_name", ["auto_async", "auto_sync", "host_orch", "no_profile"])
def test_spmv_host_chunked_copy_out(mode_name):
    """dysel_spmv_host: pinned x in, y out in chunks released by the SpMV's slot
    counters; h_y equals the device buffer bitwise once the stream is done and
    matches the oracle (ragged row count: the last chunk is partial)."""
    import torch
    from oracle.spmv import SPMV_TOL
    from paper_conf_asplos_changkh16_b200 import dysel as D
    ctx = D.Context(0)
    A = d4_powerlaw(n=300_001, lmax=4096)
    x = uniform_f32(31, A.n_cols)
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO)
    mode = {"auto_async": D.AUTO | D.ASYNC, "auto_sync": D.AUTO, "host_orch": D.AUTO | D.HOST_ORCH,
            "no_profile": D.NO_PROFILE}[mode_name] | (D.FORCE_PROFILE if mode_name != "no_profile" else 0)
    hx = torch.from_numpy(x).pin_memory()
    hy = torch.full((A.n_rows,), float("nan")).pin_memory()
    dx = torch.empty(A.n_cols, device="cuda")
    dy = torch.empty(A.n_rows, device="cuda")
    for _ in range(3):
        hy.fill_(float("nan"))
        ctx.spmv_host(plan, hx, hy, dx, dy, f=0.01, mode=mode)
        torch.cuda.synchronize()
        assert torch.isfinite(hy).all()
        assert torch.equal(hy, dy.cpu())
        assert spmv_err(A, x, hy) <= SPMV_TOL
    plan.destroy()
    ctx.close()
