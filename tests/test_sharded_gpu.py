"""1-GPU loopback of the row-sharded SpMV and the M-sharded SGEMM (SURVEY §8e
"Testing without 8 GPUs: a 1-GPU loopback ... tests the partition and
assembly code").  G shards, each with its own plan (rebased row_ptr, the
layout each rank's local plan has) and therefore its own selection (a mixed
version), run one after another on one device; one
cudaMemcpyAsync per shard stands in for the allgatherv.  Parity: every shard
bitwise equal to its own per-unit composition of pure runs (c-6), the whole y
within SPMV_TOL of the fp64 oracle."""
import numpy as np
import pytest
from conftest import expected_selection

from gpu_helpers import spmv_err, vec
from oracle import partition
from oracle import sgemm as osg
from oracle.spmv import SPMV_TOL
from workloads import CSR, csr_from_lengths, d3_fem, d4_powerlaw, d6_diag, sgemm_inputs, uniform_f32

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def D():
    from paper_conf_asplos_changkh16_b200 import dysel
    return dysel


@pytest.fixture(scope="module")
def ctx(gpu, D):
    c = D.Context(0)
    yield c
    c.close()


def shard_plans(ctx, D, A, bounds, default=-1):
    import torch
    plans = []
    for g in range(len(bounds) - 1):
        r0, r1 = bounds[g], bounds[g + 1]
        lo, hi = int(A.row_ptr[r0]), int(A.row_ptr[r1])
        rp = torch.from_numpy((A.row_ptr[r0:r1 + 1].astype(np.int64) - lo).astype(np.int32)).cuda()
        col = torch.from_numpy(np.ascontiguousarray(A.col[lo:hi])).cuda()
        val = torch.from_numpy(np.ascontiguousarray(A.val[lo:hi])).cuda()
        plans.append(ctx.spmv_prepare(rp, col, val, A.n_cols, default=default))
    return plans


def mixed_matrix():
    """Rows 0..n1: diagonal (thread-per-row variants win); then power-law rows
    (warp-streaming wins): shards on either side select differently."""
    n1 = 256 * 800
    Dg = d6_diag(n=n1)
    P = d4_powerlaw(n=256 * 1200, lmax=8000)
    n = n1 + P.n_rows
    L = np.concatenate([np.ones(n1, np.int64), np.diff(P.row_ptr.astype(np.int64))])
    A = csr_from_lengths(L, n, 51, 52)
    return A, n1


@pytest.mark.parametrize("G", [2, 3, 4])
@pytest.mark.parametrize("name", ["mixed", "powerlaw", "d3"])
@pytest.mark.parametrize("mode_name", ["hybrid_sync", "auto_async"])
def test_spmv_loopback(ctx, D, G, name, mode_name):
    import torch
    if name == "mixed":
        A, n1 = mixed_matrix()
    elif name == "powerlaw":
        A = d4_powerlaw(n=400_000, lmax=16384)
    else:
        A = d3_fem(grid=201)
    x = uniform_f32(5 + G, A.n_cols)
    bounds = D.partition_rows(A.row_ptr, G)
    assert bounds == partition.partition_rows(A.row_ptr, G)      # library == oracle (bit-exact integers)
    plans = shard_plans(ctx, D, A, bounds)
    xd = vec(x)
    mode = (D.HYBRID | D.SYNC | D.FORCE_PROFILE) if mode_name == "hybrid_sync" else (D.AUTO | D.ASYNC |
                                                                                       D.FORCE_PROFILE)
    # stale data in the staging buffer / y must not survive: run once with another x first
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    ctx.spmv_sharded_loopback(plans, bounds, vec(uniform_f32(1, A.n_cols)), y, f=0.02, mode=mode)
    y.fill_(float("nan"))
    reps = ctx.spmv_sharded_loopback(plans, bounds, xd, y, f=0.02, mode=mode, report=True)
    torch.cuda.synchronize()
    assert spmv_err(A, x, y) <= SPMV_TOL
    yy = y.cpu().numpy().view(np.uint32)
    sels = []
    for g, (pl, r) in enumerate(zip(plans, reps)):
        r0, r1 = bounds[g], bounds[g + 1]
        assert r["selected"] in pl.variant_ids
        sels.append(r["selected"])
        if mode_name != "hybrid_sync" or not r["profiled"]:
            continue
        # hybrid sync: the default's profiled units (seq[0, c)) + the winner's remainder (c-6)
        seq = pl.array("seq")
        seq = np.arange(pl.n_units) if seq is None else seq
        pure = {}
        for v in {pl.info.default_variant, r["selected"]}:
            t = torch.empty(r1 - r0, device="cuda")
            ctx.spmv_variant(pl, v, xd, t)
            pure[v] = t.cpu().numpy().view(np.uint32)
        for j, u in enumerate(seq):
            v = pl.info.default_variant if j < r["c"] else r["selected"]
            a, b = u * 256, min((u + 1) * 256, r1 - r0)
            assert np.array_equal(yy[r0 + a:r0 + b], pure[v][a:b]), (g, u, v)
    if name == "mixed" and G == 2:
        print("per-shard selections (mixed version):", [D.SPMV_NAMES[s] for s in sels])
    for p in plans:
        p.destroy()


def test_spmv_loopback_mixed_version_selections(ctx, D):
    """The two regimes of the mixed matrix select per shard (bounds at the
    regime boundary): the thread-per-row family on the diagonal shard, the
    warp family on the power-law shard (the ranking on B200 is measured, not
    pinned: this asserts only that each shard's selection is the argmin of
    its own scores (with the switch margin of A-50), i.e. shards decide
    independently)."""
    import torch
    A, n1 = mixed_matrix()
    bounds = [0, n1, A.n_rows]
    plans = shard_plans(ctx, D, A, bounds)
    x = uniform_f32(3, A.n_cols)
    y = torch.empty(A.n_rows, device="cuda")
    reps = ctx.spmv_sharded_loopback(plans, bounds, vec(x), y, f=0.05, mode=D.FULLY | D.SYNC | D.FORCE_PROFILE,
                                     report=True)
    assert spmv_err(A, x, y) <= SPMV_TOL
    cap = (1 << 56) - 1
    for pl, r in zip(plans, reps):
        ids = pl.variant_ids
        assert r["selected"] == expected_selection(r, ids, pl.info.default_variant)
    for p in plans:
        p.destroy()


def test_spmv_loopback_rejects_bad_bounds(ctx, D):
    import torch
    A = d4_powerlaw(n=20_000, lmax=500)
    bounds = D.partition_rows(A.row_ptr, 2)
    plans = shard_plans(ctx, D, A, bounds)
    y = torch.empty(A.n_rows, device="cuda")
    with pytest.raises(D.DyselError):
        ctx.spmv_sharded_loopback(plans, [0, bounds[1] + 256, A.n_rows], vec(np.ones(A.n_cols)), y)
    for p in plans:
        p.destroy()


@pytest.mark.parametrize("G", [2, 3, 8])
def test_sgemm_m_shards_loopback(ctx, D, G):
    """M-sharded SGEMM: each shard computes C_g from its LOCAL A_g only
    (rows dysel_sgemm_shard_rows(M, G, g)), with its own selection; the
    assembled C is within SGEMM_TOL of the oracle."""
    import torch
    M, K, N = 1000, 520, 760
    A, B, C0 = sgemm_inputs(M, K, N, 7, 8, 9)
    C = torch.from_numpy(C0.copy()).cuda()
    Bd = torch.from_numpy(B).cuda()
    covered = 0
    for g in range(G):
        m0, m1 = D.sgemm_shard_rows(M, G, g)
        assert m0 == min(M, g * ((-(-M // G) + 127) // 128 * 128))
        assert m0 == covered or m1 == m0
        covered = max(covered, m1)
        if m1 > m0:
            Ag = torch.from_numpy(np.ascontiguousarray(A[m0:m1])).cuda()   # local rows only
            ctx.sgemm(Ag, Bd, C[m0:m1], 1.5, -0.5, f=0.06, mode=D.FULLY | D.FORCE_PROFILE)
    assert covered == M
    torch.cuda.synchronize()
    ref, den = osg.sgemm(A, B, C0, 1.5, -0.5), osg.sgemm_abs(A, B, C0, 1.5, -0.5)
    assert float((np.abs(C.cpu().numpy() - ref) / den).max()) <= osg.SGEMM_TOL
