"""GPU parity of the SpMV path through the C ABI vs the fp64 oracle (SURVEY c-1,
c-3, c-4, c-6, c-7, c-10)."""
import numpy as np
import pytest
from conftest import expected_selection

from gpu_helpers import oracle_spmv, spmv_err, to_dev, unit_slices, vec
from oracle import formats, slice_plan
from oracle.spmv import SPMV_TOL
from workloads import (d1_bus, d3_fem, d4_powerlaw, d6_diag, identity, random_lengths_csr, small_int_csr,
                       small_int_vector, uniform_f32, CSR)

pytestmark = pytest.mark.gpu

MATS = {
    "d1": lambda: d1_bus(),
    "ragged": lambda: random_lengths_csr(5003, 4000, 300, 17, empty_frac=0.1),
    "d3small": lambda: d3_fem(grid=101),
    "powerlaw": lambda: d4_powerlaw(n=60_000, lmax=4000),
    "diag": lambda: d6_diag(n=70_000),
    # 16,384-entry rows: heavy units, run first by the claim kernels (A-40)
    "heavy": lambda: d4_powerlaw(n=300_000, lmax=16384),
}


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


def prepared(ctx, A, default=1, formats=None):
    import torch
    rp, col, val = to_dev(A)
    from paper_conf_asplos_changkh16_b200 import dysel
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=default,
                            formats=dysel.FMT_ALL if formats is None else formats)
    torch.cuda.synchronize()
    return plan


@pytest.mark.parametrize("name", list(MATS))
def test_formats_bit_exact(ctx, name):
    A = MATS[name]()
    plan = prepared(ctx, A)
    if formats.ell_applicable(A.row_ptr):
        W, npad, ec, ev = formats.csr_to_ell_fast(A.row_ptr, A.col, A.val)
        assert plan.info.ell_width == W
        assert np.array_equal(plan.array("ell_col"), ec)
        assert np.array_equal(plan.array("ell_val").view(np.uint32), ev.view(np.uint32))
    else:
        assert 2 not in plan.variant_ids            # A-15
    j = formats.csr_to_block_jds_fast(A.row_ptr, A.col, A.val)
    for k in ("perm", "blk_off", "jd_off", "jd_ptr", "jds_col"):
        assert np.array_equal(plan.array(k), j[k]), k
    assert np.array_equal(plan.array("jds_val").view(np.uint32), j["jds_val"].view(np.uint32))
    lens = A.lengths()
    assert np.array_equal(plan.array("jds_len"), lens[j["perm"]])
    assert plan.info.uniform == int(formats.uniform_rows(A.row_ptr))
    plan.destroy()


@pytest.mark.parametrize("name", list(MATS))
def test_variants_parity(ctx, D, name):
    import torch
    A = MATS[name]()
    x = uniform_f32(99, A.n_cols)
    plan = prepared(ctx, A)
    xd = vec(x)
    outs = {}
    for v in plan.variant_ids:
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv_variant(plan, v, xd, y)
        torch.cuda.synchronize()
        assert spmv_err(A, x, y) <= SPMV_TOL, D.SPMV_NAMES[v]
        outs[v] = y.cpu().numpy()
    # CSR-S, ELL, JDS and CSR-T accumulate in CSR order with fmaf: bit-identical
    ref = outs[0].view(np.uint32)
    for v in (2, 3, 5):
        if v in outs:
            assert np.array_equal(outs[v].view(np.uint32), ref), D.SPMV_NAMES[v]
    plan.destroy()


@pytest.mark.parametrize("name", ["d1", "ragged", "powerlaw", "heavy"])
def test_small_integer_bit_exact(ctx, name):
    import torch
    A = small_int_csr(MATS[name](), 5)
    x = small_int_vector(A.n_cols, 6)
    ys, _ = oracle_spmv(A, x)
    plan = prepared(ctx, A)
    for v in plan.variant_ids:
        y = torch.empty(A.n_rows, device="cuda")
        ctx.spmv_variant(plan, v, vec(x), y)
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ys), v
    plan.destroy()


def test_identity_and_diagonal_exact(ctx):
    import torch
    I = identity(3001)
    x = uniform_f32(1, 3001)
    plan = prepared(ctx, I)
    for v in plan.variant_ids:
        y = torch.empty(3001, device="cuda")
        ctx.spmv_variant(plan, v, vec(x), y)
        assert np.array_equal(y.cpu().numpy(), x)
    Dg = d6_diag(n=10_000)
    x = uniform_f32(2, 10_000)
    plan2 = prepared(ctx, Dg)
    expect = (Dg.val * x).astype(np.float32)      # one product, fl32(d_i x_i)
    for v in plan2.variant_ids:
        y = torch.empty(10_000, device="cuda")
        ctx.spmv_variant(plan2, v, vec(x), y)
        assert np.array_equal(y.cpu().numpy(), expect)


MODES = ["fully_sync", "fully_async", "hybrid_sync", "hybrid_async", "fully_sync_host", "fully_async_host",
         "hybrid_sync_host", "fully_contig_sync", "fully_sync_cycles", "fully_sync_seq", "hybrid_async_seq",
         "hybrid_sync_noabort", "fully_async_makespan"]


def mode_bits(D, m):
    b = D.FORCE_PROFILE
    b |= D.HYBRID if m.startswith("hybrid") else D.FULLY
    b |= D.ASYNC if "async" in m else D.SYNC
    b |= D.HOST_ORCH if m.endswith("host") else 0
    b |= D.CONTIGUOUS if "contig" in m else 0
    b |= D.SCORE_CYCLES if "cycles" in m else 0
    b |= D.SEQUENTIAL if "seq" in m else 0
    b |= D.NO_ABORT if "noabort" in m else 0
    b |= D.SCORE_MAKESPAN if "makespan" in m else 0
    return b


def unit_order(plan):
    """The plan's unit order (reading A-45): identity unless it keeps one."""
    s = plan.array("seq")
    return np.arange(plan.n_units) if s is None else s


@pytest.mark.parametrize("m", MODES)
@pytest.mark.parametrize("name", ["ragged", "powerlaw", "d3small", "heavy"])
def test_dysel_composition(ctx, D, name, m):
    """c-6: y_dysel restricted to unit u == y_full[v(u)] restricted to u, bitwise;
    every unit productively computed exactly once; parity vs oracle."""
    import torch
    A = MATS[name]()
    x = uniform_f32(7, A.n_cols)
    # solo (A-38) needs a pool without CSR-T; its remainder then runs the winner
    # through the default's (CSR-S's) claim kernel
    plan = prepared(ctx, A, default=0)
    xd = vec(x)
    full = {}
    for v in plan.variant_ids:
        y = torch.empty(A.n_rows, device="cuda")
        ctx.spmv_variant(plan, v, xd, y)
        full[v] = y.cpu().numpy().view(np.uint32)
    mode = mode_bits(D, m)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    rep = ctx.spmv(plan, xd, y, f=0.1, mode=mode, report=True, unit_map=True)
    torch.cuda.synchronize()
    assert rep["profiled"]
    assert spmv_err(A, x, y) <= SPMV_TOL
    yy = y.cpu().numpy().view(np.uint32)
    uv = rep["unit_variant"]
    K = len(plan.variant_ids)
    # oracle plan: same c, same granule count
    grouped = not (m.endswith("host") or "seq" in m)   # device path, grouped profiling (A-49, A-52)
    p = slice_plan.plan((plan.n_units,), [(1,)] * K, 0.1, ctx.n_sm, plan.variant_ids.index(0), mode,
                        [0 if plan.info.uniform else slice_plan.V_NONUNIFORM] * K,
                        min_c=slice_plan.MIN_PROF_UNITS if grouped else 0)
    assert rep["c"] == p.c and rep["n_granules"] == p.Gn
    sel = rep["selected"]
    assert sel in plan.variant_ids
    for u, (r0, r1) in enumerate(unit_slices(A.n_rows)):
        v = uv[u]
        assert v in full, (u, v)
        assert np.array_equal(yy[r0:r1], full[v][r0:r1]), (u, v)
    # profiling granules carry the ticket's variant, remainder the selection (sync).
    # Device-path hybrid (reading A-4'): the shared profiled units are the
    # winner's (its sandbox is copied in); the host path keeps the paper's
    # productive default (A-4).
    # The device path profiles the first units of the plan's unit order
    # (light units first, A-45); the host path the NDRange prefix (paper).
    # Hybrid: the default's profiled slice is the productive one (A-4).
    pool = plan.variant_ids
    owner = slice_plan.productive_cover(p, pool.index(sel))
    host = m.endswith("host")
    order = np.arange(plan.n_units) if host else unit_order(plan)
    n_prof = p.c * (K if p.mode == slice_plan.FULLY else 1)
    for j in range(p.Gn):
        u = order[j]
        if j < len(owner) and j < n_prof:
            assert uv[u] == pool[owner[j]], j
        elif "async" not in m:
            assert uv[u] == sel, j
    # Table 1: fully 0 extra outputs, hybrid K - 1 sandboxes
    assert rep["sandbox_buffers"] == (K - 1 if p.mode == slice_plan.HYBRID else 0), rep["sandbox_buffers"]
    assert rep["sandbox_bytes"] == (K - 1) * p.c * 256 * 4 * (p.mode == slice_plan.HYBRID) or host
    assert sorted(order) == list(range(plan.n_units))      # a permutation: every unit exactly once
    plan.destroy()


def test_no_profile_and_cache(ctx, D):
    import torch
    A = MATS["ragged"]()
    x = uniform_f32(8, A.n_cols)
    plan = prepared(ctx, A, default=3)
    xd = vec(x)
    ref = torch.empty(A.n_rows, device="cuda")
    ctx.spmv_variant(plan, 3, xd, ref)
    y = torch.empty(A.n_rows, device="cuda")
    rep = ctx.spmv(plan, xd, y, mode=D.NO_PROFILE, report=True)
    assert not rep["profiled"] and rep["selected"] == 3
    assert torch.equal(y.view(torch.int32), ref.view(torch.int32))       # P:L868-871 "0 profiled blocks"
    rep = ctx.spmv(plan, xd, y, f=0.2, mode=D.FULLY | D.SYNC | D.FORCE_PROFILE, report=True)
    sel = rep["selected"]
    ctx.spmv_variant(plan, sel, xd, ref)
    rep2 = ctx.spmv(plan, xd, y, mode=D.NO_PROFILE, report=True)   # activation flag: reuse the selection
    assert rep2["selected"] == sel
    assert torch.equal(y.view(torch.int32), ref.view(torch.int32))
    plan.destroy()


def test_small_workload_deactivated(ctx, D):
    import torch
    A = MATS["d1"]()        # 5 units < 128
    x = uniform_f32(9, A.n_cols)
    # forced profiling needs K <= 5 units in fully mode: pool without CSR-T
    plan = prepared(ctx, A, default=1, formats=D.FMT_ELL | D.FMT_JDS | D.FMT_STREAM)
    y = torch.empty(A.n_rows, device="cuda")
    rep = ctx.spmv(plan, vec(x), y, f=0.5, mode=D.DEFAULT_MODE, report=True)
    assert not rep["profiled"] and rep["selected"] == 1
    assert spmv_err(A, x, y) <= SPMV_TOL
    rep = ctx.spmv(plan, vec(x), y, f=0.5, mode=D.DEFAULT_MODE | D.FORCE_PROFILE, report=True)
    assert rep["profiled"]
    assert spmv_err(A, x, y) <= SPMV_TOL
    plan.destroy()


def test_edge_cases(ctx, D):
    import torch
    # all rows empty: y := 0
    n = 1000
    E = CSR(n, n, np.zeros(n + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    plan = prepared(ctx, E)
    y = torch.full((n,), 5.0, device="cuda")
    ctx.spmv(plan, vec(np.ones(n)), y, f=0.5, mode=D.FORCE_PROFILE | D.FULLY)
    assert torch.count_nonzero(y).item() == 0
    # single row, single column
    S1 = CSR(1, 1, np.array([0, 1], np.int32), np.array([0], np.int32), np.array([2.5], np.float32))
    plan = prepared(ctx, S1)
    y = torch.empty(1, device="cuda")
    for v in plan.variant_ids:
        ctx.spmv_variant(plan, v, vec(np.array([4.0])), y)
        assert y.item() == 10.0
    # invalid arguments are rejected, never crash
    with pytest.raises(D.DyselError):
        ctx.spmv(plan, vec(np.array([1.0])), y, f=2.0)
    with pytest.raises(D.DyselError) as e:
        ctx.spmv(plan, vec(np.array([1.0])), y, mode=D.SWAP | D.ASYNC)
    assert e.value.status == D.ERR_UNSUPPORTED


@pytest.mark.parametrize("name", ["powerlaw", "heavy"])
@pytest.mark.parametrize("default", [1, 3])
@pytest.mark.parametrize("asy", [False, True])
def test_remainder_hand_off(ctx, D, asy, default, name):
    """The remainder goes to the winner: the default's claim kernel runs it
    when the default wins, the switch kernel device-launches the winner's
    claim kernel otherwise (A-42).  Sync: every remainder unit is the
    winner's (eager = 0).  Async: the default's eager units are whole LIGHT
    units (A-45: an unproven default never starts a heavy or long-row unit;
    a thread-per-row default -- JDS here -- gets no eager range at all on a
    matrix with long-row units), every other remainder unit is the winner's."""
    import torch
    A = MATS[name]()
    x = uniform_f32(11, A.n_cols)
    plan = prepared(ctx, A, default=default)
    K = len(plan.variant_ids)
    order = unit_order(plan)
    n_light = plan.info.n_light
    light = set(order[:n_light].tolist())
    if name == "heavy":
        assert plan.info.n_heavy > 0 and n_light + plan.info.n_heavy == plan.n_units
    mode = D.FULLY | D.FORCE_PROFILE | (D.ASYNC if asy else 0)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    r = ctx.spmv(plan, vec(x), y, f=0.05, mode=mode, report=True, unit_map=True)
    assert spmv_err(A, x, y) <= SPMV_TOL
    P = K * r["c"]
    rem = plan.n_units - P
    uv = r["unit_variant"]
    sel = r["selected"]
    rest = [order[j] for j in range(P, plan.n_units)]
    if not asy:
        assert r["eager_units"] == 0 and r["tail_units"] == rem, r
        assert all(uv[u] == sel for u in rest)
    else:
        assert all(uv[u] in (default, sel) for u in rest)
        if default != sel:
            eager = [u for u in rest if uv[u] == default]
            assert len(eager) <= r["eager_units"]
            assert all(u in light for u in eager)                # never a heavy / long-row unit
            if default == 3 and plan.info.n_heavy > 0:
                assert r["eager_units"] == 0 and not eager       # thread-per-row default: no eager range
        else:
            assert r["eager_units"] + r["tail_units"] == rem, r
    plan.destroy()


def test_remainder_is_stream_ordered(ctx, D):
    """Work queued on the launching stream after dysel_spmv must see the whole
    remainder complete -- also a winner's claim kernel device-launched by the
    switch kernel (it belongs to its parent's completion) -- without any host
    synchronisation in between."""
    import torch
    A = d4_powerlaw(n=400_000, lmax=8000)
    x = uniform_f32(12, A.n_cols)
    xd = vec(x)
    for default in (1, 3):      # 3 (JDS) loses on this matrix: its claim kernel hands over via the switch kernel
        plan = prepared(ctx, A, default=default)
        for mode in (D.HYBRID | D.SYNC, D.HYBRID | D.ASYNC, D.FULLY | D.SYNC, D.FULLY | D.ASYNC):
            for _ in range(3):
                y = torch.full((A.n_rows,), float("nan"), device="cuda")
                ctx.spmv(plan, xd, y, f=0.01, mode=mode | D.FORCE_PROFILE)
                nan_count = torch.isnan(y).sum()          # same stream, no sync
                snap = y.clone()
                torch.cuda.synchronize()
                assert nan_count.item() == 0, mode
                assert spmv_err(A, x, snap) <= SPMV_TOL
        plan.destroy()


def test_dominance_abort_is_exact(ctx, D):
    """Hybrid sandbox units of a variant whose guaranteed busy time already
    exceeds a completed variant's total stop early; the dominated variant gets
    the maximal score and the winner is the busy-time argmin of the others
    (with the switch margin of A-50)."""
    import torch
    from workloads import csr_from_lengths
    # a few very long rows make thread-per-row variants hopeless
    L = np.full(40 * 256, 8)
    L[::97] = 6000
    A = csr_from_lengths(L, 20000, 21, 22)
    x = uniform_f32(23, A.n_cols)
    plan = prepared(ctx, A, default=1)
    y = torch.empty(A.n_rows, device="cuda")
    rep = ctx.spmv(plan, vec(x), y, f=0.5, mode=D.HYBRID | D.SYNC | D.FORCE_PROFILE, report=True)
    assert spmv_err(A, x, y) <= SPMV_TOL
    ids = plan.variant_ids
    cap = (1 << 56) - 1
    assert rep["selected"] == expected_selection(rep, ids, plan.info.default_variant)
    assert sum(rep["aborted"][v] for v in ids) > 0          # someone was stopped
    assert all(rep["score"][v] == cap for v in ids if rep["aborted"][v] > 0)
    rep2 = ctx.spmv(plan, vec(x), y, f=0.5, mode=D.HYBRID | D.SYNC | D.FORCE_PROFILE | D.NO_ABORT, report=True)
    assert sum(rep2["aborted"][v] for v in ids) == 0
    assert spmv_err(A, x, y) <= SPMV_TOL
    plan.destroy()


def test_long_rows_vector_path(ctx):
    """Rows >= 128 entries take CSR-V's 128-bit path (head / body / tail)."""
    import torch
    L = np.array([0, 1, 127, 128, 129, 131, 255, 256, 257, 1000, 4093, 5000] * 30)
    A = d4_powerlaw(n=2, lmax=2)   # placeholder for type
    from workloads import csr_from_lengths
    A = csr_from_lengths(L, 6000, 3, 4)
    x = uniform_f32(5, 6000)
    plan = prepared(ctx, A)
    y = torch.empty(A.n_rows, device="cuda")
    ctx.spmv_variant(plan, 1, vec(x), y)
    assert spmv_err(A, x, y) <= SPMV_TOL
    # unaligned base pointers disable the vector body but keep parity
    rp, col, val = to_dev(A)
    col2 = torch.empty(col.numel() + 1, dtype=torch.int32, device="cuda")[1:]
    val2 = torch.empty(val.numel() + 1, dtype=torch.float32, device="cuda")[1:]
    col2.copy_(col)
    val2.copy_(val)
    plan2 = ctx.spmv_prepare(rp, col2, val2, A.n_cols)
    ctx.spmv_variant(plan2, 1, vec(x), y)
    assert spmv_err(A, x, y) <= SPMV_TOL


@pytest.mark.parametrize("name", ["d3", "diag_big"])
def test_csr_tma_multi_slot(ctx, D, name):
    """CSR-T with several 32-row slots per warp (grid > one wave of claims):
    the staging buffers and their mbarrier are reused slot after slot.
    Bit-identical to CSR-S (same per-row fma order) and within tolerance."""
    import torch
    A = d3_fem() if name == "d3" else d6_diag(n=300_000)
    x = uniform_f32(31, A.n_cols)
    plan = prepared(ctx, A, default=0, formats=D.FMT_TMA)
    assert D.SPMV_CSR_TMA in plan.variant_ids
    outs = {}
    for v in (D.SPMV_CSR_SCALAR, D.SPMV_CSR_TMA):
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        for _ in range(2):   # second run: warps start on buffers left by the first
            ctx.spmv_variant(plan, v, vec(x), y)
        outs[v] = y.cpu().numpy()
    assert spmv_err(A, x, torch.from_numpy(outs[D.SPMV_CSR_TMA])) <= SPMV_TOL
    assert np.array_equal(outs[D.SPMV_CSR_TMA].view(np.uint32), outs[D.SPMV_CSR_SCALAR].view(np.uint32))
    plan.destroy()


def test_gather_probe_runs_and_validates(ctx, D):
    """dysel_spmv_gather_probe (measurement only): every flavour
    run on an aligned plan and write every one of d_out's n_rows floats; a bad
    flavour is rejected with DYSEL_ERR_INVALID."""
    import torch
    A = MATS["powerlaw"]()
    plan = prepared(ctx, A)
    x = vec(uniform_f32(5, A.n_cols))
    for fl in (0, 1, 2, 3, 4):   # 3: TMA gather4 values checked against x[col] on the device
        out = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv_gather_probe(plan, fl, x, out)
        torch.cuda.synchronize()
        assert bool(torch.isfinite(out).all())
    with pytest.raises(Exception):
        ctx.spmv_gather_probe(plan, 5, x, out)
    plan.destroy()


@pytest.mark.parametrize("name", ["heavy", "powerlaw", "d3small"])
def test_unit_order(ctx, D, name):
    """Readings A-40 / A-45: the plan's unit order (light units in index
    order, then heavy / long-row units by nonzeros descending) equals the
    oracle's restatement of the rule bit for bit; every pure variant's
    heavy-first claim run is within tolerance of the oracle, and CSR-S / ELL /
    JDS stay bit-identical."""
    import torch
    A = MATS[name]()
    plan = prepared(ctx, A)
    seq, n_light = slice_plan.unit_order(A.row_ptr, ctx.n_sm)
    got = plan.array("seq")
    if seq is None:
        assert got is None and plan.info.n_heavy == 0 and plan.info.n_light == plan.n_units
    else:
        assert np.array_equal(got, np.asarray(seq, np.int32))
        assert plan.info.n_light == n_light and plan.info.n_heavy == plan.n_units - n_light
    if name == "heavy":
        assert seq is not None and n_light < plan.n_units
    x = uniform_f32(9, A.n_cols)
    xd = vec(x)
    ys = {}
    for v in plan.variant_ids:
        y = torch.full((A.n_rows,), float("nan"), device="cuda")
        ctx.spmv_variant(plan, v, xd, y)
        ys[v] = y.cpu().numpy()
        assert spmv_err(A, x, y) <= SPMV_TOL, v
    for v in (0, 2, 3):   # CSR-S, ELL, JDS: bit-identical by construction
        if v in ys:
            assert np.array_equal(ys[v], ys[0]), v
    plan.destroy()


def test_hybrid_unaligned_output_view(ctx, D):
    """the output may be any float pointer (a tensor view y[1:]):
    the device path must not use 16-byte stores on it."""
    import torch
    A = MATS["heavy"]()
    x = uniform_f32(81, A.n_cols)
    plan = prepared(ctx, A, default=D.SPMV_DEFAULT_AUTO)
    buf = torch.full((A.n_rows + 1,), float("nan"), device="cuda")
    y = buf[1:]
    for mode in (D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.HYBRID | D.FORCE_PROFILE):
        y.fill_(float("nan"))
        ctx.spmv(plan, vec(x), y, f=0.05, mode=mode)
        torch.cuda.synchronize()
        assert spmv_err(A, x, y) <= SPMV_TOL
    plan.destroy()


def test_auto_initial_version_by_l2_residency(ctx, D):
    """Readings A-30b / A-30c: a uniform matrix whose CSR arrays exceed the L2
    and whose rows hold 8..32 entries gets CSR-T as its initial version (when
    in the pool); uniform rows of < 8 entries CSR-S; other uniform ones ELL; a
    non-uniform one CSR-W.  The result is exact either way."""
    import torch
    from workloads import d3_fem
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    big = d3_fem(grid=1500)                      # 56.2M nnz: 0.46 GB of CSR
    assert 8 * big.nnz + 4 * (big.n_rows + 1) > l2
    small = d3_fem(grid=383)                     # 30.9 MB of CSR
    assert 8 * small.nnz + 4 * (small.n_rows + 1) < l2
    import numpy as np
    from workloads import csr_from_lengths
    long_rows = csr_from_lengths(np.full(1_000_000, 48, np.int64), 1_000_000, 21, 22)   # > L2, rows of 48 > 32
    short_rows = csr_from_lengths(np.full(4_000_000, 5, np.int64), 4_000_000, 23, 24)   # > L2, rows of 5 < 8
    assert 8 * long_rows.nnz > l2 and 8 * short_rows.nnz > l2
    for A, want in ((big, D.SPMV_CSR_TMA), (small, D.SPMV_ELL), (MATS["powerlaw"](), D.SPMV_CSR_STREAM),
                    (long_rows, D.SPMV_ELL), (short_rows, D.SPMV_CSR_SCALAR)):
        plan = prepared(ctx, A, default=D.SPMV_DEFAULT_AUTO)
        assert plan.info.default_variant == want, (D.SPMV_NAMES[plan.info.default_variant], D.SPMV_NAMES[want])
        plan.destroy()
    plan = prepared(ctx, big, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ELL | D.FMT_STREAM)   # no CSR-T
    assert plan.info.default_variant == D.SPMV_ELL
    x = uniform_f32(15, big.n_cols)
    y = torch.empty(big.n_rows, device="cuda")
    plan2 = prepared(ctx, big, default=D.SPMV_DEFAULT_AUTO)
    ctx.spmv(plan2, vec(x), y, f=0.02, mode=D.AUTO | D.ASYNC)
    torch.cuda.synchronize()
    assert spmv_err(big, x, y) <= SPMV_TOL
    plan.destroy()
    plan2.destroy()


def test_min_profiling_slice_a52(ctx, D):
    """Reading A-52: at a tiny f the device path grows each variant's slice to
    12 units (oracle plan with min_c), the result stays exact, and on a
    regular FEM matrix the selection is ELL (the pure best) instead of CSR-S."""
    import torch
    from workloads import d3_fem
    A = d3_fem(grid=1500)
    x = uniform_f32(5, A.n_cols)
    plan = prepared(ctx, A, default=D.SPMV_DEFAULT_AUTO, formats=D.FMT_ELL | D.FMT_JDS | D.FMT_STREAM)
    K = len(plan.variant_ids)
    y = torch.empty(A.n_rows, device="cuda")
    sels = []
    for _ in range(5):
        rep = ctx.spmv(plan, vec(x), y, f=0.001, mode=D.AUTO | D.ASYNC, report=True)
        sels.append(rep["selected_name"])
    p = slice_plan.plan((plan.n_units,), [(1,)] * K, 0.001, ctx.n_sm, plan.variant_ids.index(plan.info.default_variant),
                        D.AUTO | D.ASYNC, [0] * K, wave_units=0, min_c=slice_plan.MIN_PROF_UNITS)
    assert rep["c"] == p.c == slice_plan.MIN_PROF_UNITS
    torch.cuda.synchronize()
    assert spmv_err(A, x, y) <= SPMV_TOL
    assert sels.count("ell") >= 4, sels
    plan.destroy()


def test_small_matrix_unprofiled_a3c(ctx, D):
    """Reading A-3c: below 64 MiB of algorithmic bytes a call is not profiled
    (the initial version runs: CSR-S for the 1-entry diagonal, A-30c) unless
    FORCE_PROFILE; the oracle plan with work_bytes agrees; results exact."""
    import torch
    from workloads import d6_diag
    A = d6_diag()
    x = uniform_f32(17, A.n_cols)
    plan = prepared(ctx, A, default=D.SPMV_DEFAULT_AUTO)
    assert plan.info.default_variant == D.SPMV_CSR_SCALAR
    b = 8 * A.nnz + 4 * (A.n_rows + 1) + 4 * A.n_cols + 4 * A.n_rows
    K = len(plan.variant_ids)
    y = torch.empty(A.n_rows, device="cuda")
    for mode, want in ((D.AUTO | D.ASYNC, False), (D.AUTO | D.ASYNC | D.FORCE_PROFILE, True)):
        rep = ctx.spmv(plan, vec(x), y, f=0.02, mode=mode, report=True)
        p = slice_plan.plan((plan.n_units,), [(1,)] * K, 0.02, ctx.n_sm, plan.variant_ids.index(D.SPMV_CSR_SCALAR),
                            mode, [0] * K, work_bytes=b, min_c=slice_plan.MIN_PROF_UNITS)
        assert rep["profiled"] == want == p.active, (rep["profiled"], want, p.active)
        torch.cuda.synchronize()
        assert spmv_err(A, x, y) <= SPMV_TOL
    plan.destroy()
