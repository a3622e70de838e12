"""GPU parity of the atomic scatter pool y += A^T x (dysel_spmtv, SURVEY §8f
f-1) through the C ABI vs the fp64 oracle: the swap-based partial-productive
mode on a real kernel with overlapping outputs (§2.2
§3.3, Table 1).  fp32 reductions in no fixed order: within
SPMV_TOL of the oracle; small integers: bit-exact in any order."""
import numpy as np
import pytest

from gpu_helpers import to_dev, vec
from oracle.spmv import SPMV_TOL, rel_error, spmtv, spmtv_abs
from workloads import d1_bus, d4_powerlaw, random_lengths_csr, small_int_csr, small_int_vector, uniform_f32

pytestmark = pytest.mark.gpu

MATS = {
    "d1": lambda: d1_bus(),
    "ragged_nonsquare": lambda: random_lengths_csr(5003, 4000, 300, 17, empty_frac=0.1),
    # 2,344 units: more than one wave of either variant -> profiled
    "powerlaw": lambda: d4_powerlaw(n=600_000, lmax=2000),
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


def _plan(ctx, A):
    import torch
    rp, col, val = to_dev(A)
    plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
    torch.cuda.synchronize()
    return plan, (rp, col, val)


def _err(A, x, y0, y):
    ys = spmtv(A.row_ptr, A.col, A.val, x, y0)
    return rel_error(y.cpu().numpy(), ys, spmtv_abs(A.row_ptr, A.col, A.val, x, y0))


@pytest.mark.parametrize("name", list(MATS))
def test_spmtv_variants_parity(ctx, D, name):
    import torch
    A = MATS[name]()
    x = uniform_f32(31, A.n_rows)
    y0 = uniform_f32(32, A.n_cols)
    plan, keep = _plan(ctx, A)
    for v in range(len(D.SPMTV_NAMES)):
        y = vec(y0)
        ctx.spmtv_variant(plan, v, vec(x), y)
        torch.cuda.synchronize()
        assert _err(A, x, y0, y) <= SPMV_TOL, D.SPMTV_NAMES[v]
    plan.destroy()


@pytest.mark.parametrize("name", list(MATS))
@pytest.mark.parametrize("m", ["auto", "swap_host", "fully", "no_profile", "auto_forced", "auto_async",
                               "auto_async_forced"])
def test_spmtv_modes_parity(ctx, D, name, m):
    """Every unit's contribution lands in y exactly once, whichever variant
    profiled or ran it; AUTO resolves to swap (DYSEL_V_ATOMICS)."""
    import torch
    A = MATS[name]()
    x = uniform_f32(41, A.n_rows)
    y0 = uniform_f32(42, A.n_cols)
    plan, keep = _plan(ctx, A)
    mode = {"auto": D.AUTO, "swap_host": D.SWAP | D.HOST_ORCH, "fully": D.FULLY, "no_profile": D.AUTO | D.NO_PROFILE,
            "auto_forced": D.AUTO | D.FORCE_PROFILE, "auto_async": D.AUTO | D.ASYNC,
            "auto_async_forced": D.AUTO | D.ASYNC | D.FORCE_PROFILE}[m]
    for rep_i in range(3):   # cached selection on later calls must not change the result
        y = vec(y0)
        rep = ctx.spmtv(plan, vec(x), y, f=0.05, mode=mode, report=True)
        torch.cuda.synchronize()
        assert _err(A, x, y0, y) <= SPMV_TOL, (m, rep_i)
        assert 0 <= rep["selected"] < len(D.SPMTV_NAMES)
        if m != "fully" and rep["profiled"]:
            assert rep["mode_used"] & 3 == D.SWAP
            # reading A-47b: eager light units only on the additive (device) swap with ASYNC
            assert bool(rep["mode_used"] & D.ASYNC) == m.startswith("auto_async")
            if not m.startswith("auto_async"):
                assert rep["eager_units"] == 0
    if m in ("auto_forced", "auto_async_forced"):
        assert rep["profiled"]
    if name == "powerlaw" and m in ("auto", "auto_async"):
        assert not rep["profiled"]   # 101 MiB: under the SpMTV pool's A-3c line (128 MiB)
    plan.destroy()


def test_spmtv_small_integer_bit_exact(ctx, D):
    """Integer products and sums below 2^24 are exact in any reduction order."""
    import torch
    A = small_int_csr(MATS["powerlaw"](), 5)
    x = small_int_vector(A.n_rows, 6)
    y0 = small_int_vector(A.n_cols, 7)
    ys = spmtv(A.row_ptr, A.col, A.val, x, y0)
    assert np.max(np.abs(ys)) < 2 ** 24
    plan, keep = _plan(ctx, A)
    for mode in (D.AUTO | D.FORCE_PROFILE, D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.SWAP | D.HOST_ORCH,
                 D.FULLY | D.FORCE_PROFILE):
        y = vec(y0)
        ctx.spmtv(plan, vec(x), y, f=0.05, mode=mode)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ys), mode
    # A-47b: the eager / remainder hand-off is timing-dependent -- repeat it; a
    # lost or doubled unit breaks exactness
    xd = vec(x)
    for i in range(12):
        y = vec(y0)
        ctx.spmtv(plan, xd, y, f=(0.01, 0.03, 0.1)[i % 3], mode=D.AUTO | D.ASYNC | D.FORCE_PROFILE)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ys), i
    plan.destroy()


def test_spmtv_swap_async_rejected_and_edges(ctx, D):
    """Table 1 / P:L735-740: the copy-back swap (HOST_ORCH) cannot run
    asynchronously; the additive device swap can (reading A-47b)."""
    import torch
    from paper_conf_asplos_changkh16_b200.dysel import DyselError
    A = MATS["ragged_nonsquare"]()
    plan, keep = _plan(ctx, A)
    x, y = vec(uniform_f32(51, A.n_rows)), vec(uniform_f32(52, A.n_cols))
    with pytest.raises(DyselError):
        ctx.spmtv(plan, x, y, f=0.05, mode=D.SWAP | D.ASYNC | D.HOST_ORCH)
    with pytest.raises(DyselError):
        ctx.spmtv(plan, x, y, f=0.05, mode=D.AUTO | D.ASYNC | D.HOST_ORCH)   # AUTO -> swap, no async (Table 1)
    ctx.spmtv(plan, x, y, f=0.05, mode=D.SWAP | D.ASYNC)   # additive swap: the final output is y (A-47b)
    with pytest.raises(DyselError):
        ctx.spmtv_variant(plan, 7, x, y)
    plan.destroy()
    # nnz = 0: y unchanged
    from workloads import CSR
    n = 1000
    E = CSR(n, n, np.zeros(n + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    plan, keep = _plan(ctx, E)
    y0 = uniform_f32(53, n)
    y = vec(y0)
    ctx.spmtv(plan, vec(uniform_f32(54, n)), y, f=0.05, mode=D.AUTO)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy(), y0)
    plan.destroy()


def test_spmtv_bench_size_parity(ctx, D):
    """The bench's 2M-row power-law SpMTV (40M nnz) in its launch configuration
    (AUTO -> swap, f = 0.01, profiled) against the fp64 oracle, every entry."""
    import torch
    A = d4_powerlaw(n=2_000_000, lmax=4096)
    x = uniform_f32(61, A.n_rows)
    y0 = uniform_f32(62, A.n_cols)
    plan, keep = _plan(ctx, A)
    for mode in (D.AUTO, D.AUTO | D.ASYNC, D.AUTO | D.NO_PROFILE):
        y = vec(y0)
        rep = ctx.spmtv(plan, vec(x), y, f=0.01, mode=mode, report=True)
        torch.cuda.synchronize()
        assert rep["profiled"] == (mode != D.AUTO | D.NO_PROFILE)
        if mode == D.AUTO | D.ASYNC:   # the idle SMs reduced light units before the selection (A-47b)
            assert rep["eager_units"] > 0 and rep["mode_used"] & D.ASYNC
            assert rep["eager_units"] + rep["tail_units"] + rep["c"] == rep["n_granules"]
        assert _err(A, x, y0, y) <= SPMV_TOL, mode
    plan.destroy()


@pytest.mark.parametrize("offset", [0, 1])
def test_spmtv_swap_odd_columns_and_unaligned_y(ctx, D, offset):
    """n_cols % 4 != 0 on a matrix big enough that a losing
    variant is dominated mid-profile -- nothing of a partial private output
    may reach y -- and an output y that is not 16-byte aligned (a tensor
    view): the device swap path's add-in must not assume alignment."""
    import torch
    A = d4_powerlaw(n=600_002, lmax=3000)          # n_cols = 600,002 (mod 4 = 2)
    x = uniform_f32(71, A.n_rows)
    y0 = uniform_f32(72, A.n_cols)
    plan, keep = _plan(ctx, A)
    for mode in (D.AUTO | D.FORCE_PROFILE, D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.SWAP | D.HOST_ORCH):
        buf = torch.empty(A.n_cols + 1, device="cuda")
        y = buf[offset:offset + A.n_cols]
        y.copy_(vec(y0))
        rep = ctx.spmtv(plan, vec(x), y, f=0.02, mode=mode, report=True)
        torch.cuda.synchronize()
        assert rep["profiled"] and rep["mode_used"] & 3 == D.SWAP
        assert rep["sandbox_buffers"] == len(D.SPMTV_NAMES)              # Table 1: K private outputs
        assert _err(A, x, y0, y) <= SPMV_TOL, (mode, offset)
    plan.destroy()


def test_spmtv_async_non_default_winner(ctx, D):
    """A-47b with a winner other than the initial version: rows of 0-8 entries
    plus one 100-entry row in 1,000 -- the longest row exceeds A-30d's 64, so
    scatter-warp starts, but a warp per row idles most lanes and scatter-thread
    wins: the switch kernel launches the winner's remainder while the
    default's eager CTAs drain.  Eager light units (default), the winner's
    add-in, heavy and remaining light units must each land in y once."""
    import torch
    from workloads import csr_from_lengths, rng
    n = 3_000_000   # 146 MiB: profiled without FORCE_PROFILE (A-3c line: 128 MiB)
    L = rng(91).integers(0, 9, n)
    L[::1000] = 100
    A = csr_from_lengths(L, n, 92, 93)
    x = uniform_f32(82, A.n_rows)
    y0 = uniform_f32(83, A.n_cols)
    plan, keep = _plan(ctx, A)
    assert plan.info.max_row_len == 100
    sels = []
    for mode in (D.AUTO | D.ASYNC, D.AUTO | D.ASYNC | D.FORCE_PROFILE, D.AUTO):
        for _ in range(3):
            y = vec(y0)
            rep = ctx.spmtv(plan, vec(x), y, f=0.02, mode=mode, report=True)
            torch.cuda.synchronize()
            assert rep["profiled"], mode
            assert _err(A, x, y0, y) <= SPMV_TOL, (mode, rep["selected_name"])
            assert rep["eager_units"] + rep["tail_units"] + rep["c"] == rep["n_granules"]
            sels.append(rep["selected_name"])
    print("selections", sels)
    assert any(s != "scatter_warp" for s in sels)   # the switch path ran
    # activation flag off: the cached selection of the last profiled call runs
    y = vec(y0)
    rep = ctx.spmtv(plan, vec(x), y, mode=D.AUTO | D.NO_PROFILE, report=True)
    torch.cuda.synchronize()
    assert not rep["profiled"] and rep["selected_name"] == sels[-1]
    assert _err(A, x, y0, y) <= SPMV_TOL
    plan.destroy()


def test_spmtv_initial_version_a30d_and_small_a3c(ctx, D):
    """Reading A-30d: scatter-thread starts when no row exceeds 64 entries,
    scatter-warp otherwise; reading A-3c: under 128 MiB the call runs the
    initial version unprofiled (FORCE_PROFILE overrides).  Parity either way."""
    import torch
    cases = [(random_lengths_csr(1_500_000, 1_200_000, 2, 81), "scatter_thread", False),
             (d4_powerlaw(n=1_000_000, lmax=2000), "scatter_warp", True)]
    for A, want_def, big in cases:
        plan, keep = _plan(ctx, A)
        x = uniform_f32(94, A.n_rows)
        y0 = uniform_f32(95, A.n_cols)
        y = vec(y0)
        rep = ctx.spmtv(plan, vec(x), y, f=0.02, mode=D.AUTO | D.ASYNC, report=True)
        torch.cuda.synchronize()
        assert _err(A, x, y0, y) <= SPMV_TOL
        assert rep["profiled"] == big
        if not big:
            assert rep["selected_name"] == want_def and rep["mode_used"] & 3 == D.SWAP
            y = vec(y0)
            rep = ctx.spmtv(plan, vec(x), y, f=0.02, mode=D.AUTO | D.FORCE_PROFILE, report=True)
            torch.cuda.synchronize()
            assert rep["profiled"] and _err(A, x, y0, y) <= SPMV_TOL
        else:   # the initial version is the eager one: heavy-tailed rows -> scatter-warp
            assert rep["eager_units"] > 0
        plan.destroy()
