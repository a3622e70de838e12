"""Generic dysel_launch end to end with known-cost variants (c-5, c-7, c-8, c-9)."""
import numpy as np
import pytest

from oracle import selection, slice_plan

pytestmark = pytest.mark.gpu

COSTS = [6000, 1500, 4000, 3000]      # ns per unit -> variant 1 must win


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


def run(ctx, D, sig, U, mode, f=0.1, costs=COSTS, default=0):
    import torch
    ctx.register_spin_variants(sig, costs, default)
    out = torch.zeros(U, dtype=torch.int32, device="cuda")
    rep = ctx.launch(sig, (U,), [out], f=f, mode=mode, sandbox_bytes=[U * 4], report=True, unit_map=U)
    torch.cuda.synchronize()
    return rep, out.cpu().numpy()


@pytest.mark.parametrize("m", ["fully_sync", "fully_host_sync", "fully_host_async", "hybrid_sync", "hybrid_host_async",
                               "swap_sync", "swap_host_sync", "fully_contig_sync"])
def test_known_cost_selection(ctx, D, m):
    U = 600
    mode = D.FULLY
    if m.startswith("hybrid"):
        mode = D.HYBRID
    if m.startswith("swap"):
        mode = D.SWAP
    mode |= D.HOST_ORCH if "host" in m else 0
    mode |= D.ASYNC if "async" in m else 0
    mode |= D.CONTIGUOUS if "contig" in m else 0
    rep, out = run(ctx, D, "spin." + m, U, mode)
    expect = selection.select(COSTS)
    assert rep["profiled"] and rep["selected"] == expect == 1
    p = slice_plan.plan((U,), [(1,)] * 4, 0.1, ctx.n_sm, 0, mode & ~D.ASYNC | (mode & D.ASYNC))
    assert rep["c"] == p.c and rep["n_granules"] == p.Gn
    # every unit productively written exactly once, by the variant the plan says
    owner = slice_plan.productive_cover(p, expect)
    if "async" in m:     # eager chunks ran the best-so-far: valid variants only
        assert set(np.unique(out)) <= {1, 2, 3, 4}
        prof = p.c * (4 if p.mode == slice_plan.FULLY else 1)
        assert np.array_equal(out[:prof], np.array(owner[:prof]) + 1)
        assert rep["eager_units"] >= 0
    else:
        assert np.array_equal(out, np.array(owner) + 1), m
    # scores follow the costs (makespan of c units ~ cost), argmin exact
    sc = rep["score"][:4]
    assert selection.select(sc) == expect


def test_async_eager_starts_with_default(ctx, D):
    # Profiling slow enough (tens of us) that the host poll loop can launch
    # eager chunks before it finishes; with us-scale profiling the paper saw
    # "few or even zero eager dispatches".
    slow = [c * 50 for c in COSTS]
    rep, out = run(ctx, D, "spin.eager", 3000, D.FULLY | D.ASYNC | D.HOST_ORCH, f=0.05, costs=slow, default=3)
    assert rep["selected"] == 1
    assert rep["eager_units"] > 0                 # eager chunks were launched
    eager = out[4 * rep["c"]: 4 * rep["c"] + rep["eager_units"]]
    assert eager[0] == 4                          # first chunk = initial version (default 3)


def test_swap_async_rejected(ctx, D):
    import torch
    ctx.register_spin_variants("spin.swapasync", COSTS, 0)
    out = torch.zeros(600, dtype=torch.int32, device="cuda")
    with pytest.raises(D.DyselError) as e:
        ctx.launch("spin.swapasync", (600,), [out], f=0.1, mode=D.SWAP | D.ASYNC, sandbox_bytes=[2400])
    assert e.value.status == D.ERR_UNSUPPORTED


def test_deactivation_and_cache(ctx, D):
    rep, out = run(ctx, D, "spin.small", 100, D.FULLY, f=0.5, default=2)       # < 128 CTAs
    assert not rep["profiled"] and rep["selected"] == 2 and (out == 3).all()
    rep, out = run(ctx, D, "spin.cache", 600, D.FULLY, f=0.1)
    assert rep["selected"] == 1
    import torch
    o2 = torch.zeros(600, dtype=torch.int32, device="cuda")
    rep2 = ctx.launch("spin.cache", (600,), [o2], mode=D.NO_PROFILE, report=True)
    assert rep2["selected"] == 1 and (o2.cpu().numpy() == 2).all()
    assert ctx.get_selection("spin.cache") == 1
    ctx.reset_selection("spin.cache")
    assert ctx.get_selection("spin.cache") is None


def test_device_path_cache_without_report(ctx, D):
    import torch
    ctx.register_spin_variants("spin.norep", COSTS, 0)
    out = torch.zeros(600, dtype=torch.int32, device="cuda")
    ctx.launch("spin.norep", (600,), [out], f=0.1, mode=D.FULLY)     # no report, never blocks
    assert ctx.get_selection("spin.norep") == 1                      # resolved lazily


def test_timer_calibration(ctx):
    tick, cpn = ctx.timer_calibrate()
    assert 0 < tick <= 2000
    assert 0.3 < cpn < 3.0      # SM clock 0.3-3 GHz


def test_timer_makespan_vs_cuda_events(ctx, D):
    """c-9: a variant's device-measured makespan (earliest %globaltimer CTA
    start .. latest CTA end over its slice) matches the known spin cost of a
    unit (its c CTAs run side by side), and a full one-wave launch of the
    same spin variant timed by CUDA events on the launching stream takes that
    cost plus launch latency (slices >= 100 us, SURVEY c-9)."""
    import torch
    costs = [150_000, 100_000, 300_000, 250_000]
    rep, _ = run(ctx, D, "spin.c9", 600, D.FULLY, costs=costs)
    assert rep["profiled"] and rep["selected"] == 1
    for v, c in enumerate(costs):
        ms = rep["makespan_ns"][v]
        assert c <= ms <= 1.2 * c + 30_000, (v, c, ms)
    out = torch.zeros(100, dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ctx.launch("spin.c9", (100,), [out], mode=D.NO_PROFILE)   # warm
    torch.cuda.synchronize()
    a.record(s)
    ctx.launch("spin.c9", (100,), [out], mode=D.NO_PROFILE)   # cached winner: 100 us per unit
    b.record(s)
    torch.cuda.synchronize()
    ev_ns = a.elapsed_time(b) * 1e6
    assert costs[1] <= ev_ns <= 1.2 * costs[1] + 30_000, ev_ns
    assert abs(ev_ns - rep["makespan_ns"][1]) <= 0.2 * costs[1] + 30_000
    assert set(np.unique(out.cpu().numpy())) == {2}
