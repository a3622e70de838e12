"""GPU parity of the stencil pool through the C ABI vs the
fp64 oracle; composition of DySel launches (c-6) with 3-D work assignment."""
import numpy as np
import pytest

from oracle import slice_plan
from oracle import stencil as ost

pytestmark = pytest.mark.gpu

# (nz, ny, nx); nx % 4 == 0 takes V2's TMA plane ring, the others its z-march column fallback
SHAPES = [(130, 37, 70), (64, 64, 64), (3, 5, 33), (1, 1, 1), (4, 3, 2), (70, 9, 200), (65, 6, 36), (200, 3, 8),
          (2, 2, 4), (37, 100, 260), (17, 8, 128), (16, 9, 132)]
C0, C1 = 0.8125, 0.15625


@pytest.fixture(scope="module")
def ctx(gpu):
    from paper_conf_asplos_changkh16_b200 import dysel
    c = dysel.Context(0)
    yield c
    c.close()


def field(shape, seed):
    return np.random.default_rng(seed).uniform(-1, 1, shape).astype(np.float32)


@pytest.mark.parametrize("shape", SHAPES)
def test_variants_parity_and_bit_identity(ctx, shape):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    a = field(shape, 1)
    inp = torch.from_numpy(a).cuda()
    ref = ost.stencil(a, C0, C1)
    den = ost.stencil_abs(a, C0, C1)
    outs = []
    for v in range(D.DYSEL_STENCIL_NVARIANTS if hasattr(D, "DYSEL_STENCIL_NVARIANTS") else 3):
        out = torch.full_like(inp, float("nan"))
        ctx.stencil_variant(v, inp, out, C0, C1)
        o = out.cpu().numpy()
        assert ost.rel_error(o, ref, den) <= ost.STENCIL_TOL, (v, shape)
        outs.append(o)
    for o in outs[1:]:
        assert np.array_equal(o.view(np.uint32), outs[0].view(np.uint32))


def test_small_integer_exact(ctx):
    import torch
    g = np.random.default_rng(5)
    a = g.integers(-4, 5, (66, 20, 90)).astype(np.float32)
    inp = torch.from_numpy(a).cuda()
    ref = ost.stencil(a, 3.0, 2.0)
    for v in range(3):
        out = torch.empty_like(inp)
        ctx.stencil_variant(v, inp, out, 3.0, 2.0)
        assert np.array_equal(out.cpu().numpy().astype(np.float64), ref), v


@pytest.mark.parametrize("mode_name", ["fully", "fully_async", "hybrid", "hybrid_async", "fully_host"])
def test_dysel_stencil_composition(ctx, mode_name):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    mode = {"fully": D.FULLY, "fully_async": D.FULLY | D.ASYNC, "hybrid": D.HYBRID,
            "hybrid_async": D.HYBRID | D.ASYNC, "fully_host": D.FULLY | D.HOST_ORCH}[mode_name]
    shape = (256, 64, 512)          # 8 x 16 x 4 = 512 granules of (64 x 4 x 64) points
    a = field(shape, 3)
    inp = torch.from_numpy(a).cuda()
    base = torch.empty_like(inp)
    ctx.stencil_variant(0, inp, base, C0, C1)
    out = torch.full_like(inp, float("nan"))
    rep = ctx.stencil(inp, out, C0, C1, f=0.1, mode=mode | D.FORCE_PROFILE, report=True, unit_map=True)
    torch.cuda.synchronize()
    assert rep["profiled"] and 0 <= rep["selected"] < 3
    # every point written exactly once by some variant; all variants bit-identical
    assert np.array_equal(out.cpu().numpy().view(np.uint32), base.cpu().numpy().view(np.uint32))
    assert set(rep["unit_variant"]) <= {0, 1, 2}


def test_deactivated_small_and_invalid(ctx):
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    a = field((8, 8, 40), 4)
    inp = torch.from_numpy(a).cuda()
    out = torch.empty_like(inp)
    rep = ctx.stencil(inp, out, C0, C1, report=True)
    assert not rep["profiled"] and rep["selected"] == D.STENCIL_TILED   # < 128 CTAs: default
    assert ost.rel_error(out.cpu().numpy(), ost.stencil(a, C0, C1), ost.stencil_abs(a, C0, C1)) <= ost.STENCIL_TOL
    with pytest.raises(Exception):
        ctx.stencil(inp, inp, C0, C1)                            # in-place is not a Jacobi step


@pytest.mark.parametrize("shape,f,mode_name", [((256, 64, 512), 0.1, "fully"), ((130, 37, 700), 0.05, "hybrid"),
                                               ((64, 256, 256), 0.3, "fully_contig")])
def test_stencil_plan_matches_oracle(ctx, shape, f, mode_name):
    """a-2 with a 3-D LCM granule (4 x 2 x 64 units): the library's slice plan
    and per-granule producers equal the oracle's (c-5, c-6)."""
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    mode = {"fully": D.FULLY, "hybrid": D.HYBRID, "fully_contig": D.FULLY | D.CONTIGUOUS}[mode_name] | D.FORCE_PROFILE
    nz, ny, nx = shape
    inp = torch.from_numpy(field(shape, 9)).cuda()
    out = torch.empty_like(inp)
    rep = ctx.stencil(inp, out, C0, C1, f=f, mode=mode, report=True, unit_map=True)
    torch.cuda.synchronize()
    U = (-(-nx // 32), -(-ny // 4), nz)
    p = slice_plan.plan(U, [(1, 1, 1), (1, 1, 64), (4, 2, 16)], f, ctx.n_sm, D.STENCIL_TILED, mode)
    assert rep["c"] == p.c and rep["n_granules"] == p.Gn and rep["profiled"] == p.active
    owner = slice_plan.productive_cover(p, rep["selected"])
    assert list(rep["unit_variant"][:p.Gn]) == owner     # sync: profiled slices + the winner's remainder


def test_tma_tile_multi_item_ring(ctx):
    """2,048 V2 items over one persistent wave (4 full round-robin rounds and
    a last round split in z over all CTAs): every CTA's plane ring and its
    mbarrier phases run on across items.  All variants stay bit-identical; the
    oracle is checked on sampled z-planes (boundary, item / granule edges,
    interior)."""
    import torch
    from paper_conf_asplos_changkh16_b200 import dysel as D
    shape = (256, 256, 512)
    a = field(shape, 11)
    inp = torch.from_numpy(a).cuda()
    outs = []
    for v in range(3):
        out = torch.full_like(inp, float("nan"))
        ctx.stencil_variant(v, inp, out, C0, C1)
        outs.append(out)
    torch.cuda.synchronize()
    assert torch.equal(outs[1].view(torch.int32), outs[0].view(torch.int32))
    assert torch.equal(outs[2].view(torch.int32), outs[0].view(torch.int32))
    o = outs[1].cpu().numpy()
    for z in (0, 1, 63, 64, 65, 127, 128, 200, 254, 255):
        lo, hi = max(0, z - 1), min(shape[0], z + 2)
        sub = a[lo:hi]
        ref = ost.stencil(sub, C0, C1)[z - lo]
        den = ost.stencil_abs(sub, C0, C1)[z - lo]
        if 0 < z < shape[0] - 1:   # a 3-plane window's middle plane is interior in z
            assert ost.rel_error(o[z], ref, den) <= ost.STENCIL_TOL, z
        else:
            assert np.array_equal(o[z], a[z]), z


def test_tma_tile_unaligned_view_fallback(ctx):
    """V2 on buffers that are not 16-byte aligned (a view one float into the
    allocation) cannot use TMA: the same items run the z-march column code,
    bit-identical to the other variants and to V2 on aligned buffers."""
    import torch
    shape = (40, 24, 136)
    a = field(shape, 12)
    n = a.size
    big_in = torch.zeros(n + 4, device="cuda")
    big_out = torch.full((n + 4,), float("nan"), device="cuda")
    inp = big_in[1:n + 1].view(shape)
    inp.copy_(torch.from_numpy(a))
    out_u = big_out[1:n + 1].view(shape)
    ctx.stencil_variant(2, inp, out_u, C0, C1)
    out_a = torch.empty(shape, device="cuda")
    ctx.stencil_variant(2, inp.contiguous().clone(), out_a, C0, C1)
    out_z = torch.empty(shape, device="cuda")
    ctx.stencil_variant(1, inp, out_z, C0, C1)
    torch.cuda.synchronize()
    assert torch.equal(out_u.view(torch.int32), out_a.view(torch.int32))
    assert torch.equal(out_u.view(torch.int32), out_z.view(torch.int32))
    assert ost.rel_error(out_u.cpu().numpy(), ost.stencil(a, C0, C1), ost.stencil_abs(a, C0, C1)) <= ost.STENCIL_TOL
    assert torch.isnan(big_out[0]) and torch.isnan(big_out[n + 1])   # nothing written outside the view
