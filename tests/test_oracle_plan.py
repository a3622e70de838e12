"""Pins for oracle/slice_plan.py and oracle/selection.py (SURVEY c-5, c-7, c-8)."""
import itertools
import os

import pytest

from oracle import selection as S
from oracle import slice_plan as P

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_fig3_worked_example():
    # WA 3:2 -> A launches 2 WGs, B launches 3.
    for line in open(os.path.join(GOLD, "fig3_worked_example.txt")):
        if line.startswith("#") or not line.strip():
            continue
        lhs, rhs = line.split("->")
        wa_a, wa_b = map(int, lhs.split())
        g, n_a, n_b = map(int, rhs.split())
        p = P.plan((600,), [(wa_a,), (wa_b,)], 0.1, 148, 0, P.FULLY | P.FORCE_PROFILE)
        assert p.g[0] == g
        assert p.h == [n_a, n_b]


def test_table1_counts():
    rows = {}
    for line in open(os.path.join(GOLD, "table1_modes.txt")):
        if line.startswith("#") or not line.strip():
            continue
        m, prod, extra, asy = line.split()
        rows[m] = (prod, extra, asy)
    for K in (2, 3, 4, 7):
        wa = [(1,)] * K
        for name, mode in (("fully", P.FULLY), ("hybrid", P.HYBRID), ("swap", P.SWAP)):
            p = P.plan((10000,), wa, 0.05, 148, 0, mode | P.FORCE_PROFILE)
            prod, extra = P.table1_counts(p)
            e_prod = K if rows[name][0] == "K" else int(rows[name][0])
            e_extra = {"0": 0, "K-1": K - 1, "K": K}[rows[name][1]]
            assert prod == e_prod and extra == e_extra, (name, K)
            if rows[name][2] == "no":
                with pytest.raises(P.Unsupported):
                    P.plan((10000,), wa, 0.05, 148, 0, mode | P.ASYNC)
            else:
                P.plan((10000,), wa, 0.05, 148, 0, mode | P.ASYNC)


def test_fig6_defaults_are_fully_async():
    vals = dict(l.split() for l in open(os.path.join(GOLD, "fig6_api_defaults.txt"))
                if l.strip() and not l.startswith("#"))
    assert vals == {"profiling": "true", "mode": "fully_async"}
    default_mode = P.FULLY | P.ASYNC
    p = P.plan((10000,), [(1,)] * 4, 0.02, 148, 0, default_mode)
    assert p.active and p.mode == P.FULLY


def test_small_workload_deactivation():
    # < 128 work-groups => profiling off.
    p = P.plan((127,), [(1,)] * 2, 1.0, 148, 0, P.FULLY)
    assert not p.active
    p = P.plan((128,), [(1,)] * 2, 0.5, 148, 0, P.FULLY)
    assert p.active
    p = P.plan((128,), [(1,)] * 2, 0.5, 148, 0, P.FULLY | P.NO_PROFILE)   # activation flag
    assert not p.active and p.remainder == list(range(128))


def test_single_wave_deactivation_reading_a3b():
    # D3: 574 units fit in one wave (8 CTAs/SM x 148 SMs) -> off; D4 does not
    assert not P.plan((574,), [(1,)] * 4, 0.02, 148, 0, P.FULLY, wave_units=8 * 148).active
    assert P.plan((574,), [(1,)] * 4, 0.02, 148, 0, P.FULLY | P.FORCE_PROFILE, wave_units=8 * 148).active
    assert P.plan((39063,), [(1,)] * 3, 0.02, 148, 0, P.HYBRID, wave_units=4 * 148).active


def test_survey_sgemm_d2m_numbers():
    # SGEMM medium 1024x992x1056, unit = 32x32 tile: U = (33, 32); tilings
    # 64x64 (2,2), 128x128 (4,4), 128x64 (N=64 -> 2, M=128 -> 4), 128x128.
    U = (33, 32)
    wa = [(2, 2), (4, 4), (2, 4), (4, 4)]
    p = P.plan(U, wa, 0.02, 148, 0, P.FULLY)
    assert p.g == (4, 4, 1) and p.G == (9, 8, 1) and p.Gn == 72
    assert not p.active                                   # c = floor(0.36) = 0
    p = P.plan(U, wa, 0.06, 148, 0, P.FULLY)
    assert p.active and p.c == 1 and p.h == [4, 1, 2, 1]


def test_sm_rounding_reading_a2():
    # D4-like: G_n = 39063, K = 3, f = 0.02: c = 260 -> multiple of floor(148/3) = 49
    p = P.plan((39063,), [(1,)] * 3, 0.02, 148, 0, P.HYBRID)
    assert p.c == 245
    p = P.plan((574,), [(1,)] * 4, 0.02, 148, 0, P.FULLY)     # D3: c = 2
    assert p.c == 2


def test_small_matrix_deactivation_reading_a3c():
    # D6 diagonal: 2^21 rows, 1 nnz: 8*2^21 + 4*(2^21+1) + 4*2^21 + 4*2^21 = 41,943,044 B < 64 MiB
    b = 8 * 2 ** 21 + 4 * (2 ** 21 + 1) + 4 * 2 ** 21 + 4 * 2 ** 21
    assert b == 41943044
    assert not P.plan((8192,), [(1,)] * 5, 0.02, 148, 0, P.FULLY, work_bytes=b).active
    assert P.plan((8192,), [(1,)] * 5, 0.02, 148, 0, P.FULLY | P.FORCE_PROFILE, work_bytes=b).active
    assert P.plan((8192,), [(1,)] * 5, 0.02, 148, 0, P.FULLY, work_bytes=64 << 20).active      # boundary: on
    assert not P.plan((8192,), [(1,)] * 5, 0.02, 148, 0, P.FULLY, work_bytes=(64 << 20) - 1).active
    assert P.plan((8192,), [(1,)] * 5, 0.02, 148, 0, P.FULLY).active                          # rule not applied


def test_min_profiling_slice_reading_a52():
    # D3x default pool: G_n = 8789, K = 5, f = 0.002 -> c = 3 < 12, and
    # 5 * 12 * 16 = 960 <= 8789 -> c = 12 (hand computed)
    p = P.plan((8789,), [(1,)] * 5, 0.002, 148, 0, P.FULLY, min_c=P.MIN_PROF_UNITS)
    assert p.active and p.c == 12
    assert p.slices[0].granules == [5 * i for i in range(12)] and p.remainder[0] == 60
    assert P.plan((8789,), [(1,)] * 5, 0.002, 148, 0, P.FULLY).c == 3        # without the rule
    # D4 at f = 0.001: c = floor(39063 * 0.001 / 4) = 9 -> 12; f = 0.02 -> 195 (A-2: multiple of 37) unchanged
    assert P.plan((39063,), [(1,)] * 4, 0.001, 148, 0, P.HYBRID, min_c=12).c == 12
    assert P.plan((39063,), [(1,)] * 4, 0.02, 148, 0, P.HYBRID, min_c=12).c == 185
    # small grid: K * 12 * 16 = 768 > 700 -> the slice stays as computed
    assert P.plan((700,), [(1,)] * 4, 0.02, 148, 0, P.FULLY, min_c=12).c == 3
    # boundary: G_n = 768 grows, 767 does not
    assert P.plan((768,), [(1,)] * 4, 0.02, 148, 0, P.FULLY, min_c=12).c == 12
    assert P.plan((767,), [(1,)] * 4, 0.02, 148, 0, P.FULLY, min_c=12).c == 3
    # inactive plans are untouched
    assert P.plan((8789,), [(1,)] * 5, 0.002, 148, 0, P.FULLY | P.NO_PROFILE, min_c=12).c == 0


@pytest.mark.parametrize("mode", [P.FULLY, P.FULLY | P.CONTIGUOUS, P.HYBRID, P.SWAP])
def test_cover_invariant_exhaustive(mode):
    for U in (1, 5, 17, 64):
        for K in (2, 3, 4):
            for wa in itertools.product((1, 2, 3, 4, 8), repeat=K):
                for f in (0.1, 0.5, 1.0):
                    p = P.plan((U,), [(w,) for w in wa], f, 148, 0, mode | P.FORCE_PROFILE)
                    for sel in range(K):
                        owner = P.productive_cover(p, sel)
                        assert all(o >= 0 for o in owner)            # each granule exactly once
                    if p.active:
                        assert p.c * K <= max(1, f * p.Gn) + 1e-9 or p.c == 1
                        if p.mode == P.FULLY:
                            assert len(p.remainder) == p.Gn - K * p.c
                        else:
                            assert len(p.remainder) == p.Gn - p.c
                        # per-variant CTA count = c * lcm / wa
                        for v in range(K):
                            assert p.profiled_ctas(v) == p.c * p.g[0] // wa[v]


def test_ticket_order_covers_granules():
    for mode in (P.FULLY, P.FULLY | P.CONTIGUOUS, P.HYBRID):
        p = P.plan((50,), [(1,)] * 3, 0.3, 148, 1, mode | P.FORCE_PROFILE)
        seen = {}
        for t in range(P.n_tickets(p)):
            j, v, role = P.ticket(p, t, mode, 1)
            if role in (P.ROLE_PRODUCTIVE, P.ROLE_BATCH):
                assert j not in seen
                seen[j] = v
        assert sorted(seen) == list(range(p.Gn))
        # profiling tickets come first
        roles = [P.ticket(p, t, mode, 1)[2] for t in range(P.n_tickets(p))]
        first_batch = roles.index(P.ROLE_BATCH)
        assert all(r == P.ROLE_BATCH for r in roles[first_batch:])
        assert first_batch == 3 * p.c


def test_granule_units_2d_edges():
    p = P.plan((33, 32), [(2, 2), (4, 4)], 0.5, 148, 0, P.FULLY)
    allu = [u for j in range(p.Gn) for u in P.granule_units(p, j, (33, 32))]
    assert sorted(allu) == sorted((x, y, 0) for x in range(33) for y in range(32))
    assert len(P.granule_units(p, 8, (33, 32))) == 4      # last column granule: 1 x 4 units


def test_mode_resolution():
    assert P.resolve_mode(P.AUTO, [0, 0]) == P.FULLY
    assert P.resolve_mode(P.AUTO, [0, P.V_NONUNIFORM]) == P.HYBRID
    assert P.resolve_mode(P.AUTO, [P.V_ATOMICS, P.V_NONUNIFORM]) == P.SWAP
    with pytest.raises(P.Unsupported):
        P.resolve_mode(P.AUTO | P.ASYNC, [P.V_ATOMICS])
    assert P.resolve_mode(P.HYBRID | P.ASYNC, [P.V_ATOMICS]) == P.HYBRID   # user override wins


def test_selection_packed_argmin():
    assert S.select([5, 3, 3, 9]) == 1              # tie -> lowest id (A-8)
    assert S.select([7]) == 0
    assert S.pack(3, 2) < S.pack(3, 5) < S.pack(4, 0)
    assert S.makespan(100, 350) == 250
    assert S.cycles_per_unit(1000, 4) == 250
    # known-cost variants: c_v ns per unit => argmin c_v
    costs = [40, 10, 25, 10]
    units = 7
    assert S.select([c * units for c in costs]) == 1
    assert S.exhaustive_best([3.0, 1.0, 1.0]) == 1
    assert S.within(1.04, 1.0) and not S.within(1.06, 1.0)


def test_partition_balanced_and_cover():
    import numpy as np
    from oracle import partition
    from workloads import d4_powerlaw, identity
    I = identity(256 * 40)
    assert partition.partition_rows(I.row_ptr, 4) == [0, 2560, 5120, 7680, 10240]
    A = d4_powerlaw(n=20000, lmax=1000)
    for G in (2, 3, 8):
        b = partition.partition_rows(A.row_ptr, G)
        assert b[0] == 0 and b[-1] == A.n_rows and all(x <= y for x, y in zip(b, b[1:]))
        assert all(x % 256 == 0 for x in b[:-1])
        nz = np.diff(A.row_ptr.astype(np.int64)[b])
        # each shard within one unit's nnz of the ideal share
        assert np.abs(nz - A.nnz / G).max() <= A.row_ptr[-1] / A.n_rows * 256 * 4 + A.lengths().max()


def test_unit_order_hand_example():
    """Readings A-40 / A-45 restated on a hand-built matrix (n_sm = 1, so the
    rule applies from 4 units): 6 units of 256 rows; unit 1 holds one
    2,000-entry row (long: > max(1024, 8 x ceil(mean row))), unit 4 holds
    256 rows of 40 entries (10,240 >= max(8192, 4 x floor(nnz / 6))): heavy.
    seq = light units in index order, then heavy / long by nonzeros desc."""
    import numpy as np
    L = np.full(6 * 256, 2)
    L[256 + 7] = 2000
    L[4 * 256:5 * 256] = 40
    rp = np.concatenate([[0], np.cumsum(L)])
    nnz = int(rp[-1])   # thr = max(8192, 4 * (14798 // 6)) = 9864, lcap = max(1024, 8 * 10) = 1024
    assert nnz == 4 * 512 + (255 * 2 + 2000) + 256 * 40
    seq, n_light = P.unit_order(rp, 1)
    # unit nnz: u1 = 2510, u4 = 10240 -> rest sorted desc: [4, 1]
    assert seq == [0, 2, 3, 5, 4, 1] and n_light == 4
    # fewer than 4 units per SM: index order
    assert P.unit_order(rp, 2) == (None, 6)
    # uniform rows: nothing heavy or long -> index order
    rp2 = np.arange(0, 2 * 6 * 256 + 1, 2)
    assert P.unit_order(rp2, 1) == (None, 6)


def test_select_with_margin_hand_cases():
    """A-50 on hand cases: 1/9 margin around the initial version's score."""
    cap = (1 << 56) - 1
    assert S.select_with_margin([100, 90, 95], 0) == 0      # 90 * 9 = 810 > 800: within the margin
    assert S.select_with_margin([100, 88, 95], 0) == 1      # 88 * 9 = 792 <= 800: switch
    assert S.select_with_margin([100, 89, 95], 0) == 0      # 89 * 9 = 801 > 800: keep (boundary)
    assert S.select_with_margin([cap, 500, 400], 0) == 2    # a dominated default never blocks the switch
    assert S.select_with_margin([300, 200, 100], 2) == 2    # the default is the argmin
    assert S.select_with_margin([50, 50, 60], 1) == 1       # tie: the default stays (no switch to a tie)
