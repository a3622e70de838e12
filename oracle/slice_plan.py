"""Slice planning, mode resolution and ticket order.
TEST INFRASTRUCTURE ONLY.  Integer work: the CUDA runtime must agree bit-exactly.

Paper passages followed, in order:
  * safe-point analysis: "normalized to the least common multiple (LCM) among
    all related assignments ... the number of work-groups in each variant ...
    defined as the LCM divided by each work assignment factor"; then "multiply
    ... by a constant to make the total workload become a multiple of the
    number of ... SMs" (§3.4); worked example WA 3:2 => 2 and 3
    work-groups (§2.2, Fig. 3).
  * small-workload deactivation: "profiling-based kernel selection is
    deactivated for small workload", < 128 work-groups rare (§2.1).
  * profiling activation flag (§3.1).
  * modes: fully-productive = K disjoint productive slices; hybrid = all run
    the same slice, only the first (initial) version writes the output, the
    rest write sandboxes; swap = private outputs, no async (§2.2,
    Table 1).
  * uniform-workload / side-effect analyses choose hybrid / swap
    (§3.4) -> replaced by variant flags (readings A-10/A-11/A-13).

Readings: A-1 c = floor(f*G_n/K) in fp64; A-2 SM rounding
(below); A-3 deactivation when the default variant's full grid has < 128 CTAs
or c = 0; A-4 hybrid productive variant = default; A-24 fully-mode granules
interleaved (j mod K) unless CONTIGUOUS.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

# mode bits (restated from DESIGN.md §Boundary; the oracle does not include the C header)
FULLY, HYBRID, SWAP, AUTO = 0, 1, 2, 3
ASYNC = 4
NO_PROFILE = 8
HOST_ORCH = 16
FORCE_PROFILE = 32
CONTIGUOUS = 64
SCORE_CYCLES = 128

V_ATOMICS = 1
V_NONUNIFORM = 2

ROLE_PRODUCTIVE, ROLE_SANDBOX, ROLE_BATCH, ROLE_PRIVATE = 0, 1, 2, 3

MIN_CTAS = 128
# reading A-52 (SpMV device path, grouped profiling): a slice of fewer than
# MIN_PROF_UNITS units per variant grows to MIN_PROF_UNITS when K x
# MIN_PROF_UNITS x MIN_PROF_FRAC <= G_n (applied after A-2 and activation)
MIN_PROF_UNITS = 12
MIN_PROF_FRAC = 16
# reading A-3c (SpMV device path): a matrix below MIN_PROF_BYTES of
# algorithmic bytes is not profiled unless FORCE_PROFILE
MIN_PROF_BYTES = 64 << 20


class Unsupported(Exception):
    pass


@dataclass
class Slice:
    variant: int
    role: int
    granules: list  # linear granule ids, in slice order


@dataclass
class Plan:
    K: int
    g: tuple
    G: tuple
    Gn: int
    h: list            # CTAs per granule per variant
    c: int
    active: bool
    mode: int          # resolved FULLY / HYBRID / SWAP
    slices: list = field(default_factory=list)
    remainder: list = field(default_factory=list)   # granule ids for the selected variant

    def profiled_ctas(self, v):
        return self.c * self.h[v]


def lcm_list(xs):
    out = 1
    for x in xs:
        out = out * x // math.gcd(out, x)
    return out


def resolve_mode(mode, vflags):
    base = mode & 3
    if base == AUTO:
        if any(f & V_ATOMICS for f in vflags):
            base = SWAP
        elif any(f & V_NONUNIFORM for f in vflags):
            base = HYBRID
        else:
            base = FULLY
    if base == SWAP and (mode & ASYNC):
        raise Unsupported("swap-based profiling cannot run asynchronously (Table 1, P:L735-739)")
    return base


def plan(U, wa, f, n_sm, default_variant, mode, vflags=None, min_ctas=MIN_CTAS, wave_units=0,
         min_c=0, work_bytes=None) -> Plan:
    """U: units per dim (3-tuple); wa: per-variant 3-tuples of units per CTA.

    wave_units (reading A-3b, SpMV device path): profiling is also off when
    the whole grid (G_n granules) fits in one wave of the default variant —
    everything runs concurrently, so no remainder can benefit.
    min_c (reading A-52, SpMV device path with grouped profiling: pass
    MIN_PROF_UNITS): an active slice smaller than min_c granules per variant
    grows to min_c when K * min_c * MIN_PROF_FRAC <= G_n.
    work_bytes (reading A-3c, SpMV device path): when given and below
    MIN_PROF_BYTES, profiling is off unless FORCE_PROFILE.
    """
    K = len(wa)
    vflags = vflags or [0] * K
    if not (1 <= K <= 16) or not (0.0 <= f <= 1.0) or not (0 <= default_variant < K):
        raise ValueError("invalid plan arguments")
    U = tuple(int(u) for u in U) + (1,) * (3 - len(U))
    wa = [tuple(int(w) for w in v) + (1,) * (3 - len(v)) for v in wa]
    if any(w <= 0 for v in wa for w in v):
        raise ValueError("wa must be positive")
    g = tuple(lcm_list([v[d] for v in wa]) for d in range(3))
    G = tuple(-(-U[d] // g[d]) for d in range(3))
    Gn = G[0] * G[1] * G[2]
    h = [(g[0] // v[0]) * (g[1] // v[1]) * (g[2] // v[2]) for v in wa]
    rmode = resolve_mode(mode, vflags)
    c = int(math.floor(float(f) * float(Gn) / float(K)))
    # reading A-2: round c down so the smallest per-variant CTA count is a
    # multiple of floor(#SM / K) once it reaches it
    q = n_sm // K
    if q > 0:
        hmin = min(h)
        cq = q // math.gcd(q, hmin)
        if c >= cq:
            c = (c // cq) * cq
    default_ctas = 1
    for d in range(3):
        default_ctas *= -(-U[d] // wa[default_variant][d])
    active = (not (mode & NO_PROFILE)) and K >= 2 and Gn > 0
    if active:
        if mode & FORCE_PROFILE:
            if c == 0:
                c = 1 if (Gn >= K if rmode == FULLY else Gn >= 1) else 0
            active = c >= 1
        else:
            active = c >= 1 and default_ctas >= min_ctas and Gn > wave_units and (
                work_bytes is None or work_bytes >= MIN_PROF_BYTES)
    if active and min_c and c < min_c and K * min_c * MIN_PROF_FRAC <= Gn:
        c = min_c
    p = Plan(K, g, G, Gn, h, c if active else 0, active, rmode)
    if not active:
        p.remainder = list(range(Gn))
        return p
    if rmode == FULLY:
        for v in range(K):
            if mode & CONTIGUOUS:
                gr = [v * c + i for i in range(c)]
            else:
                gr = [v + K * i for i in range(c)]
            p.slices.append(Slice(v, ROLE_PRODUCTIVE, gr))
        p.remainder = list(range(K * c, Gn))
    elif rmode == HYBRID:
        for v in range(K):
            role = ROLE_PRODUCTIVE if v == default_variant else ROLE_SANDBOX
            p.slices.append(Slice(v, role, list(range(c))))
        p.remainder = list(range(c, Gn))
    else:  # SWAP
        for v in range(K):
            p.slices.append(Slice(v, ROLE_PRIVATE, list(range(c))))
        p.remainder = list(range(c, Gn))
    return p


def productive_cover(p: Plan, selected: int):
    """granule -> variant that productively computed it (c-6 / c-7).  In swap
    mode the winner's private prefix becomes the output."""
    owner = [-1] * p.Gn
    for s in p.slices:
        if s.role == ROLE_PRODUCTIVE or (s.role == ROLE_PRIVATE and s.variant == selected):
            for j in s.granules:
                if owner[j] != -1:
                    raise AssertionError("granule produced twice")
                owner[j] = s.variant
    for j in p.remainder:
        if owner[j] != -1:
            raise AssertionError("remainder overlaps a productive slice")
        owner[j] = selected
    return owner


def table1_counts(p: Plan):
    """(productive profiled outputs, extra output spaces) — Table 1."""
    prod = sum(1 for s in p.slices if s.role == ROLE_PRODUCTIVE)
    extra = sum(1 for s in p.slices if s.role in (ROLE_SANDBOX, ROLE_PRIVATE))
    if p.mode == SWAP:
        prod = 1 if p.slices else 0
    return prod, extra


# ------------------------------------------------------------ device ticket order
def n_tickets(p: Plan) -> int:
    """Tickets of the persistent SpMV dispatcher (SURVEY §8a device protocol)."""
    if not p.active:
        return p.Gn
    if p.mode == HYBRID:
        return p.Gn + (p.K - 1) * p.c
    return p.Gn


def ticket(p: Plan, t: int, mode: int, default_variant: int):
    """(granule, variant or None for 'selected', role) claimed by ticket t.
    Profiling tickets come first (priority, P:L666-668 / reading A-11)."""
    K, c = p.K, p.c
    if not p.active:
        return t, None, ROLE_BATCH
    P = K * c
    if t < P:
        if p.mode == FULLY:
            if mode & CONTIGUOUS:
                return t, t // c, ROLE_PRODUCTIVE
            return t, t % K, ROLE_PRODUCTIVE
        v = t % K
        return t // K, v, (ROLE_PRODUCTIVE if v == default_variant else ROLE_SANDBOX)
    if p.mode == FULLY:
        return t, None, ROLE_BATCH
    return t - (K - 1) * c, None, ROLE_BATCH


def granule_units(p: Plan, j: int, U):
    """Units (ux, uy, uz) covered by linear granule j (x fastest), clipped to U."""
    U = tuple(U) + (1,) * (3 - len(U))
    gx = j % p.G[0]
    gy = (j // p.G[0]) % p.G[1]
    gz = j // (p.G[0] * p.G[1])
    out = []
    for z in range(gz * p.g[2], min(U[2], (gz + 1) * p.g[2])):
        for y in range(gy * p.g[1], min(U[1], (gy + 1) * p.g[1])):
            for x in range(gx * p.g[0], min(U[0], (gx + 1) * p.g[0])):
                out.append((x, y, z))
    return out


# ----------------------------------------------------- SpMV unit order (A-40, A-45)
UNIT_ROWS = 256
HEAVY_UNIT_NNZ = 8192
LONG_ROW = 1024


def unit_order(row_ptr, n_sm):
    """The SpMV plan's unit order (readings A-40 and A-45): returns
    (seq, n_light) or (None, n_units) for index order.

    The paper's NDRange runs work-groups in index order and profiles a prefix
    (P:L865-869); on a heavy-tailed matrix the device path instead (A-45)
    profiles, and lets the not-yet-proven initial version run eagerly, only
    LIGHT units, and the winner runs the others first, longest first (A-40).
      unit u = rows [256 u, 256 u + 256); nnz_u, max_u = its nonzeros / longest row
      thr  = max(8192, 4 * floor(nnz / n_units))       (heavy: nnz_u >= thr)
      lcap = max(1024, 8 * ceil(nnz / n_rows))          (long:  max_u > lcap)
      applied when n_units >= 4 * n_sm and some unit is heavy or long;
      seq = light units in index order ++ the others by nnz_u descending (stable).
    Integer work: the library must agree bit-exactly."""
    rp = [int(v) for v in row_ptr]
    n = len(rp) - 1
    nnz = rp[-1] if n >= 0 else 0
    nu = (n + UNIT_ROWS - 1) // UNIT_ROWS
    if nu == 0:
        return None, 0
    mean = nnz // nu
    thr = max(HEAVY_UNIT_NNZ, 4 * mean)
    lcap = max(LONG_ROW, 8 * ((nnz + n - 1) // n)) if n > 0 else LONG_ROW
    if nu < 4 * n_sm:
        return None, nu
    light, rest, nz = [], [], []
    for u in range(nu):
        r0, r1 = u * UNIT_ROWS, min((u + 1) * UNIT_ROWS, n)
        cnt = rp[r1] - rp[r0]
        mx = max(rp[r + 1] - rp[r] for r in range(r0, r1))
        nz.append(cnt)
        (light if (cnt < thr and mx <= lcap) else rest).append(u)
    if not rest:
        return None, nu
    rest = sorted(rest, key=lambda u: -nz[u])      # Python's sort is stable
    return light + rest, len(light)
