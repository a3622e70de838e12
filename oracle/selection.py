"""Selection oracle.  TEST INFRASTRUCTURE ONLY.

* Per-variant score: makespan = latest end - earliest start over the variant's
  profiling blocks ("Atomic operations are used to mark the earliest and the
  latest cycles among the participating thread blocks", §3.3; Fig. 7b
  P:L899-917), or, with SCORE_CYCLES, sum of per-CTA cycle counts / units
  (reading A-6).
* Winner: argmin; ties -> lowest variant id, which is what one atomicMin on
  (score << 8 | v) produces (readings A-7, A-8).
* Switch margin (reading A-50, the SpMV / SpMTV device paths): the argmin
  replaces the initial version d only if its score is below 8/9 of d's own
  completed score (score[best] * 9 <= score[d] * 8); a dominated d (maximal
  score) never blocks the switch.
* Exhaustive oracle: "the single pure version that delivers the shortest
  runtime" (§4.1): T* = min_v T_v.
* Known-cost model: a variant that spins c_v ns per unit has score ∝ c_v, so
  the expected winner is argmin c_v (c-8 pin).
"""
from __future__ import annotations

U64 = (1 << 64) - 1


def makespan(t_start_min: int, t_end_max: int) -> int:
    return int(t_end_max) - int(t_start_min)


def cycles_per_unit(cycles: int, units: int) -> int:
    return int(cycles) // int(units) if units else U64 >> 8


def pack(score: int, v: int) -> int:
    score = min(int(score), (1 << 56) - 1)
    return (score << 8) | int(v)


def select(scores) -> int:
    """argmin with lowest-id tie-break (the packed-min semantics)."""
    best = min(pack(s, v) for v, s in enumerate(scores))
    return best & 0xFF


def select_with_margin(scores, default: int) -> int:
    """Reading A-50: argmin (packed-min semantics) unless the initial
    version's completed score is within 1/9 of it, then the initial version."""
    best = select(scores)
    cap = (1 << 56) - 1
    sd = min(int(scores[default]), cap)
    if best != default and sd != cap and min(int(scores[best]), cap) * 9 > sd * 8:
        return default
    return best


def exhaustive_best(times) -> int:
    """Index of the best single pure variant."""
    return min(range(len(times)), key=lambda v: (times[v], v))


def within(t, t_star, tol=0.05) -> bool:
    """DySel target: T <= (1 + tol) * T* (BASELINE.json north_star)."""
    return t <= (1.0 + tol) * t_star
