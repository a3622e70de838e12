"""Selection accuracy sweep (default pool and all formats): for a spread of
synthetic matrices, the pure variants' b2b times and DySel's pick over 10
calls at f = 0.001 and 0.01 (exact = the pure best, within 5% of it)."""
import os, sys, collections, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from bench import time_b2b
from paper_conf_asplos_changkh16_b200 import dysel as D
from workloads import (csr_from_lengths, d3_fem, d4_powerlaw, d6_diag, d6_random, laplacian_2d, powerlaw_lengths,
                       uniform_f32)
ctx = D.Context(0); s = torch.cuda.current_stream()
def fixed(n, L, seed):
    return csr_from_lengths(np.full(n, L, np.int64), n, seed, seed + 1)
def uni(n, lo, hi, seed):
    return csr_from_lengths(np.random.default_rng(seed).integers(lo, hi + 1, n), n, seed + 1, seed + 2)
MATS_ALL = [("fem_2.25M", lambda: d3_fem(grid=1500)), ("powerlaw_2M", lambda: d4_powerlaw(n=2_000_000, lmax=4096)),
        ("d6_random", d6_random), ("d6_diag", d6_diag), ("rows5_4M", lambda: fixed(4_000_000, 5, 11)),
        ("rows50_1M", lambda: fixed(1_000_000, 50, 12)), ("rows500_200k", lambda: fixed(200_000, 500, 13)),
        ("uni1-64_2M", lambda: uni(2_000_000, 1, 64, 14)), ("uni1-2000_200k", lambda: uni(200_000, 1, 2000, 15)),
            ("laplace5_4M", lambda: laplacian_2d(2000))]
MATS = [m for m in MATS_ALL if not os.environ.get("ONLY") or m[0] in os.environ["ONLY"].split(",")]
res = []
for name, mk in MATS:
    A = mk()
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    x = torch.from_numpy(uniform_f32(3, A.n_cols)).cuda(); y = torch.empty(A.n_rows, device="cuda")
    for pool, kw in (("default", {}), ("all", {"formats": D.FMT_ALL})):
        try:
            plan = ctx.spmv_prepare(rp, col, val, A.n_cols, default=D.SPMV_DEFAULT_AUTO, **kw)
        except Exception as e:
            print(name, pool, "prepare failed", e, flush=True); continue
        T = {D.SPMV_NAMES[v]: time_b2b(lambda: ctx.spmv_variant(plan, v, x, y), 10, s) for v in plan.variant_ids}
        best = min(T, key=T.get)
        for f in (0.001, 0.01):
            c = collections.Counter(); prof = 0
            for _ in range(10):
                r = ctx.spmv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC, report=True)
                c[r["selected_name"]] += 1; prof += r["profiled"]
            within = sum(n for v, n in c.items() if T[v] <= 1.05 * T[best])
            td = time_b2b(lambda: ctx.spmv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC), 10, s)
            line = {"mat": name, "pool": pool, "f": f, "profiled": prof, "best": best,
                    "pure_us": {k: round(v * 1e6, 1) for k, v in T.items()}, "picks": dict(c),
                    "exact": c[best], "within5": within, "default": D.SPMV_NAMES[plan.info.default_variant],
                    "dysel_us": round(td * 1e6, 1), "ovh_pct": round((td / T[best] - 1) * 100, 1)}
            res.append(line)
            print(json.dumps(line), flush=True)
        plan.destroy()
    del rp, col, val, A
