"""SpMTV swap-mode timeline on the bench's 2M-row power-law matrix: the pure
variants, the DySel call (b2b), and per-call report timelines (publish, first /
last remainder claim) to see where the single-shot overhead goes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_changkh16_b200 import dysel as D  # noqa: E402
from workloads import d4_powerlaw, uniform_f32  # noqa: E402

ctx = D.Context(0)
A = d4_powerlaw(n=2_000_000, lmax=4096)
rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
plan = ctx.spmv_prepare(rp, col, val, A.n_cols)
x = torch.from_numpy(uniform_f32(61, A.n_rows)).cuda()
y = torch.zeros(A.n_cols, device="cuda")
st = torch.cuda.current_stream()


def b2b(fn, n=20):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(n):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1e3


for v in range(len(D.SPMTV_NAMES)):
    print(D.SPMTV_NAMES[v], f"{b2b(lambda: ctx.spmtv_variant(plan, v, x, y)):.1f} us")
fs = [float(s) for s in os.environ.get("FS", "0.01").split(",")]
for f in fs:
    t = b2b(lambda: ctx.spmtv(plan, x, y, f=f, mode=D.AUTO))
    print(f"f={f}: dysel {t:.1f} us")
    for _ in range(4):
        r = ctx.spmtv(plan, x, y, f=f, mode=D.AUTO, report=True)
        tl = r["timeline_ns"]
        print(f"  sel {r['selected_name']} c {r['c']} units/variant {r['units']}  aborted {r['aborted']} "
              f"publish {tl[1] / 1e3 if tl[1] is not None else None} us, first claim "
              f"{tl[5] / 1e3 if tl[5] is not None else None}, last {tl[6] / 1e3 if tl[6] is not None else None}")
for f in fs:
    t = b2b(lambda: ctx.spmtv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC))
    print(f"f={f} ASYNC: dysel {t:.1f} us")
    for _ in range(4):
        r = ctx.spmtv(plan, x, y, f=f, mode=D.AUTO | D.ASYNC, report=True)
        tl = r["timeline_ns"]
        print(f"  sel {r['selected_name']} eager {r['eager_units']} tail {r['tail_units']} aborted {r['aborted'][:3]} "
              f"publish {tl[1] / 1e3 if tl[1] is not None else None} us, first claim "
              f"{tl[5] / 1e3 if tl[5] is not None else None}, last {tl[6] / 1e3 if tl[6] is not None else None}")
for f in fs:
    for m, nm in ((D.AUTO, "sync"), (D.AUTO | D.ASYNC, "async")):
        sels = [ctx.spmtv(plan, x, y, f=f, mode=m, report=True)["selected_name"] for _ in range(20)]
        print(f"f={f} {nm}: selections of 20", {n: sels.count(n) for n in sorted(set(sels))})


def per_call(fn, n=30, sync=False):
    ts = []
    for _ in range(n):
        if sync:
            torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        fn()
        e1.record(st)
        ts.append((e0, e1))
    torch.cuda.synchronize()
    v = sorted(a.elapsed_time(b) * 1e3 for a, b in ts)
    return v[len(v) // 2], v[0], v[-1]


for f in fs:
    for m, nm in ((D.AUTO, "sync"), (D.AUTO | D.ASYNC, "async")):
        for sy in (False, True):
            md, lo, hi = per_call(lambda: ctx.spmtv(plan, x, y, f=f, mode=m), sync=sy)
            print(f"f={f} {nm} {'idle-start' if sy else 'b2b'} per-call median {md:.1f} min {lo:.1f} max {hi:.1f}")
md, lo, hi = per_call(lambda: ctx.spmtv_variant(plan, 1, x, y))
print(f"scatter_warp pure per-call median {md:.1f} min {lo:.1f} max {hi:.1f}")
for m, nm in ((D.AUTO, "sync"), (D.AUTO | D.ASYNC, "async")):
    rows = []
    for _ in range(20):
        r = ctx.spmtv(plan, x, y, f=fs[0], mode=m, report=True)
        sc = [s / 1e3 if s < 2 ** 55 else None for s in r["score"][:3]]
        rows.append((r["selected_name"], sc, [b / 1e3 for b in r["busy_ns"][:3]]))
    print(nm, "score us (thread, warp, segment) / busy us:")
    for row in rows[:20]:
        print("  ", row[0], row[1], row[2])
