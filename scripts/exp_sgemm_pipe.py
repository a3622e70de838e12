"""Per-call GPU time of pure SGEMM variant calls replayed from a CUDA graph
(host launch cost excluded), and the host cost per call; DYSEL_LIB selects an
A/B build.  Used for profiles/sgemm_pipeline_r2.txt (its stage ablation used
temporary compile-time knobs, since removed).
python scripts/exp_sgemm_pipe.py [MxKxN ...]  (env VARIANTS=2,3)"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_changkh16_b200 import dysel as D
ctx = D.Context(0)
lib = os.path.basename(D.LIB_PATH)
shapes = [tuple(int(v) for v in a.split("x")) for a in (sys.argv[1:] or
          ["1024x992x1056", "1024x32x1056", "1024x256x1056", "1024x2048x1056", "4096x4096x4096"])]
vs = [int(v) for v in os.environ.get("VARIANTS", "2,3").split(",")]
for (M, K, N) in shapes:
    g = torch.Generator().manual_seed(1)
    Ad = (torch.rand(M, K, generator=g) * 2 - 1).cuda(); Bd = (torch.rand(K, N, generator=g) * 2 - 1).cuda()
    C = torch.empty((M, N), device="cuda")
    fl = 2.0 * M * N * K
    for v in vs:
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            for _ in range(3): ctx.sgemm_variant(v, Ad, Bd, C)
        torch.cuda.synchronize()
        reps = 20
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr, stream=st):
            for _ in range(reps): ctx.sgemm_variant(v, Ad, Bd, C)
        gr.replay(); torch.cuda.synchronize()
        ts = []
        for _ in range(10):
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record(); gr.replay(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b) / reps)
        t = float(np.median(ts)) * 1e-3
        h0 = time.perf_counter()
        for _ in range(50): ctx.sgemm_variant(v, Ad, Bd, C)
        h = (time.perf_counter() - h0) / 50
        torch.cuda.synchronize()
        print(f"{lib} {M}x{K}x{N} {D.SGEMM_NAMES[v]:18s} graph {t*1e6:8.2f} us {fl/t/1e12:7.1f} TFLOP/s  host {h*1e6:6.1f} us/call", flush=True)
