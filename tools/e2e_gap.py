"""Development probe: where the end-to-end C2 step loses time against the
device-timed makespan -- the same AUTO pair-job back to back, wall clock vs
device span, without the host copies (the bench's e2e adds them)."""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
w = bench.make_c2(S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.arrival_ms = 0.0
for _ in range(3):
    bench.run_schedule("slate", w, sA, sB, kA, kB, S)
n = 10
spans, walls, subs = [], [], []
for _ in range(n):
    t0 = time.perf_counter()
    ia = bench.submit(sA, kA, w.a, placement=S.PLACE_AUTO)
    ib = bench.submit(sB, kB, w.b, placement=S.PLACE_AUTO)
    t1 = time.perf_counter()
    sA.sync(0)
    sB.sync(0)
    t2 = time.perf_counter()
    qa, qb = bench.collect(sA, ia), bench.collect(sB, ib)
    a0, a1 = bench.span(qa)
    b0, b1 = bench.span(qb)
    spans.append(max(a1, b1) - min(a0, b0))
    walls.append((t2 - t0) * 1e3)
    subs.append((t1 - t0) * 1e3)
print("device span ms", [round(x, 2) for x in spans])
print("wall ms (submit + sync)", [round(x, 2) for x in walls])
print("submit ms", [round(x, 2) for x in subs])
