"""Diagnostic: one C2 pair-job under the AUTO selector with the server's debug
log on (SLATE_DEBUG=1 in the environment): selection, splits, resizes."""
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
w = bench.make_c2(S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
pb = sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
print("arrival_ms", w.arrival_ms, file=sys.stderr, flush=True)
for i in range(2):
    r = bench.run_schedule("slate", w, sA, sB, kA, kB, S)
    print("makespan", r[0], "turn a", r[1], "turn b", r[2], file=sys.stderr, flush=True)
