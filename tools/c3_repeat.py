"""Development probe: the C3 co-run (GEMM 8192^3 + copy 4 GiB arriving at 25%)
under Slate AUTO, repeated, with each run's makespan and per-job spans -- the
spread of the bench's C3 median between runs.

    python tools/c3_repeat.py [runs]"""
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

runs = int(sys.argv[1]) if len(sys.argv) > 1 else 30
dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
w = bench.make_c3(S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
pb = sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.split = 0
w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
out = []
for i in range(runs + 3):
    bench.flush_l2(flush)
    mk, ta, tb, qa, qb, ja, jb = bench.run_schedule("slate", w, sA, sB, kA, kB, S)
    if i < 3:
        continue
    qa0, qb0 = qa[0], qb[0]
    out.append({"makespan": round(mk, 4), "gemm": round(ja, 4), "copy": round(jb, 4),
                "gemm_resizes": list(zip(qa0["resize_kind"], [round(v, 1) for v in qa0["resize_us"]])),
                "gemm_topups": qa0["n_topups"], "copy_range": (qb0["sm_lo"], qb0["sm_hi"])})
for r in out:
    print(json.dumps(r))
ms = [r["makespan"] for r in out]
print(json.dumps({"median": statistics.median(ms), "min": min(ms), "max": max(ms),
                  "gemm_median": statistics.median(r["gemm"] for r in out)}))
