"""Diagnostic: pair-job makespan under forced co-run splits (tenant B on the top
s SMs, grown to all SMs when A's job drains), for the C2 or C3 workload.

    SLATE_SWEEP_SPLITS=24,37,49 python tools/pair_sweep.py c2
"""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
w = {"c2": bench.make_c2, "c3": bench.make_c3}[cfg](S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
out = {}
for base in ("seq_cuda", "seq_slate"):
    bench.run_schedule(base, w, sA, sB, kA, kB, S)
    out[base] = bench.median_schedule(base, w, sA, sB, kA, kB, S, flush, 3)[0]
print(cfg, {k: round(v, 3) for k, v in out.items()}, flush=True)
for s_b in [int(x) for x in os.environ.get("SLATE_SWEEP_SPLITS", "24,32,40,48,56,64,72,80").split(",")]:
    w.split = s_b
    bench.run_schedule("slate_forced", w, sA, sB, kA, kB, S)
    r = bench.median_schedule("slate_forced", w, sA, sB, kA, kB, S, flush, 3)
    out[s_b] = {"makespan": round(r[0], 3), "G_vs_seq_cuda": round(out["seq_cuda"] / r[0], 4),
                "G_vs_seq_slate": round(out["seq_slate"] / r[0], 4),
                "turnaround_a": round(r[1], 3), "turnaround_b": round(r[2], 3),
                "topups": sum(q["n_topups"] for q in r[3] + r[4])}
    print(s_b, out[s_b], flush=True)
json.dump(out, open(os.environ.get("SLATE_SWEEP_OUT", "gpurun_out/%s_sweep.json" % cfg), "w"), indent=1)
