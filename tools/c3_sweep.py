"""Diagnostic: C3 pair-job makespan under forced splits (copy on the top s SMs)."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
w = bench.make_c3(S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
w.n_sms = 148
w.arrival_ms = 0.25 * pa["solo_ms"] * w.a.reps
seq = bench.median_schedule("seq_cuda", w, sA, sB, kA, kB, S, flush, 3)[0]
out = {"seq_cuda_ms": seq}
print("seq_cuda_ms", round(seq, 3), "gemm solo", round(pa["solo_ms"], 3), flush=True)
for s_b in [int(x) for x in os.environ.get("SLATE_SWEEP_SPLITS", "24,32,40,48,56,64,72,80").split(",")]:
    w.split = s_b
    bench.run_schedule("slate_forced", w, sA, sB, kA, kB, S)
    r = bench.median_schedule("slate_forced", w, sA, sB, kA, kB, S, flush, 3)
    out[s_b] = {"makespan": round(r[0], 3), "G": round(seq / r[0], 4),
                "gemm_launch": [round(q["end_ms"] - q["start_ms"], 3) for q in r[3]],
                "copy_launch": [round(q["end_ms"] - q["start_ms"], 3) for q in r[4]],
                "resize_us": [v for q in r[3] + r[4] for v in q["resize_us"]],
                "topups": sum(q["n_topups"] for q in r[3] + r[4])}
    print(s_b, out[s_b], flush=True)
json.dump(out, open(os.environ.get("SLATE_SWEEP_OUT", "gpurun_out/c3_sweep.json"), "w"), indent=1)
