"""Diagnostic: the bench's resize storm (bench.resize_storm) on a C2 tenant:
Black-Scholes 2^23 x 32 scenarios (one launch ~0.42 ms) or the SpMV worker on
a 2^22-row matrix with task size 1 (one launch ~1.6 ms).

    python tools/storm_tenant.py bs|spmv
"""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "bs"
dev = "cuda:0"
s = S.Session(None, 0)
if which == "bs":
    Sx, X, T, r = I.bs_inputs(1 << 23, 5)
    Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
    sig = torch.from_numpy(I.bs_sigmas(32)).to(dev)
    cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
    args, grid = S.bs_args(Sx, X, T, cl, pu, sig, r)
    job = bench.Job("blackscholes", S.KIND_BLACKSCHOLES, args, grid, 1, 0, 0, 0)
    per, gap = int(os.environ.get("STORM_PER", "4")), float(os.environ.get("STORM_GAP", "80"))
else:
    rp, col, val, x = (torch.from_numpy(v).to(dev) for v in I.spmv_inputs(1 << 22, 6))
    y = torch.zeros(1 << 22, device=dev)
    args, grid = S.spmv_args(rp, col, val, x, y)
    job = bench.Job("spmv", S.KIND_SPMV_CSR, args, grid, 1, 0, 0, 0)
    per, gap = int(os.environ.get("STORM_PER", "8")), float(os.environ.get("STORM_GAP", "100"))
torch.cuda.synchronize()
r = bench.resize_storm(S, s, job, s.info()["num_sms"], n_resizes=int(os.environ.get("STORM_N", "60")),
                       per_launch=per, gap_us=gap)
print(which, json.dumps(r))
s.close()
