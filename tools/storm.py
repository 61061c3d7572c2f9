"""Diagnostic: the bench's C3 resize storm alone (bench.resize_storm), optionally
with a longer GEMM (K = 4 x 8192) so each launch lives through every resize."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
kmul = int(os.environ.get("STORM_KMUL", "1"))
m = n = 8192
k = 8192 * kmul
g = torch.Generator(device=dev)
g.manual_seed(5)
A = (torch.rand(m, k, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
B = (torch.rand(n, k, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
C = torch.zeros(m, n, device=dev)
torch.cuda.synchronize()
args, grid = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
job = bench.Job("gemm_bf16", S.KIND_GEMM_BF16, args, grid, 1, 0, 0, 2.0 * m * n * k)
r = bench.resize_storm(S, s, job, s.info()["num_sms"], per_launch=int(os.environ.get("STORM_PER", "12")),
                       gap_us=float(os.environ.get("STORM_GAP", "100")))
print(json.dumps(r))
s.close()
