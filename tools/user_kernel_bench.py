"""NEXT-3 cost (the paper's Fig. 6 counts injection + compilation):
NVRTC transformation + compile + load time of a user kernel, and its per-launch
time as a slate worker against its original kernel (100 launches, one batch).

    python tools/user_kernel_bench.py
"""
import ctypes
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

SRC = r"""
__global__ void axpb2d(const float* __restrict__ x, float* y, float a, float b, int w, int h) {
  int col = blockIdx.x * blockDim.x + threadIdx.x;
  int row = blockIdx.y;
  if (col < w && row < h) y[row * w + col] = fmaf(a, x[row * w + col], b);
}
"""


class Args(ctypes.Structure):
    _fields_ = [("x", ctypes.c_uint64), ("y", ctypes.c_uint64), ("a", ctypes.c_float), ("b", ctypes.c_float),
                ("w", ctypes.c_int32), ("h", ctypes.c_int32)]


w, h, T = 8192, 8192, 256
x = torch.rand(h, w, device="cuda:0")
y = torch.zeros(h, w, device="cuda:0")
args = Args(x.data_ptr(), y.data_ptr(), 2.0, 1.0, w, h)
grid = (w // T, h, 1)
out = {}
with S.Session(None, 0) as s:
    t0 = time.perf_counter()
    k = s.register_source(SRC, "axpb2d", Args, threads=T, bytes_per_block=8.0 * T)
    out["register_source_ms"] = round((time.perf_counter() - t0) * 1e3, 1)
    torch.cuda.synchronize()
    for label, kw in (("original", {"mode": S.MODE_STANDALONE}), ("slate", {"placement": S.PLACE_SOLO})):
        for rep in range(2):
            ids = s.launch_n(k, args, grid, 100, **kw)
            s.sync(0)
        qs = [s.query(i) for i in ids]
        span = max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)
        out[label + "_us_per_launch"] = round(span / 100 * 1e3, 2)
        out[label + "_GBps"] = round(8.0 * w * h / (span / 100 * 1e-3) / 1e9, 1)
    p = s.profile(k, args, grid, S.PROF_CURVE)
    out["profile"] = {"class": p["category_name"], "hbm_gbps": round(p["hbm_gbps"], 1)}
print(json.dumps(out))
