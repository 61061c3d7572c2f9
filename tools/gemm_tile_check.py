"""Compare GEMM tile widths: correctness (integer inputs, exact) and 8192^3 speed.
   SLATE_LIB=.../libslate_bn256.so SLATE_TILE_N=256 python tools/gemm_tile_check.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from oracle import tenants as OT  # noqa: E402
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

TN = int(os.environ.get("SLATE_TILE_N", "0"))
s = S.Session(None, 0)
TN = TN or S.GEMM_TILE_N
for m, n, k in [(256, 512, 512), (1024, 768, 2048)]:
    A, B = I.gemm_inputs(m, n, k, 9, "int")
    Ad = torch.from_numpy(A.view(np.int16)).cuda()
    Bd = torch.from_numpy(B.view(np.int16)).cuda()
    C = torch.zeros(m, n, device="cuda")
    torch.cuda.synchronize()
    args, _ = S.gemm_args(Ad, Bd, C)
    grid = (n // TN, m // 128, 1)
    kw = s.register_kernel(S.KIND_GEMM_BF16, flags=S.KFLAG_COVERAGE)
    cov = torch.zeros(grid[0] * grid[1], dtype=torch.int32, device="cuda")
    torch.cuda.synchronize()
    lid = s.launch(kw, args, grid, placement=S.PLACE_CORUN, sm=(0, 147), coverage=cov)
    s.sync(lid)
    ok = np.array_equal(C.cpu().numpy().astype(np.float64), OT.gemm_bf16(A, B))
    print("tile_n", TN, (m, n, k), "exact", ok, "cov", s.query(lid)["coverage_ok"], flush=True)
m = n = k = 8192
A = (torch.rand(m, k, device="cuda") * 2 - 1).to(torch.bfloat16)
B = (torch.rand(n, k, device="cuda") * 2 - 1).to(torch.bfloat16)
C = torch.zeros(m, n, device="cuda")
torch.cuda.synchronize()
args, _ = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
grid = (n // TN, m // 128, 1)
kw = s.register_kernel(S.KIND_GEMM_BF16)
p = s.profile(kw, args, grid, S.PROF_CURVE)
print("tile_n %d: 8192^3 %.3f ms = %.1f TFLOP/s; curve %s" % (TN, p["solo_ms"], p["tc_tflops"],
      [(a, round(b, 3)) for a, b in zip(p["curve_sms"], p["curve_ms"])]))
ref = A.float() @ B.float().T
print("max abs err", float((C - ref).abs().max()))
s.close()
