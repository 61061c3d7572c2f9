"""ncu target (round 2): the C2 SpMV worker on 74 SMs (its co-run share) and on
all SMs, its original kernel, the Black-Scholes P=32 worker, and the C4 stencil
worker and original kernel.  Each launched twice; capture with -c / -k."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
n = s.info()["num_sms"]
rp, col, val, x = (torch.from_numpy(v).to(dev) for v in I.spmv_inputs(1 << 20, I.seed_for(2, 0)))
y = torch.zeros(1 << 20, device=dev)
Sx, X, T, r = I.bs_inputs(1 << 23, I.seed_for(2, 1))
Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
sig = torch.from_numpy(I.bs_sigmas(32)).to(dev)
cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
f = torch.rand(8192, 8192, device=dev)
o = torch.zeros_like(f)
torch.cuda.synchronize()
jobs = [(S.KIND_SPMV_CSR, S.spmv_args(rp, col, val, x, y), [(0, 73), (0, n - 1)]),
        (S.KIND_BLACKSCHOLES, S.bs_args(Sx, X, T, cl, pu, sig, r), [(0, n - 1)]),
        (S.KIND_STENCIL2D, S.stencil_args(f, o), [(0, n - 1)])]
for kind, (args, grid), ranges in jobs:
    k = s.register_kernel(kind)
    for sm in ranges:
        for _ in range(2):
            s.sync(s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=sm))
    for _ in range(2):
        s.sync(s.launch(k, args, grid, mode=S.MODE_STANDALONE))
s.close()
print("ncu target done")
