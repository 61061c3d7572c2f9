"""ncu target: the Tab II short-block tenants (TR transpose 8192^2, Black-Scholes
P = 1 on 2^23 options) as slate workers and as original kernels, solo on all
SMs, a few times each (kernel replay serialises)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 1
dev = "cuda:0"
s = S.Session(None, 0)
a = torch.from_numpy(I.transpose_inputs(8192, 8192, 1)).to(dev)
o = torch.zeros(8192, 8192, device=dev)
Sx, X, T, r = I.bs_inputs(1 << 23, 2)
Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
sig = torch.from_numpy(I.bs_sigmas(1)).to(dev)
cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
torch.cuda.synchronize()
for kind, (args, grid) in [(S.KIND_TRANSPOSE, S.transpose_args(a, o)),
                           (S.KIND_BLACKSCHOLES, S.bs_args(Sx, X, T, cl, pu, sig, r))]:
    k = s.register_kernel(kind)
    for _ in range(reps):
        s.sync(s.launch(k, args, grid, placement=S.PLACE_SOLO))
    for _ in range(reps):
        s.sync(s.launch(k, args, grid, mode=S.MODE_STANDALONE))
s.close()
print("ncu target done")
