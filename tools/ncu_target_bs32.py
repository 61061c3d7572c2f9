"""ncu target: Black-Scholes P = 32 on 2^23 options (C2's H_C tenant) as the
original kernel and as a slate worker, solo on all SMs."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
Sx, X, T, r = I.bs_inputs(1 << 23, 2)
Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
sig = torch.from_numpy(I.bs_sigmas(32)).to(dev)
cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
torch.cuda.synchronize()
args, grid = S.bs_args(Sx, X, T, cl, pu, sig, r)
k = s.register_kernel(S.KIND_BLACKSCHOLES)
s.sync(s.launch(k, args, grid, mode=S.MODE_STANDALONE))
s.sync(s.launch(k, args, grid, placement=S.PLACE_SOLO))
s.close()
print("ncu target done")
