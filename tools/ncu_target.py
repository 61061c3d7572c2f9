"""ncu target: the C2 tenants' slate workers (and standalone kernels) run solo a few
times on all SMs, so ncu can capture them one by one (kernel replay serialises)."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
dev = "cuda:0"
s = S.Session(None, 0)
rp, col, val, x = (torch.from_numpy(v).to(dev) for v in I.spmv_inputs(1 << 20, I.seed_for(2, 0)))
y = torch.zeros(1 << 20, device=dev)
Sx, X, T, r = I.bs_inputs(1 << 23, I.seed_for(2, 1))
Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
sig = torch.from_numpy(I.bs_sigmas(32)).to(dev)
cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
torch.cuda.synchronize()
for kind, (args, grid) in [(S.KIND_SPMV_CSR, S.spmv_args(rp, col, val, x, y)),
                           (S.KIND_BLACKSCHOLES, S.bs_args(Sx, X, T, cl, pu, sig, r))]:
    k = s.register_kernel(kind)
    for _ in range(reps):
        s.sync(s.launch(k, args, grid, placement=S.PLACE_SOLO))
    for _ in range(reps):
        s.sync(s.launch(k, args, grid, mode=S.MODE_STANDALONE))
s.close()
print("ncu target done")
