"""ncu target: the C2 SpMV worker on 74 SMs (the co-run share) and on all SMs,
and the original kernel; each launched twice (ncu captures the second)."""
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
torch.cuda.synchronize()
args, grid = S.spmv_args(rp, col, val, x, y)
k = s.register_kernel(S.KIND_SPMV_CSR)
for sm in ((0, 73), (0, n - 1)):
    for _ in range(2):
        s.sync(s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=sm))
for _ in range(2):
    s.sync(s.launch(k, args, grid, mode=S.MODE_STANDALONE))
s.close()
print("ncu target done")
