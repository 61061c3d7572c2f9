"""ncu target: the C3 tenants (bf16 GEMM 8192^3, copy 2^30) run solo through the worker."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
dev = "cuda:0"
s = S.Session(None, 0)
A = (torch.rand(8192, 8192, device=dev) * 2 - 1).to(torch.bfloat16)
B = (torch.rand(8192, 8192, device=dev) * 2 - 1).to(torch.bfloat16)
C = torch.zeros(8192, 8192, device=dev)
cb, ca = torch.rand(1 << 30, device=dev), torch.empty(1 << 30, device=dev)
torch.cuda.synchronize()
for kind, (args, grid) in [(S.KIND_GEMM_BF16, S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)),
                           (S.KIND_COPY, S.copy_args(ca, cb))]:
    k = s.register_kernel(kind)
    for _ in range(reps):
        s.sync(s.launch(k, args, grid, placement=S.PLACE_SOLO))
s.close()
print("ncu target done")
