"""Development probe: the C3 STREAM copy (2^30 fp32) worker's T(s) curve."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
n = 1 << 30
a, b = torch.empty(n, device=dev), torch.rand(n, device=dev)
torch.cuda.synchronize()
args, grid = S.copy_args(a, b)
k = s.register_kernel(S.KIND_COPY)
p = s.profile(k, args, grid, S.PROF_CURVE | S.PROF_FORCE)
out = {"curve_ms": {str(x): round(y, 4) for x, y in zip(p["curve_sms"], p["curve_ms"])},
       "curve_tbs": {str(x): round(8.0 * n / (y * 1e-3) / 1e12, 3) for x, y in zip(p["curve_sms"], p["curve_ms"])}}
for sms in (60, 48, 40, 32):
    s.sync(s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=(0, sms - 1)))
    lid = s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=(0, sms - 1))
    s.sync(lid)
    q = s.query(lid)
    out["tbs_%d" % sms] = round(8.0 * n / ((q["end_ms"] - q["start_ms"]) * 1e-3) / 1e12, 3)
print(json.dumps(out))
