"""Development probe: the C4 stencil (8192^2 fp32 sweep) -- worker T(s) curve and the original kernel."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
f = torch.rand(8192, 8192, device=dev)
o = torch.zeros_like(f)
torch.cuda.synchronize()
args, grid = S.stencil_args(f, o)
k = s.register_kernel(S.KIND_STENCIL2D)
p = s.profile(k, args, grid, S.PROF_CURVE | S.PROF_FORCE)
by = 8.0 * 8192 * 8192
out = {"curve_us": {str(a): round(b * 1e3, 1) for a, b in zip(p["curve_sms"], p["curve_ms"])},
       "curve_tbs": {str(a): round(by / (b * 1e-3) / 1e12, 3) for a, b in zip(p["curve_sms"], p["curve_ms"])}}
ks = s.register_kernel(S.KIND_STENCIL2D)
ids = s.launch_n(ks, args, grid, 16, mode=S.MODE_STANDALONE)
s.sync(0)
qs = [s.query(i) for i in ids]
t = (max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)) / 16
out["standalone_us"] = round(t * 1e3, 1)
out["standalone_tbs"] = round(by / (t * 1e-3) / 1e12, 3)
print(json.dumps(out))
