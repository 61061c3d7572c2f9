"""Development probe: the C2 SpMV (2^20 rows x 16 nnz, banded) -- worker T(s)
curve, the original kernel, and a 640-launch job solo and on a sub-range."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
s = S.Session(None, 0)
n = s.info()["num_sms"]
rp, col, val, x = I.spmv_inputs(1 << 20, I.seed_for(2, 0))
nnz = int(rp[-1])
rp, col, val, x = (torch.from_numpy(v).to(dev) for v in (rp, col, val, x))
y = torch.zeros(1 << 20, device=dev)
torch.cuda.synchronize()
args, grid = S.spmv_args(rp, col, val, x, y)
bytes_ = 8.0 * nnz + 4.0 * (2 * (1 << 20) + 1) + 4.0 * (1 << 20)
out = {}
k = s.register_kernel(S.KIND_SPMV_CSR)
p = s.profile(k, args, grid, S.PROF_CURVE | S.PROF_FORCE)
out["curve_us"] = {str(a): round(b * 1e3, 2) for a, b in zip(p["curve_sms"], p["curve_ms"])}
out["curve_tbs"] = {str(a): round(bytes_ / (b * 1e-3) / 1e12, 3) for a, b in zip(p["curve_sms"], p["curve_ms"])}
out["category"] = p["category_name"]
for sms in (n, 74, 48):
    ids = s.launch_n(k, args, grid, 640, placement=S.PLACE_CORUN, sm=(0, sms - 1))
    s.sync(0)
    ids = s.launch_n(k, args, grid, 640, placement=S.PLACE_CORUN, sm=(0, sms - 1))
    s.sync(0)
    qs = [s.query(i) for i in ids]
    t = max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)
    out["job640_%dsms_us_per_launch" % sms] = round(t / 640 * 1e3, 2)
    out["job640_%dsms_tbs" % sms] = round(bytes_ * 640 / (t * 1e-3) / 1e12, 3)
ks = s.register_kernel(S.KIND_SPMV_CSR)
ids = s.launch_n(ks, args, grid, 64, mode=S.MODE_STANDALONE)
s.sync(0)
qs = [s.query(i) for i in ids]
out["standalone_us_per_launch"] = round((max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)) / 64 * 1e3, 2)
print(json.dumps(out))
