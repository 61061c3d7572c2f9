"""Development check of the tcgen05 GEMM tenant: correctness at small sizes, then speed."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
from gpu_helpers import make_gemm  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

s = S.Session(None, 0)
for (m, n, k, mode) in [(256, 256, 64, "int"), (256, 512, 512, "int"), (512, 256, 1024, "float"), (768, 512, 2048, "float")]:
    t = make_gemm(m, n, k, 7, mode)
    ks = s.register_kernel(S.KIND_GEMM_BF16)
    s.sync(s.launch(ks, t.args, t.grid, mode=S.MODE_STANDALONE), timeout_us=10_000_000)
    ref = t.snapshot()
    ok, err = t.check(ref)
    print("standalone", m, n, k, mode, ok, err, flush=True)
    t.zero_outputs()
    kw = s.register_kernel(S.KIND_GEMM_BF16, flags=S.KFLAG_COVERAGE)
    cov = torch.zeros(int(np.prod(t.grid)), dtype=torch.int32, device="cuda:0")
    torch.cuda.synchronize()
    lid = s.launch(kw, t.args, t.grid, placement=S.PLACE_CORUN, sm=(0, 147), coverage=cov)
    s.sync(lid, timeout_us=10_000_000)
    out = t.snapshot()
    print("slate", ok, t.check(out), "bitexact", all(torch.equal(a, b) for a, b in zip(out, ref)),
          "cov", s.query(lid)["coverage_ok"], flush=True)
# speed at 8192^3
m = n = k = 8192
A = torch.randn(m, k, device="cuda:0").to(torch.bfloat16)
B = torch.randn(n, k, device="cuda:0").to(torch.bfloat16)
C = torch.zeros(m, n, device="cuda:0")
torch.cuda.synchronize()
args, grid = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
kw = s.register_kernel(S.KIND_GEMM_BF16)
p = s.profile(kw, args, grid, S.PROF_CURVE)
print("gemm 8192^3 slate solo ms %.3f TFLOP/s %.1f curve %s" % (p["solo_ms"], p["tc_tflops"], list(zip(p["curve_sms"], [round(x, 3) for x in p["curve_ms"]]))))
ks = s.register_kernel(S.KIND_GEMM_BF16)
ts = []
for _ in range(5):
    lid = s.launch(ks, args, grid, mode=S.MODE_STANDALONE)
    s.sync(lid)
    q = s.query(lid)
    ts.append(q["end_ms"] - q["start_ms"])
print("standalone ms", sorted(ts)[2], "TFLOP/s", 2 * m * n * k / sorted(ts)[2] / 1e9)
ref = (A.float() @ B.float().T)
print("max abs err vs torch fp32", float((C - ref).abs().max()), "scale", float(ref.abs().max()))
s.close()
