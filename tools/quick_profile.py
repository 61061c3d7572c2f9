"""Development probe: solo profiles (T(s) curves) of every tenant at bench size."""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
g = torch.Generator(device=dev)
g.manual_seed(1)
s = S.Session(None, 0)
print(s.info())
out = {}


def prof(name, kind, args, grid, iters=0):
    k = s.register_kernel(kind, iters=iters)
    t0 = time.time()
    p = s.profile(k, args, grid, S.PROF_CURVE | S.PROF_FORCE)
    # standalone timing
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ks = s.register_kernel(kind)
    s.sync(s.launch(ks, args, grid, mode=S.MODE_STANDALONE))
    ts = []
    for _ in range(3):
        lid = s.launch(ks, args, grid, mode=S.MODE_STANDALONE)
        s.sync(lid)
        q = s.query(lid)
        ts.append(q["end_ms"] - q["start_ms"])
    p["standalone_ms"] = sorted(ts)[1]
    print(name, json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in p.items()}),
          "%.1fs" % (time.time() - t0), flush=True)
    out[name] = p


n = 1 << 26
a, b, c = (torch.rand(n, device=dev, generator=g) for _ in range(3))
prof("triad_2^26", S.KIND_TRIAD, *S.triad_args(a, b, c, 3.0))
del a, b, c
n = 1 << 30
a, b = torch.empty(n, device=dev), torch.rand(n, device=dev, generator=g)
prof("copy_2^30", S.KIND_COPY, *S.copy_args(a, b))
del a, b
rp, col, val, x = I.spmv_inputs(1 << 20, I.seed_for(2, 0))
rp, col, val, x = (torch.from_numpy(v).to(dev) for v in (rp, col, val, x))
y = torch.zeros(1 << 20, device=dev)
prof("spmv_2^20", S.KIND_SPMV_CSR, *S.spmv_args(rp, col, val, x, y))
Sx, X, T, r = I.bs_inputs(1 << 23, I.seed_for(2, 1))
Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
for P in (1, 8, 32):
    sig = torch.from_numpy((np.float32(0.3) + np.float32(0.01) * np.arange(P, dtype=np.float32))).to(dev)
    cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
    prof("bs_2^23_P%d" % P, S.KIND_BLACKSCHOLES, *S.bs_args(Sx, X, T, cl, pu, sig, r))
f = torch.rand(8192, 8192, device=dev, generator=g)
o = torch.zeros_like(f)
prof("stencil_8192", S.KIND_STENCIL2D, *S.stencil_args(f, o))
A, B = torch.rand(1024, 1024, device=dev, generator=g), torch.rand(1024, 1024, device=dev, generator=g)
C = torch.zeros(1024, 1024, device=dev)
prof("sgemm_1024", S.KIND_SGEMM_NAIVE, *S.sgemm_args(A, B, C))
json.dump(out, open("gpurun_out/quick_profile.json", "w"), indent=1)
s.close()
