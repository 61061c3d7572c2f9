import sys, json
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import torch
from gpu_helpers import make_bs
from paper_conf_ipps_allenf019_b200 import slate as S
s = S.Session(None, 0)
t = make_bs(1 << 23, 77, n_scen=1)
out = {}
for label, mode in (("cuda", S.MODE_STANDALONE), ("slate", S.MODE_SLATE)):
    k = s.register_kernel(t.kind, iters=(0 if mode == S.MODE_STANDALONE else int(sys.argv[1]) if len(sys.argv) > 1 else 4))
    kw = {"mode": mode} if mode == S.MODE_STANDALONE else {"placement": S.PLACE_SOLO}
    s.launch_n(k, t.args, t.grid, 64, **kw); s.sync(0)
    ids = s.launch_n(k, t.args, t.grid, 256, **kw); s.sync(0)
    qs = [s.query(i) for i in ids]
    out[label] = (max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)) / 256 * 1e3
ref = t.snapshot()
print(json.dumps(out), t.check(ref))
