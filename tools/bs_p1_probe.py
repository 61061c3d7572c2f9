"""Development probe: Black-Scholes with one scenario (Tab II's BS), the
original kernel vs the worker, per launch in 256-launch batches, at several
sizes and task sizes (separates per-launch from per-block costs)."""
import json
import sys

sys.path.insert(0, '.')
sys.path.insert(0, 'tests')
import torch  # noqa: E402
from gpu_helpers import make_bs  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

s = S.Session(None, 0)
out = {}
for lg in (22, 23, 24):
    t = make_bs(1 << lg, 77, n_scen=1)
    for label, mode, iters in (("cuda", S.MODE_STANDALONE, 0), ("slate_it2", S.MODE_SLATE, 2),
                               ("slate_it4", S.MODE_SLATE, 4), ("slate_it8", S.MODE_SLATE, 8)):
        k = s.register_kernel(t.kind, iters=iters)
        kw = {"mode": mode} if mode == S.MODE_STANDALONE else {"placement": S.PLACE_SOLO}
        s.launch_n(k, t.args, t.grid, 32, **kw)
        s.sync(0)
        ids = s.launch_n(k, t.args, t.grid, 128, **kw)
        s.sync(0)
        qs = [s.query(i) for i in ids]
        out["2^%d %s" % (lg, label)] = round((max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)) / 128 * 1e3, 2)
    assert t.check(t.snapshot())[0]
print(json.dumps(out))
