"""Per-launch cost of the slate worker vs the original kernel, for the Tab II
tenants and the C2 tenants: `n` back-to-back launches (one slate_launch_n job)
standalone and as workers at several task sizes; reports the job span / n and
the mean event-timed launch.  Run with SLATE_LIB=<variant .so> to compare builds.

    python tools/worker_overhead.py [n]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

DEV = "cuda:0"
n_l = int(sys.argv[1]) if len(sys.argv) > 1 else 100
s = S.Session(None, 0)
keep = []


def t(x):
    x = torch.from_numpy(np.ascontiguousarray(x)).to(DEV)
    keep.append(x)
    return x


def z(*shape):
    x = torch.zeros(*shape, device=DEV)
    keep.append(x)
    return x


cases = {}
Sx, X, T, r = I.bs_inputs(1 << 23, 1)
cases["bs_p1"] = (S.KIND_BLACKSCHOLES,) + S.bs_args(t(Sx), t(X), t(T), z(1 << 23), z(1 << 23), t(I.bs_sigmas(1)), float(r))
cases["bs_p32"] = (S.KIND_BLACKSCHOLES,) + S.bs_args(t(Sx), t(X), t(T), z(1 << 23), z(1 << 23), t(I.bs_sigmas(32)), float(r))
cases["tr"] = (S.KIND_TRANSPOSE,) + S.transpose_args(t(I.transpose_inputs(8192, 8192, 2)), z(8192, 8192))
cases["rg"] = (S.KIND_QRNG,) + S.qrng_args(t(I.qrng_table(3, 3).view(np.int32)), z(3, 1 << 24))
a0, b0 = I.gauss_inputs(4096)
ga, gb, gm = t(a0), t(b0), z(4096, 4096)
cases["gs_fan2_t0"] = (S.KIND_GAUSS_FAN2,) + S.gauss_fan2_args(ga, gb, gm, 0)
cases["gs_fan2_t2048"] = (S.KIND_GAUSS_FAN2,) + S.gauss_fan2_args(ga, gb, gm, 2048)
cases["gs_fan1_t0"] = (S.KIND_GAUSS_FAN1,) + S.gauss_fan1_args(ga, gb, gm, 0)
A, B = I.sgemm_inputs(2048, 2048, 2048, 4)
cases["mm"] = (S.KIND_SGEMM_TILED,) + S.sgemm_tiled_args(t(A), t(B), z(2048, 2048))
cases["triad_2^26"] = (S.KIND_TRIAD,) + S.triad_args(z(1 << 26), z(1 << 26), z(1 << 26), 3.0)
torch.cuda.synchronize()


def job(k, args, grid, **kw):
    ids = s.launch_n(k, args, grid, n_l, **kw)
    s.sync(0)
    qs = [s.query(i) for i in ids]
    span = max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)
    ev = float(np.mean([q["end_ms"] - q["start_ms"] for q in qs]))
    ok = [q for q in qs if q["t_first_ns"] and q["t_last_ns"] and q["t_enter_ns"] and q["t_exit_ns"]]
    if not ok:
        return round(span / n_l * 1e3, 2), round(ev * 1e3, 2)
    m = lambda f: round(float(np.mean([f(q) for q in ok])) / 1e3, 2)   # noqa: E731
    # span/launch, event, iters, enter->first task, first->last block, last block->last exit
    return (round(span / n_l * 1e3, 2), round(ev * 1e3, 2), qs[0]["iters"], m(lambda q: q["t_first_ns"] - q["t_enter_ns"]),
            m(lambda q: q["t_last_ns"] - q["t_first_ns"]), m(lambda q: q["t_exit_ns"] - q["t_last_ns"]))


out = {"lib": S.LIB_PATH, "n": n_l}
only = os.environ.get("WO_CASES")
for name, (kind, args, grid) in cases.items():
    if only and name not in only.split(","):
        continue
    rec = {}
    k0 = s.register_kernel(kind)
    job(k0, args, grid, mode=S.MODE_STANDALONE)
    rec["cuda"] = job(k0, args, grid, mode=S.MODE_STANDALONE)[:2]
    for it in (0, 1, 4):
        if it == 1 and os.environ.get("WO_QUICK"):
            continue
        k = s.register_kernel(kind, iters=it)
        job(k, args, grid, placement=S.PLACE_SOLO)
        rec["slate_it%d" % it] = job(k, args, grid, placement=S.PLACE_SOLO)
    out[name] = rec
    print(name, json.dumps(rec), flush=True)
s.close()
print(json.dumps(out))
