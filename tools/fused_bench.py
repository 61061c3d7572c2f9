"""NEXT-1 measurement: the fused co-run worker against the separate-kernel
co-run and the best sequential schedule, and its resize latencies.

    python tools/fused_bench.py        (prints one JSON line)

Pair: Black-Scholes 2^23 options x 32 scenarios (compute) + 2-D stencil
16384^2 (memory), one launch each, both from their own session.  Schedules
(median of 5 after 2 warm-ups, server CUDA-event / device-stamp times):
  seq      each job alone on all SMs, the faster of original kernel and worker;
  corun    two separate worker launches on [0, n-s-1] / [n-s, n-1], the
           survivor grown by the server (top-up launch) when the other drains;
  fused    slate_launch_fused with the same split: one kernel, grow on drain
           in the kernel.
Resize storm on a fused pair: 40 complementary resizes; shrink/grow latencies
from slate_query (device clock mapped to the host's, reading Q30)."""
import json
import random
import statistics
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
sa, sb = S.Session(None, 0), S.Session(None, 0)
n = sa.info()["num_sms"]
PAIR = sys.argv[1] if len(sys.argv) > 1 else "bs+stencil"
if PAIR == "bs+stencil":
    Sx, X, T, r = I.bs_inputs(1 << 23, I.seed_for(2, 1))
    Sx, X, T = (torch.from_numpy(v).to(dev) for v in (Sx, X, T))
    sig = torch.from_numpy(I.bs_sigmas(32)).to(dev)
    cl, pu = torch.zeros(1 << 23, device=dev), torch.zeros(1 << 23, device=dev)
    f = torch.rand(16384, 16384, device=dev)
    o = torch.zeros_like(f)
    A = S.bs_args(Sx, X, T, cl, pu, sig, r)
    B = S.stencil_args(f, o)
    kinds = (S.KIND_BLACKSCHOLES, S.KIND_STENCIL2D)
    desc = "Black-Scholes 2^23 x 32 scenarios (A) + stencil 16384^2 (B), one launch each"
else:   # the C1 kinds at a size that runs ~1 ms: naive SGEMM 1024^3 (A) + triad 2^27 (B)
    Am, Bm, Cm = (torch.rand(1024, 1024, device=dev) for _ in range(3))
    a, b, c = (torch.rand(1 << 27, device=dev) for _ in range(3))
    A = S.sgemm_args(Am, Bm, Cm)
    B = S.triad_args(a, b, c, 3.0)
    kinds = (S.KIND_SGEMM_NAIVE, S.KIND_TRIAD)
    desc = "naive SGEMM 1024^3 (A) + STREAM triad 2^27 (B), one launch each (config C1's kinds)"
torch.cuda.synchronize()
ka, kb = sa.register_kernel(kinds[0]), sb.register_kernel(kinds[1])
pa = sa.profile(ka, *A, S.PROF_CURVE)
pb = sb.profile(kb, *B, S.PROF_CURVE)
ca = dict(zip(pa["curve_sms"], pa["curve_ms"]))
cb = dict(zip(pb["curve_sms"], pb["curve_ms"]))
split, pred = S.choose_split(ca, cb, n, 2)


def span(qs):
    return min(q["start_ms"] for q in qs), max(q["end_ms"] for q in qs)


def run(kind):
    if kind == "seq":
        t = []
        for s_, k, (args, grid) in ((sa, ka, A), (sb, kb, B)):
            best = 1e9
            for mode in (S.MODE_STANDALONE, S.MODE_SLATE):
                lid = s_.launch(k, args, grid, placement=S.PLACE_SOLO, mode=mode)
                s_.sync(lid)
                q = s_.query(lid)
                best = min(best, q["end_ms"] - q["start_ms"])
            t.append(best)
        return sum(t), t
    if kind == "corun":
        la = sa.launch(ka, *A, placement=S.PLACE_CORUN, sm=(0, n - split - 1))
        lb = sb.launch(kb, *B, placement=S.PLACE_CORUN, sm=(n - split, n - 1))
    else:
        la, lb = S.launch_fused(sa, ka, A[0], A[1], sb, kb, B[0], B[1], split)
    sa.sync(la)
    sb.sync(lb)
    qa, qb = sa.query(la), sb.query(lb)
    a0, a1 = span([qa])
    b0, b1 = span([qb])
    return max(a1, b1) - min(a0, b0), [a1 - min(a0, b0), b1 - min(a0, b0), qa["n_topups"] + qb["n_topups"]]


out = {"pair": desc,
       "split_sms_b": split, "predicted_makespan_ms": round(pred, 4)}
for kind in ("seq", "corun", "fused"):
    for _ in range(2):
        run(kind)
    rs = sorted((run(kind) for _ in range(5)), key=lambda x: x[0])
    out[kind] = {"makespan_ms": round(rs[2][0], 4), "detail": [round(v, 4) for v in rs[2][1]],
                 "all_ms": [round(x[0], 4) for x in rs]}
out["gain_corun_vs_seq"] = round(out["seq"]["makespan_ms"] / out["corun"]["makespan_ms"], 4)
out["gain_fused_vs_seq"] = round(out["seq"]["makespan_ms"] / out["fused"]["makespan_ms"], 4)

# resize storm on fused pairs: complementary ranges, 100 us apart
rng = random.Random(7)
lat = {"shrink": [], "grow": []}
issued = 0
while issued < 120:
    la, lb = S.launch_fused(sa, ka, A[0], A[1], sb, kb, B[0], B[1], split)
    time.sleep(50e-6)
    for _ in range(12):
        k = rng.randrange(16, n - 16)
        if sa.resize(la, 0, k - 1) == S.DONE or sb.resize(lb, k, n - 1) == S.DONE:
            break
        issued += 2
        t0 = time.perf_counter()
        while time.perf_counter() - t0 < 100e-6:
            pass
    sa.sync(la)
    sb.sync(lb)
    for q in (sa.query(la), sb.query(lb)):
        for v, kd in zip(q["resize_us"], q["resize_kind"]):
            if kd in lat and v >= 0:
                lat[kd].append(v)


def stats(v):
    return {"n": len(v), "p50": round(statistics.median(v), 2) if v else None,
            "p99": round(float(np.percentile(v, 99)), 2) if v else None, "max": round(max(v), 2) if v else None}


out["fused_resize_us"] = {"shrink": stats(lat["shrink"]), "grow": stats(lat["grow"]), "resizes_issued": issued}
print(json.dumps(out))
sa.close()
sb.close()
