"""NEXT-2: the paper's own workload on B200.

The five Tab II applications as Slate tenants -- BS (Black-Scholes,
one scenario: the SDK kernel), GS (Rodinia Gaussian elimination: a Fan1 and a
Fan2 launch per step), MM (SDK matrixMul), RG (SDK quasirandomGenerator), TR
(SDK transpose) -- each a job of back-to-back launches, sized to a
few tens of ms solo on B200.  Measured here:

  * Tab II on B200: each app's solo profile (HBM GB/s, FP32 GFLOP/s) and its
    class under reading Q9 (the paper's Titan Xp labels beside it);
  * §V-B solo study: original kernels vs Slate workers on all SMs;
  * Fig 5 task-size sweep: Slate solo at iters 1, 2, 4, 10, 20 and auto;
  * Fig 7: all 15 pairings under sequential CUDA, plain
    concurrent streams (the hardware leftover policy, in place of MPS),
    Slate with Tab I alone (TABLE) and Slate HYBRID (Q31), with G = T_seq /
    makespan, STP and ANTT, and whether the two jobs actually overlapped.

    python tools/paper_pairs.py [--out gpurun_out/paper_pairs.json] [--reps 3]
"""
import argparse
import itertools
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ipps_allenf019_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

DEV = "cuda:0"
# Tab II as printed: compute / memory intensity on a Titan Xp
PAPER_TAB2 = {"BS": ("Med", "Med"), "GS": ("Low", "Med"), "MM": ("High", "Med"), "RG": ("Low", "Low"),
              "TR": ("Low", "High")}
# Slate co-runs RG with every other app; all other pairings run solo
PAPER_CORUN = {("BS", "RG"), ("GS", "RG"), ("MM", "RG"), ("RG", "RG"), ("RG", "TR")}

SIZES = {"BS": 1 << 23, "TR": 8192, "MM": 2048, "RG": 1 << 24, "GS": 4096}


class App:
    """One instance of an application: device buffers and its job's launches."""

    def __init__(self, name, inst):
        self.name, self.inst = name, inst
        seed = I.seed_for(6, 10 * inst + "BS GS MM RG TR".split().index(name))
        self.restore_pairs = []
        if name == "BS":
            n = SIZES["BS"]
            Sx, X, T, r = I.bs_inputs(n, seed)
            self.buf = [torch.from_numpy(v).to(DEV) for v in (Sx, X, T, I.bs_sigmas(1))]
            call, put = torch.zeros(n, device=DEV), torch.zeros(n, device=DEV)
            self.buf += [call, put]
            args, grid = S.bs_args(self.buf[0], self.buf[1], self.buf[2], call, put, self.buf[3], float(r))
            self.kinds, self.reps = [S.KIND_BLACKSCHOLES], int(os.environ.get("PP_BS_REPS", 800))
            self.launches = [(0, args, grid)]
        elif name == "TR":
            h = w = SIZES["TR"]
            a = torch.from_numpy(I.transpose_inputs(h, w, seed)).to(DEV)
            o = torch.zeros(w, h, device=DEV)
            self.buf = [a, o]
            args, grid = S.transpose_args(a, o)
            self.kinds, self.reps = [S.KIND_TRANSPOSE], int(os.environ.get("PP_TR_REPS", 300))
            self.launches = [(0, args, grid)]
        elif name == "MM":
            m = SIZES["MM"]
            A, B = I.sgemm_inputs(m, m, m, seed)
            A, B, C = torch.from_numpy(A).to(DEV), torch.from_numpy(B).to(DEV), torch.zeros(m, m, device=DEV)
            self.buf = [A, B, C]
            args, grid = S.sgemm_tiled_args(A, B, C)
            self.kinds, self.reps = [S.KIND_SGEMM_TILED], int(os.environ.get("PP_MM_REPS", 30))
            self.launches = [(0, args, grid)]
        elif name == "RG":
            n, dims = SIZES["RG"], 3
            t = torch.from_numpy(I.qrng_table(dims, seed).view(np.int32)).to(DEV)
            o = torch.zeros(dims, n, device=DEV)
            self.buf = [t, o]
            args, grid = S.qrng_args(t, o, 0)
            self.kinds, self.reps = [S.KIND_QRNG], int(os.environ.get("PP_RG_REPS", 700))
            self.launches = [(0, args, grid)]
        elif name == "GS":
            n = SIZES["GS"]
            a0, b0 = I.gauss_inputs(n)
            a, b = torch.from_numpy(a0).to(DEV), torch.from_numpy(b0).to(DEV)
            m = torch.zeros(n, n, device=DEV)
            self.buf = [a, b, m]
            self.restore_pairs = [(a, a.clone()), (b, b.clone())]
            self.kinds, self.reps = [S.KIND_GAUSS_FAN1, S.KIND_GAUSS_FAN2], 1
            self.launches = []
            for t in range(n - 1):
                self.launches.append((0,) + S.gauss_fan1_args(a, b, m, t))
                self.launches.append((1,) + S.gauss_fan2_args(a, b, m, t))
        torch.cuda.synchronize()

    def restore(self):
        for dst, src in self.restore_pairs:
            dst.copy_(src)

    def register(self, sess, iters=0):
        return [sess.register_kernel(k, iters=iters) for k in self.kinds]

    def submit(self, sess, ks, **kw):
        if len(self.launches) == 1:
            ki, args, grid = self.launches[0]
            return sess.launch_n(ks[ki], args, grid, self.reps, **kw)
        # GS: the elimination's 2(n-1) launches in one call (one batch)
        return sess.launch_many([(ks[ki], args, grid) for ki, args, grid in self.launches], **kw)

    def profile(self, sess, ks):
        # the representative (largest) launch: the job's first Fan2 for GS
        ki, args, grid = self.launches[-1] if len(self.launches) == 1 else self.launches[1]
        p = sess.profile(ks[ki], args, grid, S.PROF_CURVE)
        self.restore()
        return p


def collect(sess, ids):
    sess.sync(0)
    qs = [sess.query(i) for i in ids]
    bad = [q for q in qs if q["state"] != 2 or q["end_ms"] <= 0]
    if bad:
        raise RuntimeError("%d launches did not complete: %r" % (len(bad), bad[0]))
    return min(q["start_ms"] for q in qs), max(q["end_ms"] for q in qs)


def flush(buf):
    buf.fill_(1.0)
    torch.cuda.synchronize()


def run(schedule, A, B, sA, sB, kA, kB):
    """One pair-job; returns (makespan, end_A, end_B, overlap_ms), times from the first start."""
    A.restore()
    B.restore()
    torch.cuda.synchronize()
    if schedule == "seq_cuda":
        ia = A.submit(sA, kA, mode=S.MODE_STANDALONE)
        ib = B.submit(sA, kB, mode=S.MODE_STANDALONE)
        (a0, a1), (b0, b1) = collect(sA, ia), collect(sA, ib)
    elif schedule == "streams":
        ia = A.submit(sA, kA, mode=S.MODE_STANDALONE)
        ib = B.submit(sB, kB, mode=S.MODE_STANDALONE)
        (a0, a1), (b0, b1) = collect(sA, ia), collect(sB, ib)
    elif schedule == "seq_slate":
        ia = A.submit(sA, kA, placement=S.PLACE_SOLO)
        ib = B.submit(sA, kB, placement=S.PLACE_SOLO)
        (a0, a1), (b0, b1) = collect(sA, ia), collect(sA, ib)
    elif schedule in ("slate", "slate_table"):
        if schedule == "slate_table":
            sA.set_policy(S.POLICY_TABLE)
        try:
            ia = A.submit(sA, kA, placement=S.PLACE_AUTO)
            ib = B.submit(sB, kB, placement=S.PLACE_AUTO)
            (a0, a1), (b0, b1) = collect(sA, ia), collect(sB, ib)
        finally:
            sA.set_policy(S.POLICY_HYBRID)
    else:
        raise ValueError(schedule)
    t0 = min(a0, b0)
    overlap = max(0.0, min(a1, b1) - max(a0, b0))
    return max(a1, b1) - t0, a1 - t0, b1 - t0, overlap


def median_run(schedule, A, B, sA, sB, kA, kB, fl, reps):
    run(schedule, A, B, sA, sB, kA, kB)                       # warm-up
    rs = []
    for _ in range(reps):
        flush(fl)
        rs.append(run(schedule, A, B, sA, sB, kA, kB))
    rs.sort(key=lambda r: r[0])
    return rs[len(rs) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "paper_pairs.json"))
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--apps", default="BS,GS,MM,RG,TR")
    args = ap.parse_args()
    names = args.apps.split(",")
    fl = torch.empty(64 << 20, device=DEV)                    # 256 MB > L2
    sA, sB = S.Session(None, 0), S.Session(None, 0)
    n_sms = sA.info()["num_sms"]
    out = {"n_sms": n_sms, "sizes": SIZES, "apps": {}, "pairs": {}}
    apps = {n: [App(n, 0), App(n, 1)] for n in names}
    kern = {n: (apps[n][0].register(sA), apps[n][1].register(sB)) for n in names}

    # ---- Tab II on B200, §V-B solo study, Fig 5 task-size sweep
    for n in names:
        A = apps[n][0]
        p = A.profile(sA, kern[n][0])
        rec = {"paper_tab2": PAPER_TAB2[n], "category": p["category_name"], "hbm_gbps": round(p["hbm_gbps"], 1),
               "fp32_gflops": round(p["fp32_gflops"], 1), "hbm_frac": round(p["hbm_frac"], 4),
               "fp32_frac": round(p["fp32_frac"], 4), "launch_solo_ms": round(p["solo_ms"], 4),
               "curve": {str(s): round(t, 4) for s, t in zip(p["curve_sms"], p["curve_ms"])},
               "launches_per_job": len(A.launches) * A.reps}
        solo = {}
        # Fig 5's task sizes: 1, 2, 4, 10, 20 blocks per task, and the automatic size (Q38)
        for label, iters, mode in (("cuda", 0, S.MODE_STANDALONE), ("slate_auto", 0, S.MODE_SLATE),
                                   ("slate_iters1", 1, S.MODE_SLATE), ("slate_iters2", 2, S.MODE_SLATE),
                                   ("slate_iters4", 4, S.MODE_SLATE), ("slate_iters10", 10, S.MODE_SLATE),
                                   ("slate_iters20", 20, S.MODE_SLATE)):
            ks = A.register(sA, iters) if iters else kern[n][0]
            ts = []
            for _ in range(args.reps + 1):
                A.restore()
                flush(fl)
                kw = {"mode": mode} if mode == S.MODE_STANDALONE else {"placement": S.PLACE_SOLO}
                a0, a1 = collect(sA, A.submit(sA, ks, **kw))
                ts.append(a1 - a0)
            solo[label] = round(statistics.median(ts[1:]), 3)
        rec["job_ms"] = solo
        rec["slate_vs_cuda"] = round(solo["cuda"] / solo["slate_auto"], 4)
        rec["best_slate_vs_cuda"] = round(solo["cuda"] / min(v for k, v in solo.items() if k != "cuda"), 4)
        out["apps"][n] = rec
        print(n, json.dumps(rec), flush=True)

    # ---- Fig 7: the 15 pairings
    for a, b in itertools.combinations_with_replacement(names, 2):
        A, B = apps[a][0], apps[b][1]
        kA, kB = kern[a][0], kern[b][1]
        res = {}
        for sch in ("seq_cuda", "streams", "seq_slate", "slate_table", "slate"):
            t0 = time.time()
            mk, ea, eb, ov = median_run(sch, A, B, sA, sB, kA, kB, fl, args.reps)
            res[sch] = {"makespan_ms": round(mk, 3), "end_a_ms": round(ea, 3), "end_b_ms": round(eb, 3),
                        "overlap_ms": round(ov, 3), "wall_s": round(time.time() - t0, 1)}
        seq = res["seq_cuda"]
        solo_a, solo_b = seq["end_a_ms"], seq["makespan_ms"] - seq["end_a_ms"]
        for sch, r in res.items():
            r["G"] = round(seq["makespan_ms"] / r["makespan_ms"], 4)
            ta, tb = r["end_a_ms"], r["end_b_ms"]
            r["stp"] = round(solo_a / ta + solo_b / tb, 4)
            r["antt"] = round((ta / solo_a + tb / solo_b) / 2, 4)
        key = "%s-%s" % (a, b)
        res["paper_corun"] = (a, b) in PAPER_CORUN or (b, a) in PAPER_CORUN
        res["slate_corun"] = res["slate"]["overlap_ms"] > 0.1 * min(solo_a, solo_b)
        res["slate_vs_streams"] = round(res["streams"]["makespan_ms"] / res["slate"]["makespan_ms"], 4)
        out["pairs"][key] = res
        print(key, json.dumps(res), flush=True)
    sA.close()
    sB.close()
    g = [r["slate"]["G"] for r in out["pairs"].values()]
    vs = [r["slate_vs_streams"] for r in out["pairs"].values()]
    out["summary"] = {"mean_G_slate_vs_cuda": round(float(np.mean(g)), 4), "max_G": round(max(g), 4),
                      "mean_slate_vs_streams": round(float(np.mean(vs)), 4), "max_slate_vs_streams": round(max(vs), 4),
                      "corun_pairs": sorted(k for k, r in out["pairs"].items() if r["slate_corun"])}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)
    print("summary", json.dumps(out["summary"]), flush=True)


if __name__ == "__main__":
    main()
