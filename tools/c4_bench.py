"""C4 (BASELINE configs[3]): a 4-tenant mix -- triad, SpMV, 2-D stencil, bf16 GEMM --
from four separate client processes through one `slated` server (shared-memory
command slots, buffers by CUDA IPC), AUTO placement: the selector pairs the
GEMM (H_C) with a memory tenant at a time and runs memory tenants solo with
each other (Tab I).  Compared with the same four jobs run back to back with
the original kernels by one client.  Device times come from the server's
CUDA events (slate_query start/end, one clock for every client).

    python tools/c4_bench.py [--steps K]     (prints one JSON line)
"""
import argparse
import json

import numpy as np
import os
import signal
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

JOBS = {   # kind -> launches per job (each job ~ 8-18 ms solo)
    "triad": 64, "spmv": 256, "stencil": 64, "gemm": 96,
}


def build(kind, S, dev):
    import torch
    from paper_conf_ipps_allenf019_b200 import inputs as I
    g = torch.Generator(device=dev)
    g.manual_seed(20190520 + 400 + len(kind))
    if kind == "triad":
        n = 1 << 26
        a, b, c = torch.zeros(n, device=dev), torch.rand(n, device=dev, generator=g), torch.rand(n, device=dev, generator=g)
        keep = (a, b, c)
        args, grid = S.triad_args(a, b, c, 3.0)
        k = S.KIND_TRIAD
    elif kind == "spmv":
        rp, col, val, x = (torch.from_numpy(v).to(dev) for v in I.spmv_inputs(1 << 20, I.seed_for(4, 1)))
        y = torch.zeros(1 << 20, device=dev)
        keep = (rp, col, val, x, y)
        args, grid = S.spmv_args(rp, col, val, x, y)
        k = S.KIND_SPMV_CSR
    elif kind == "stencil":
        f = torch.rand(8192, 8192, device=dev, generator=g)
        o = torch.zeros_like(f)
        keep = (f, o)
        args, grid = S.stencil_args(f, o)
        k = S.KIND_STENCIL2D
    else:
        A = (torch.rand(4096, 4096, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
        B = (torch.rand(4096, 4096, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
        C = torch.zeros(4096, 4096, device=dev)
        keep = (A, B, C)
        args, grid = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
        k = S.KIND_GEMM_BF16
    torch.cuda.synchronize()
    return k, args, grid, keep


def client(endpoint, kind, steps, go_path, device=0):
    """One tenant process: profile, then `steps` jobs, each released by the parent."""
    from paper_conf_ipps_allenf019_b200 import slate as S
    import torch
    torch.cuda.set_device(device)
    s = S.Session(endpoint)
    k, args, grid, keep = build(kind, S, "cuda:%d" % device)
    for t in keep:
        s.share_buffer(t)
    kid = s.register_kernel(k)
    s.profile(kid, args, grid, S.PROF_CURVE)
    print("READY", flush=True)
    out = []
    for step in range(steps):
        while not os.path.exists("%s.%d" % (go_path, step)):
            time.sleep(0.0005)
        t_go = time.time()
        # the job in one call (slate_launch_n: the selector sees the whole job, its
        # launches go out as one batch; C4_PER_LAUNCH=1: one call per launch)
        if os.environ.get("C4_PER_LAUNCH"):
            ids = [s.launch(kid, args, grid, placement=S.PLACE_AUTO) for _ in range(JOBS[kind])]
        else:
            ids = s.launch_n(kid, args, grid, JOBS[kind], placement=S.PLACE_AUTO)
        t_sub = time.time()
        s.sync(0)
        qs = [s.query(i) for i in ids]
        slow = sorted(qs, key=lambda q: q["start_ms"] - q["end_ms"])[:3]   # the longest launches (diagnostics)
        out.append([min(q["start_ms"] for q in qs), max(q["end_ms"] for q in qs),
                    sum(len(q["resize_us"]) for q in qs), [v for q in qs for v in q["resize_us"]],
                    [{"ms": round(q["end_ms"] - q["start_ms"], 3), "start": round(q["start_ms"], 3),
                      "workers": q["workers_started"], "topups": q["n_topups"], "resizes": q["n_resizes"],
                      "iters": q["iters"], "sm": [q["sm_lo"], q["sm_hi"]]} for q in slow], [t_go, t_sub]])
        open("%s.%d.%s" % (go_path, step, kind), "w").close()   # this client is ready for the next step
    print("RESULT " + json.dumps(out), flush=True)
    s.close()


def sequential(endpoint, device=0, slate=False):
    """The four jobs back to back, one client: the original kernels (vanilla
    CUDA), or with slate=True the workers on every SM (Slate-sequential)."""
    from paper_conf_ipps_allenf019_b200 import slate as S
    import torch
    torch.cuda.set_device(device)
    s = S.Session(endpoint)
    built = {k: build(k, S, "cuda:%d" % device) for k in JOBS}
    for k, (_, _, _, keep) in built.items():
        for t in keep:
            s.share_buffer(t)
    kids = {k: s.register_kernel(v[0]) for k, v in built.items()}
    times = []
    for rep in range(4):
        ids = []
        per = {}
        for k, (_, args, grid, _) in built.items():
            if slate:
                first = s.launch_n(kids[k], args, grid, JOBS[k], placement=S.PLACE_SOLO)
                li = list(first) if isinstance(first, (list, tuple)) else list(range(first, first + JOBS[k]))
            else:
                li = [s.launch(kids[k], args, grid, mode=S.MODE_STANDALONE) for _ in range(JOBS[k])]
            ids += li
            per[k] = li
        s.sync(0)
        qs = {i: s.query(i) for i in ids}
        t0 = min(q["start_ms"] for q in qs.values())
        t1 = max(q["end_ms"] for q in qs.values())
        solo = {k: max(qs[i]["end_ms"] for i in li) - min(qs[i]["start_ms"] for i in li) for k, li in per.items()}
        if rep:
            times.append((t1 - t0, solo))
    s.close()
    times.sort(key=lambda x: x[0])
    return times[len(times) // 2]


def run(steps, device=0):
    """Run the C4 measurement (daemon + 4 client processes) on GPU `device`; returns the result dict."""
    from paper_conf_ipps_allenf019_b200 import slate as S
    cmd = [sys.executable, __file__, "--steps", str(steps), "--device", str(device)]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    if not lines:
        raise RuntimeError("c4 failed: " + out.stderr[-500:])
    return json.loads(lines[-1])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--client", nargs=3)
    ap.add_argument("--device", type=int, default=0)
    a = ap.parse_args()
    if a.client:
        client(a.client[0], a.client[1], a.steps, a.client[2], a.device)
        return
    from paper_conf_ipps_allenf019_b200 import slate as S
    ep = "/slate-c4-%d" % os.getpid()
    go = "/tmp/slate_c4_go_%d" % os.getpid()
    log = os.environ.get("C4_DAEMON_LOG")           # diagnostics: the daemon's stderr (SLATE_DEBUG output)
    d = subprocess.Popen([S.DAEMON, "--device", str(a.device), "--endpoint", ep],
                         stderr=open(log, "w") if log else subprocess.DEVNULL)
    for _ in range(300):
        try:
            S.Session(ep).close()
            break
        except S.SlateError:
            time.sleep(0.2)
    seq_ms, solo_cuda = sequential(ep, a.device)
    seq_slate_ms, solo_slate = sequential(ep, a.device, slate=True)
    # every job's best solo time (original kernels or workers), the baseline of the gains
    solo = {k: min(solo_cuda[k], solo_slate[k]) for k in JOBS}
    best_seq = sum(solo.values())
    ps = {k: subprocess.Popen([sys.executable, __file__, "--steps", str(a.steps), "--device", str(a.device),
                               "--client", ep, k, go],
                              stdout=subprocess.PIPE, text=True) for k in JOBS}
    for p in ps.values():
        assert "READY" in p.stdout.readline()
    # a step is released once every client finished reading the previous one
    # (the SpMV client's 256 per-launch queries once overran a fixed 0.3-s gap,
    # so its next job started up to 0.5 s late and the step's span measured that)
    for step in range(a.steps):
        if step:
            while not all(os.path.exists("%s.%d.%s" % (go, step - 1, k)) for k in JOBS):
                time.sleep(0.001)
            time.sleep(0.05)
        open("%s.%d" % (go, step), "w").close()
    res = {}
    for k, p in ps.items():
        out, _ = p.communicate(timeout=600)
        res[k] = json.loads([l for l in out.splitlines() if l.startswith("RESULT ")][0][7:])
    d.send_signal(signal.SIGTERM)
    d.wait(timeout=30)
    for step in range(a.steps):
        os.unlink("%s.%d" % (go, step))
        for k in JOBS:
            os.unlink("%s.%d.%s" % (go, step, k))
    spans, stps, resize = [], [], []
    for step in range(a.steps):
        t0 = min(res[k][step][0] for k in JOBS)
        t1 = max(res[k][step][1] for k in JOBS)
        spans.append(t1 - t0)
        # turnaround of each job from the step's release (all four arrive together)
        stps.append(sum(solo[k] / (res[k][step][1] - t0) for k in JOBS))
        resize += [v for k in JOBS for v in res[k][step][3]]
    if os.environ.get("C4_TIMELINE"):   # diagnostics: each job's [start, end] from the step's first start (ms)
        for step in range(a.steps):
            t0 = min(res[k][step][0] for k in JOBS)
            sys.stderr.write("C4 step %d: %s\n" % (step, "  ".join(
                "%s %.2f-%.2f" % (k, res[k][step][0] - t0, res[k][step][1] - t0) for k in JOBS)))
    spans_sorted = sorted(spans)
    mk = spans_sorted[len(spans) // 2]
    # a step far above the median: report each tenant's longest launches (stderr)
    for step, sp in enumerate(spans):
        if sp > 2 * mk:
            sys.stderr.write("C4 step %d: %.1f ms\n" % (step, sp))
            for k in JOBS:
                sys.stderr.write("  %s span %.1f, host go %.3f submitted %.3f: %s\n" % (
                    k, res[k][step][1] - res[k][step][0], res[k][step][5][0], res[k][step][5][1],
                    json.dumps(res[k][step][4])))
    print(json.dumps({"config": "C4: triad 2^26, SpMV 2^20, stencil 8192^2, bf16 GEMM 4096^3 from 4 client processes "
                                "via slated (AUTO)",
                      "jobs": JOBS, "seq_cuda_ms": round(seq_ms, 3), "seq_slate_ms": round(seq_slate_ms, 3),
                      "best_sequential_ms": round(best_seq, 3),
                      "solo_ms": {k: round(v, 3) for k, v in solo.items()},
                      "solo_cuda_ms": {k: round(v, 3) for k, v in solo_cuda.items()},
                      "solo_slate_ms": {k: round(v, 3) for k, v in solo_slate.items()},
                      "corun_makespan_ms": round(mk, 3), "gain_vs_sequential": round(best_seq / mk, 4),
                      "gain_vs_seq_cuda": round(seq_ms / mk, 4),
                      "stp_median": round(sorted(stps)[len(stps) // 2], 4), "makespans_ms": [round(x, 3) for x in spans],
                      "resize_us": {"n": len(resize), "p50": round(sorted(resize)[len(resize) // 2], 2) if resize else None,
                                    "p99": round(float(np.percentile(resize, 99)), 2) if resize else None,
                                    "max": round(max(resize), 2) if resize else None,
                                    "over_50us": sum(1 for v in resize if v > 50.0)}}))


if __name__ == "__main__":
    main()
