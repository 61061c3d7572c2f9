"""Benchmark of the Slate slate-kernel path on B200 (contract: README/DESIGN.md §Measurement).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl slate|reference]

Workload (BASELINE.json configs[1], "C2"): a memory-bound CSR SpMV job (2^20 rows,
16 nnz/row, banded) co-run with a compute-bound Black-Scholes job (2^23 options x
32 volatility scenarios).  A job is a fixed number of back-to-back launches
(the paper loops kernels).  One STEP = one pair-job: both jobs submitted
to the Slate server from two sessions with AUTO placement -- the selector (Tab I
on the measured profiles) decides co-run vs solo and the split, the running
kernel shrinks on the arrival and grows on the completion of the other (no
relaunch).  value = pair-jobs per second (all ranks / max over ranks of the
device-timed region).  Beside it: the paper's throughput criterion
G = T_seq / T_corun against sequential CUDA (standalone kernels back to
back) and against Slate-sequential, plus STP / ANTT (Eyerman) for every
schedule, plain concurrent streams, resize latencies, and co-run utilisation.

Multi-GPU: independent per-GPU Slate instances (the path does not shard), one
process per GPU under torchrun, barrier + max over ranks, scaling "weak".
--impl reference: the CPU oracle (oracle/) on a bounded sample of the same
pair-job on the host cores, extrapolated to pair-jobs/s.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "co-run STP and ANTT vs sequential on 1 B200; HBM GB/s + FP32/TC % of peak"
CONFIG = {"workload": "C2: SpMV CSR 2^20 rows x 16 nnz (banded +-4096) co-run with Black-Scholes 2^23 options x 32 "
                      "scenarios; pair-job = 640 SpMV launches + 64 BS launches",
          "spmv_rows": 1 << 20, "spmv_nnz_per_row": 16, "bs_options": 1 << 23, "bs_scenarios": 32,
          "spmv_launches_per_job": 640, "bs_launches_per_job": 64,
          "l2": "inputs 137 MB + 168 MB > 126 MB L2; 256 MB L2 flush between timed steps",
          "parallelism": "replicas (independent per-GPU Slate servers, no collective)"}
R_SPMV, R_BS = CONFIG["spmv_launches_per_job"], CONFIG["bs_launches_per_job"]
N_ROWS, N_OPT, P_SCEN = CONFIG["spmv_rows"], CONFIG["bs_options"], CONFIG["bs_scenarios"]
FP32_FLOPS_PER_OPTION_SCENARIO = 50   # DESIGN.md §Work (Black-Scholes with the A&S normal CDF)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="slate", choices=["slate", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample-s", type=float, default=12.0, help="target seconds of oracle work for cpu_baseline")
    return ap.parse_args()


# ------------------------------------------------------------------ distributed plumbing
def dist_init(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        import torch
        torch.cuda.set_device(local)
        dist.init_process_group("nccl" if torch.cuda.is_available() else "gloo")
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def allmax(world, x):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ------------------------------------------------------------------ CPU oracle (reference / cpu_baseline)
_ORACLE_INPUTS = {}


def oracle_pair_seconds(sample_s):
    """Time the oracle on a bounded sample of the pair-job's blocks and
    extrapolate to one whole pair-job (640 SpMV + 64 BS launches)."""
    from oracle import tenants as OT
    from paper_conf_ipps_allenf019_b200 import inputs as I
    if not _ORACLE_INPUTS:
        _ORACLE_INPUTS["spmv"] = I.spmv_inputs(N_ROWS, I.seed_for(2, 0))
        _ORACLE_INPUTS["bs"] = I.bs_inputs(N_OPT, I.seed_for(2, 1))
    rp, col, val, x = _ORACLE_INPUTS["spmv"]
    S_, X_, T_, r = _ORACLE_INPUTS["bs"]
    sig = I.bs_sigmas(P_SCEN)
    n_bs_blocks, n_sp_blocks = N_OPT // 1024, N_ROWS // 32
    # calibrate a tiny sample, then size the real sample to ~sample_s seconds
    t0 = time.perf_counter(); OT.blackscholes(S_, X_, T_, r, sig, blocks=range(2)); t_bs = (time.perf_counter() - t0) / 2
    t0 = time.perf_counter(); OT.spmv_csr(rp, col, val, x, blocks=range(64)); t_sp = (time.perf_counter() - t0) / 64
    k_bs = max(2, int(0.5 * sample_s / max(t_bs, 1e-6)))
    k_sp = max(64, int(0.5 * sample_s / max(t_sp, 1e-6)))
    k_bs, k_sp = min(k_bs, n_bs_blocks), min(k_sp, n_sp_blocks)
    t0 = time.perf_counter(); OT.blackscholes(S_, X_, T_, r, sig, blocks=range(k_bs)); t_bs = (time.perf_counter() - t0) / k_bs
    t0 = time.perf_counter(); OT.spmv_csr(rp, col, val, x, blocks=range(k_sp)); t_sp = (time.perf_counter() - t0) / k_sp
    pair_s = R_BS * n_bs_blocks * t_bs + R_SPMV * n_sp_blocks * t_sp
    sample = "oracle (fp64 numpy, block by block) on %d of %d BS blocks and %d of %d SpMV blocks, " \
             "extrapolated to %d BS + %d SpMV launches" % (k_bs, n_bs_blocks, k_sp, n_sp_blocks, R_BS, R_SPMV)
    return pair_s, sample


def run_reference(args, world, rank):
    if rank != 0:
        return
    for _ in range(args.warmup):
        oracle_pair_seconds(min(2.0, args.cpu_sample_s / 4))
    times = []
    sample = ""
    for _ in range(args.steps):
        s, sample = oracle_pair_seconds(args.cpu_sample_s / max(1, args.steps))
        times.append(s)
    t = statistics.median(times)
    v = 1.0 / t
    line = {"metric": METRIC, "value": v, "unit": "pair-jobs/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": CONFIG, "impl": "reference",
            "cpu_baseline": {"value": v, "unit": "pair-jobs/s", "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": "pair-jobs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ clocks
class Clocks:
    def __init__(self, index):
        self.path = "/tmp/slate_bench_clocks_%d.csv" % os.getpid()
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(index), "--query-gpu=" + q,
                                       "--format=csv,noheader,nounits", "-lms", "200"], stdout=self.f,
                                      stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if not self.p:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.close()
        rows = [l.strip().split(", ") for l in open(self.path) if l.strip()]
        os.unlink(self.path)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows if len(r) >= 9 for i in range(4) if r[5 + i].strip() == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


# ------------------------------------------------------------------ the GPU workload
class Pair:
    def __init__(self, S, dev):
        import torch
        from paper_conf_ipps_allenf019_b200 import inputs as I
        self.S, self.torch = S, torch
        rp, col, val, x = I.spmv_inputs(N_ROWS, I.seed_for(2, 0))
        S_, X_, T_, r = I.bs_inputs(N_OPT, I.seed_for(2, 1))
        sig = I.bs_sigmas(P_SCEN)
        self.host = {"rp": rp, "col": col, "val": val, "x": x, "S": S_, "X": X_, "T": T_, "sig": sig}
        self.pinned = {k: torch.from_numpy(v).pin_memory() for k, v in self.host.items()}
        self.d = {k: v.to(dev) for k, v in self.pinned.items()}
        self.d["y"] = torch.zeros(N_ROWS, device=dev)
        self.d["call"] = torch.zeros(N_OPT, device=dev)
        self.d["put"] = torch.zeros(N_OPT, device=dev)
        self.out_pinned = {k: torch.empty(self.d[k].numel(), dtype=torch.float32).pin_memory()
                           for k in ("y", "call", "put")}
        self.nnz = int(rp[-1])
        self.r = float(r)
        self.flush_buf = torch.empty(64 << 20, dtype=torch.float32, device=dev)   # 256 MB > L2
        torch.cuda.synchronize()
        d = self.d
        self.spmv_args, self.spmv_grid = S.spmv_args(d["rp"], d["col"], d["val"], d["x"], d["y"])
        self.bs_args, self.bs_grid = S.bs_args(d["S"], d["X"], d["T"], d["call"], d["put"], d["sig"], self.r)
        self.h2d_bytes = sum(v.numel() * v.element_size() for v in self.pinned.values())
        self.d2h_bytes = sum(v.numel() * v.element_size() for v in self.out_pinned.values())
        # algorithmic work per launch
        self.spmv_bytes = 8.0 * self.nnz + 4.0 * (N_ROWS + 1) + 4.0 * N_ROWS + 4.0 * N_ROWS
        self.bs_bytes = 20.0 * N_OPT + 4.0 * P_SCEN
        self.bs_flops = float(FP32_FLOPS_PER_OPTION_SCENARIO) * N_OPT * P_SCEN

    def flush_l2(self):
        self.flush_buf.fill_(1.0)
        self.torch.cuda.synchronize()

    def copy_in(self):
        for k, v in self.pinned.items():
            self.d[k].copy_(v, non_blocking=True)
        self.torch.cuda.synchronize()

    def copy_out(self):
        for k, v in self.out_pinned.items():
            v.copy_(self.d[k], non_blocking=True)
        self.torch.cuda.synchronize()


def submit(sess, kernel, args, grid, reps, **kw):
    return [sess.launch(kernel, args, grid, **kw) for _ in range(reps)]


def collect(sess, ids):
    sess.sync(0)
    qs = [sess.query(i) for i in ids]
    bad = [q for q in qs if q["state"] != 2 or q["end_ms"] <= 0]
    if bad:
        raise RuntimeError("%d launches did not complete: %r" % (len(bad), bad[0]))
    return qs


def span(qs):
    return min(q["start_ms"] for q in qs), max(q["end_ms"] for q in qs)


def run_schedule(name, pair, sA, sB, kA, kB):
    """One pair-job under a schedule; A = Black-Scholes job, B = SpMV job.
    Returns (makespan_ms, turnaround_A_ms, turnaround_B_ms, queries_A, queries_B)."""
    S = pair.S
    if name == "seq_cuda":          # vanilla CUDA: the two jobs back to back, original kernels
        a = submit(sA, kA, pair.bs_args, pair.bs_grid, R_BS, mode=S.MODE_STANDALONE)
        b = submit(sA, kB, pair.spmv_args, pair.spmv_grid, R_SPMV, mode=S.MODE_STANDALONE)
        qa, qb = collect(sA, a), collect(sA, b)
    elif name == "seq_slate":       # Slate workers on all SMs, back to back
        a = submit(sA, kA, pair.bs_args, pair.bs_grid, R_BS, placement=S.PLACE_SOLO)
        b = submit(sA, kB, pair.spmv_args, pair.spmv_grid, R_SPMV, placement=S.PLACE_SOLO)
        qa, qb = collect(sA, a), collect(sA, b)
    elif name == "streams":         # plain concurrent streams: hardware leftover policy
        a = submit(sA, kA, pair.bs_args, pair.bs_grid, R_BS, mode=S.MODE_STANDALONE)
        b = submit(sB, kB, pair.spmv_args, pair.spmv_grid, R_SPMV, mode=S.MODE_STANDALONE)
        qa, qb = collect(sA, a), collect(sB, b)
    elif name == "slate":           # Slate AUTO: selector + split + shrink on arrival + grow on completion
        a = submit(sA, kA, pair.bs_args, pair.bs_grid, R_BS, placement=S.PLACE_AUTO)
        b = submit(sB, kB, pair.spmv_args, pair.spmv_grid, R_SPMV, placement=S.PLACE_AUTO)
        qa, qb = collect(sA, a), collect(sB, b)
    elif name == "slate_forced":    # diagnostic: co-run regardless of Tab I, split from the T(s) curves;
        n, s_b = pair.n_sms, pair.split   # the server shrinks A on B's arrival and grows the survivor
        a = submit(sA, kA, pair.bs_args, pair.bs_grid, R_BS, placement=S.PLACE_AUTO)
        b = submit(sB, kB, pair.spmv_args, pair.spmv_grid, R_SPMV, placement=S.PLACE_CORUN, sm=(n - s_b, n - 1))
        qa, qb = collect(sA, a), collect(sB, b)
    else:
        raise ValueError(name)
    a0, a1 = span(qa)
    b0, b1 = span(qb)
    t0 = min(a0, b0)
    return max(a1, b1) - t0, a1 - t0, b1 - t0, qa, qb


def stp_antt(solo, turn):
    stp = sum(s / t for s, t in zip(solo, turn))
    antt = sum(t / s for s, t in zip(solo, turn)) / len(solo)
    return stp, antt


def median_schedule(name, pair, sA, sB, kA, kB, reps):
    rs = []
    for _ in range(reps):
        pair.flush_l2()
        rs.append(run_schedule(name, pair, sA, sB, kA, kB))
    rs.sort(key=lambda r: r[0])
    return rs[len(rs) // 2]


def run_slate(args, world, rank, local):
    import torch
    from paper_conf_ipps_allenf019_b200 import slate as S
    dev = "cuda:%d" % local
    torch.cuda.set_device(local)
    peaks = {}
    pk_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(pk_path):
        peaks = json.load(open(pk_path))
        os.environ.setdefault("SLATE_PEAK_HBM_GBPS", str(peaks.get("hbm_gbs", 6650.0)))
        os.environ.setdefault("SLATE_PEAK_TC_TFLOPS", str(peaks.get("bf16_tflops", 1590.0)))
    peak_hbm = float(peaks.get("hbm_gbs", 6650.0))
    sA, sB = S.Session(None, local), S.Session(None, local)
    info = sA.info()
    peak_fp32 = info["peak_fp32_gflops"] / 1e3   # TFLOP/s, from 148 SMs x 128 lanes x 2 x clock
    pair = Pair(S, dev)
    kA, kB = sA.register_kernel(S.KIND_BLACKSCHOLES), sA.register_kernel(S.KIND_SPMV_CSR)
    # the profile table: solo T(s) curves that feed the selector and the split
    prof_bs = sA.profile(kA, pair.bs_args, pair.bs_grid, S.PROF_CURVE)
    prof_sp = sA.profile(kB, pair.spmv_args, pair.spmv_grid, S.PROF_CURVE)
    pair.n_sms = info["num_sms"]
    pair.split, _ = S.choose_split(dict(zip(prof_bs["curve_sms"], prof_bs["curve_ms"])),
                                   dict(zip(prof_sp["curve_sms"], prof_sp["curve_ms"])), pair.n_sms)

    # ---- baselines (each the median of 3 runs after one warm-up)
    base = {}
    for name in ("seq_cuda", "seq_slate", "streams", "slate_forced"):
        run_schedule(name, pair, sA, sB, kA, kB)
        base[name] = median_schedule(name, pair, sA, sB, kA, kB, 3)
    # solo job times: each job alone on the GPU with the original kernels (the T_k of P:L99)
    solo_a = base["seq_cuda"][1]
    solo_b = base["seq_cuda"][0] - base["seq_cuda"][1]
    t_seq = base["seq_cuda"][0]

    # ---- the timed hot path: Slate co-run steps
    for _ in range(max(3, args.warmup)):
        pair.flush_l2()
        run_schedule("slate", pair, sA, sB, kA, kB)
    clocks = Clocks(local)
    steps = []
    barrier(world)
    torch.cuda.synchronize()
    for _ in range(args.steps):
        pair.flush_l2()
        steps.append(run_schedule("slate", pair, sA, sB, kA, kB))
    torch.cuda.synchronize()
    barrier(world)
    clk = clocks.stop()
    total_ms = sum(s[0] for s in steps)
    total_ms_max = allmax(world, total_ms)
    value = world * args.steps / (total_ms_max / 1e3)
    med = sorted(steps, key=lambda s: s[0])[len(steps) // 2]
    makespan = med[0]

    # ---- e2e: host buffers in, the same co-run through the public API, results out
    e2e_times = []
    for i in range(args.steps + 1):
        pair.flush_l2()
        t0 = time.perf_counter()
        pair.copy_in()
        run_schedule("slate", pair, sA, sB, kA, kB)
        pair.copy_out()
        if i:
            e2e_times.append(time.perf_counter() - t0)
    e2e_s = allmax(world, statistics.median(e2e_times))

    # ---- metrics
    def sched_summary(r):
        mk, ta, tb = r[0], r[1], r[2]
        stp, antt = stp_antt([solo_a, solo_b], [ta, tb])
        return {"makespan_ms": round(mk, 3), "turnaround_bs_ms": round(ta, 3), "turnaround_spmv_ms": round(tb, 3),
                "gain_vs_seq_cuda": round(t_seq / mk, 4), "stp": round(stp, 4), "antt": round(antt, 4)}

    schedules = {k: sched_summary(v) for k, v in base.items()}
    schedules["slate_corun"] = sched_summary(med)
    qa, qb = med[3], med[4]
    # per-kernel durations in the co-run (CUDA events on the launching streams)
    dur_bs = [q["end_ms"] - q["start_ms"] for q in qa]
    dur_sp = [q["end_ms"] - q["start_ms"] for q in qb]
    resize = [v for q in qa + qb for v in q["resize_us"]]
    topups = sum(q["n_topups"] for q in qa + qb)
    sum_bs, sum_sp = sum(dur_bs), sum(dur_sp)
    if sum_bs >= sum_sp:
        avg = sum_bs / len(dur_bs)
        ach = pair.bs_flops / (avg * 1e-3) / 1e12
        roof = {"kernel": "slate_worker<BlackScholes>", "bound": "alu", "achieved": round(ach, 3),
                "peak": round(peak_fp32, 2), "unit": "TFLOP/s", "frac": round(ach / peak_fp32, 4),
                "traffic": None, "avg_launch_ms": round(avg, 5),
                "peak_source": "FP32 = 148 SMs x 128 lanes x 2 flop x 1.965 GHz (DESIGN.md §Roofline)"}
    else:
        avg = sum_sp / len(dur_sp)
        ach = pair.spmv_bytes / (avg * 1e-3) / 1e9
        roof = {"kernel": "slate_worker<SpmvCsr>", "bound": "hbm", "achieved": round(ach, 1), "peak": peak_hbm,
                "unit": "GB/s", "frac": round(ach / peak_hbm, 4), "traffic": None, "avg_launch_ms": round(avg, 5),
                "peak_source": "MEASURED_PEAKS.json hbm_gbs" if peaks else "fallback 6650 GB/s"}
    ncu_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(ncu_path):
        tr = json.load(open(ncu_path)).get(roof["kernel"])
        if tr:
            roof["traffic"] = tr
    job_bytes = R_BS * pair.bs_bytes + R_SPMV * pair.spmv_bytes
    job_flops = R_BS * pair.bs_flops
    util = {"U_HBM": round(job_bytes / (makespan * 1e-3) / 1e9 / peak_hbm, 4),
            "U_FP32": round(job_flops / (makespan * 1e-3) / 1e12 / peak_fp32, 4),
            "hbm_gbps": round(job_bytes / (makespan * 1e-3) / 1e9, 1),
            "fp32_tflops": round(job_flops / (makespan * 1e-3) / 1e12, 3)}
    util["U_HBM_plus_U_FP32"] = round(util["U_HBM"] + util["U_FP32"], 4)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        pair_s, sample = oracle_pair_seconds(args.cpu_sample_s)
        cpu = {"value": 1.0 / pair_s, "unit": "pair-jobs/s", "cores": 1, "kind": "oracle", "sample": sample}

    def prof_view(p):
        return {"solo_ms": round(p["solo_ms"], 4), "hbm_gbps": round(p["hbm_gbps"], 1),
                "fp32_gflops": round(p["fp32_gflops"], 1), "category": p["category_name"],
                "curve": {str(s): round(t, 4) for s, t in zip(p["curve_sms"], p["curve_ms"])}}

    n_launch = sum(len(s[3]) + len(s[4]) for s in steps) + sum(q["n_topups"] for s in steps for q in s[3] + s[4])
    line = {
        "metric": METRIC, "value": round(value, 4), "unit": "pair-jobs/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms_max / args.steps, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": CONFIG,
        "gain_vs_sequential": round(t_seq / makespan, 4),
        "gain_vs_slate_sequential": round(base["seq_slate"][0] / makespan, 4),
        "stp": schedules["slate_corun"]["stp"], "antt": schedules["slate_corun"]["antt"],
        "schedules": schedules, "forced_split_sms_spmv": pair.split,
        "resize_us": {"n": len(resize), "p50": round(statistics.median(resize), 2) if resize else None,
                      "p99": round(float(np.percentile(resize, 99)), 2) if resize else None,
                      "max": round(max(resize), 2) if resize else None, "topups": topups},
        "corun_utilisation": util,
        "profiles": {"blackscholes": prof_view(prof_bs), "spmv": prof_view(prof_sp)},
        "roofline": roof,
        "clocks": clk,
        "e2e": {"value": round(world / e2e_s, 4), "unit": "pair-jobs/s", "h2d_bytes_per_step": pair.h2d_bytes,
                "d2h_bytes_per_step": pair.d2h_bytes},
        "gpu_launches": n_launch,
    }
    if cpu:
        line["cpu_baseline"] = cpu
    if rank == 0:
        print(json.dumps(line), flush=True)
    sA.close()
    sB.close()


def main():
    args = parse()
    world, rank, local = dist_init(args)
    if args.impl == "reference":
        run_reference(args, world, rank)
    else:
        run_slate(args, world, rank, local)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
