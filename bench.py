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
SPLIT_SLACK = float(os.environ.get("SLATE_SPLIT_SLACK", "0.05"))   # reading Q41


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="slate", choices=["slate", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-c3", action="store_true", help="skip the C3 (GEMM + copy) companion measurement")
    ap.add_argument("--no-c4", action="store_true", help="skip the C4 (4 client processes via slated) measurement")
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
        if torch.cuda.is_available():
            torch.cuda.set_device(local)
        dist.init_process_group("nccl" if torch.cuda.is_available() else "gloo")
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def allmax(world, x):
    """Max over ranks (the timed region is the slowest rank's, contract)."""
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(x)], device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def aggregate(world, steps, total_ms_per_rank_max):
    """Whole-job throughput: pair-jobs of every rank / the slowest rank's device time."""
    return world * steps / (total_ms_per_rank_max / 1e3)


def gather(world, obj):
    """Every rank's `obj` (a small JSON-able dict) on every rank."""
    if world == 1:
        return [obj]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, obj)
    return out


def c5_aggregate(per_rank):
    """SURVEY §8(e) / BASELINE configs[4] (C5): independent per-GPU Slate
    instances, two client sessions per GPU (the C2 pair).  The box's wall-clock
    gain G_agg = max_g T_g^seq / max_g makespan_g (the slowest GPU sets both),
    the sum of the per-GPU STPs, and the per-GPU gains (to expose stragglers).
    per_rank: [{"t_seq_ms", "makespan_ms", "stp"}] in rank order."""
    t_seq = max(r["t_seq_ms"] for r in per_rank)
    mk = max(r["makespan_ms"] for r in per_rank)
    return {"gpus": len(per_rank), "clients": 2 * len(per_rank),
            "g_agg": round(t_seq / mk, 4), "stp_sum": round(sum(r["stp"] for r in per_rank), 4),
            "per_gpu_gain": [round(r["t_seq_ms"] / r["makespan_ms"], 4) for r in per_rank],
            "t_seq_ms_max": round(t_seq, 3), "makespan_ms_max": round(mk, 3)}


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


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _oracle_worker(job):
    """One process of the all-cores oracle run: blocks [lo, hi) of one tenant."""
    from oracle import tenants as OT
    from paper_conf_ipps_allenf019_b200 import inputs as I
    kind, lo, hi = job
    if kind == "bs":
        S_, X_, T_, r = _ORACLE_INPUTS["bs"]
        OT.blackscholes(S_, X_, T_, r, I.bs_sigmas(P_SCEN), blocks=range(lo, hi))
    else:
        rp, col, val, x = _ORACLE_INPUTS["spmv"]
        OT.spmv_csr(rp, col, val, x, blocks=range(lo, hi))
    return hi - lo


def oracle_pair_seconds_all_cores(sample_s):
    """SURVEY §8(d) oracle timing (ii): the same oracle, its blocks spread over
    every host core by worker processes (the blocks are independent), each
    tenant timed for ~sample_s/2 of wall clock and extrapolated to a pair-job."""
    import multiprocessing as mp
    oracle_pair_seconds(0.2)                      # inputs generated before the fork
    cores = len(os.sched_getaffinity(0))
    n_bs_blocks, n_sp_blocks = N_OPT // 1024, N_ROWS // 32
    os.environ["OMP_NUM_THREADS"] = "1"
    per_block = {}
    with mp.get_context("fork").Pool(cores) as pool:
        for kind, total, first in (("bs", n_bs_blocks, 4), ("spmv", n_sp_blocks, 256)):
            t0 = time.perf_counter()
            pool.map(_oracle_worker, [(kind, i * first, (i + 1) * first) for i in range(cores)])
            t_cal = (time.perf_counter() - t0) / (first * cores)
            k = min(total // cores, max(first, int(0.5 * sample_s / max(t_cal * cores, 1e-9))))
            t0 = time.perf_counter()
            done = sum(pool.map(_oracle_worker, [(kind, i * k, (i + 1) * k) for i in range(cores)]))
            per_block[kind] = (time.perf_counter() - t0) / done
    pair_s = R_BS * n_bs_blocks * per_block["bs"] + R_SPMV * n_sp_blocks * per_block["spmv"]
    return pair_s, cores


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
    """SM clock and clock-event reasons sampled through NVML every 50 ms while
    the timed region runs (a thread; nvidia-smi -lms buffers its output and
    lost the samples of sub-second regions); the first sample is taken before
    the timed work starts.  (Resize latencies are the same with a 10-ms
    sampler and without one: profiles/r2_resize_nvml_interference.json.)"""

    NAMES = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
             ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
             ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
             ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
             ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, index):
        import threading
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.stop_ev = threading.Event()
        self.th = None
        try:
            import pynvml as N
            N.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            phys = int(vis.split(",")[index]) if vis and vis.split(",")[index].strip().isdigit() else index
            self.N, self.h = N, N.nvmlDeviceGetHandleByIndex(phys)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
            self._sample()   # the first sample before the timed work starts (the recipe: start before)
            self.th = threading.Thread(target=self._run, daemon=True)
            self.th.start()
        except Exception:
            self.th = None

    def _sample(self):
        N = self.N
        try:
            self.samples.append(N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM))
            r = N.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            self.reasons.update(n for n, c in self.NAMES if getattr(N, c, 0) and (r & getattr(N, c, 0)))
        except Exception:
            pass

    def _run(self):
        while not self.stop_ev.wait(0.05):
            self._sample()

    def stop(self):
        if not self.th:
            return None
        self.stop_ev.set()
        self.th.join(timeout=2)
        if not self.samples:
            return None
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples), "source": "nvml, 50 ms"}


# ------------------------------------------------------------------ the GPU workload
class Job:
    """One tenant job: `reps` back-to-back launches of one kernel."""

    def __init__(self, name, kind, args, grid, reps, bytes_, fp32, tc):
        self.name, self.kind, self.args, self.grid, self.reps = name, kind, args, grid, reps
        self.bytes, self.fp32, self.tc = bytes_, fp32, tc      # algorithmic work per launch


class Workload:
    """A pair of jobs A (submitted first) and B (arrives `arrival_ms` later)."""

    def __init__(self, name, a, b, keep, arrival_frac=0.0):
        self.name, self.a, self.b, self._keep, self.arrival_frac = name, a, b, keep, arrival_frac
        self.arrival_ms = 0.0


def make_c2(S, dev, pinned=None):
    """The C2 pair on device buffers; `pinned` (another C2 workload's pinned host
    inputs) gives a second device set over the same host data (e2e pipelining)."""
    import torch
    from paper_conf_ipps_allenf019_b200 import inputs as I
    r = I.bs_inputs(8, I.seed_for(2, 1))[3]
    if pinned is None:
        rp, col, val, x = I.spmv_inputs(N_ROWS, I.seed_for(2, 0))
        S_, X_, T_, r = I.bs_inputs(N_OPT, I.seed_for(2, 1))
        sig = I.bs_sigmas(P_SCEN)
        host = {"rp": rp, "col": col, "val": val, "x": x, "S": S_, "X": X_, "T": T_, "sig": sig}
        pinned = {k: torch.from_numpy(v).pin_memory() for k, v in host.items()}
    rp = pinned["rp"].numpy()
    d = {k: v.to(dev) for k, v in pinned.items()}
    d["y"] = torch.zeros(N_ROWS, device=dev)
    d["call"] = torch.zeros(N_OPT, device=dev)
    d["put"] = torch.zeros(N_OPT, device=dev)
    torch.cuda.synchronize()
    nnz = int(rp[-1])
    spmv_args, spmv_grid = S.spmv_args(d["rp"], d["col"], d["val"], d["x"], d["y"])
    bs_args, bs_grid = S.bs_args(d["S"], d["X"], d["T"], d["call"], d["put"], d["sig"], float(r))
    bs = Job("blackscholes", S.KIND_BLACKSCHOLES, bs_args, bs_grid, R_BS, 20.0 * N_OPT + 4.0 * P_SCEN,
             float(FP32_FLOPS_PER_OPTION_SCENARIO) * N_OPT * P_SCEN, 0.0)
    sp = Job("spmv", S.KIND_SPMV_CSR, spmv_args, spmv_grid, R_SPMV,
             8.0 * nnz + 4.0 * (N_ROWS + 1) + 4.0 * N_ROWS + 4.0 * N_ROWS, 2.0 * nnz, 0.0)
    w = Workload("C2", bs, sp, d)
    w.pinned = pinned
    w.out_names = ("y", "call", "put")
    w.out_pinned = {k: torch.empty(d[k].numel(), dtype=torch.float32).pin_memory() for k in w.out_names}
    w.h2d_bytes = sum(v.numel() * v.element_size() for v in pinned.values())
    w.d2h_bytes = sum(v.numel() * v.element_size() for v in w.out_pinned.values())
    return w


C3 = {"workload": "C3: tensor-core bf16 GEMM 8192^3 (tcgen05) co-run with STREAM copy 2^30 fp32 (4 GiB), copy "
                  "arriving at 25% of the GEMM job (dynamic resize mid-run)",
      "gemm_launches_per_job": int(os.environ.get("SLATE_C3_REPS", "1")),
      "copy_launches_per_job": int(os.environ.get("SLATE_C3_REPS", "1"))}


def make_c3(S, dev):
    import torch
    g = torch.Generator(device=dev)
    g.manual_seed(20190520 + 300)
    m = n = k = 8192
    A = (torch.rand(m, k, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
    B = (torch.rand(n, k, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
    C = torch.zeros(m, n, device=dev)
    cb = torch.rand(1 << 30, device=dev, generator=g)
    ca = torch.empty(1 << 30, device=dev)
    torch.cuda.synchronize()
    gargs, ggrid = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
    cargs, cgrid = S.copy_args(ca, cb)
    ge = Job("gemm_bf16", S.KIND_GEMM_BF16, gargs, ggrid, C3["gemm_launches_per_job"],
             2.0 * (m * k + n * k) + 4.0 * m * n, 0.0, 2.0 * m * n * k)
    cp = Job("copy", S.KIND_COPY, cargs, cgrid, C3["copy_launches_per_job"], 8.0 * (1 << 30), 0.0, 0.0)
    return Workload("C3", ge, cp, (A, B, C, ca, cb), arrival_frac=0.25)


def submit(sess, kernel, job, **kw):
    """A job: `reps` launches of its kernel in one slate_launch_n call."""
    return sess.launch_n(kernel, job.args, job.grid, job.reps, **kw)


def collect(sess, ids):
    sess.sync(0)
    qs = [sess.query(i) for i in ids]
    bad = [q for q in qs if q["state"] != 2 or q["end_ms"] <= 0]
    if bad:
        raise RuntimeError("%d launches did not complete: %r" % (len(bad), bad[0]))
    return qs


def span(qs):
    return min(q["start_ms"] for q in qs), max(q["end_ms"] for q in qs)


def spin_ms(ms):
    t0 = time.perf_counter()
    while (time.perf_counter() - t0) * 1e3 < ms:
        pass


def run_schedule(name, w, sA, sB, kA, kB, S):
    """One pair-job under a schedule.  Returns (makespan, turnaround_A, turnaround_B, qa, qb) in ms,
    turnarounds measured from the first launch's start (B's arrival delay included)."""
    a, b = w.a, w.b
    if name == "seq_cuda":          # vanilla CUDA: the two jobs back to back, original kernels
        ia = submit(sA, kA, a, mode=S.MODE_STANDALONE)
        ib = submit(sA, kB, b, mode=S.MODE_STANDALONE)
        qa, qb = collect(sA, ia), collect(sA, ib)
    elif name == "seq_cuda_ba":     # vanilla CUDA, the other order: B's job first
        ib = submit(sA, kB, b, mode=S.MODE_STANDALONE)
        ia = submit(sA, kA, a, mode=S.MODE_STANDALONE)
        qa, qb = collect(sA, ia), collect(sA, ib)
    elif name == "seq_slate":       # Slate workers on all SMs, back to back
        ia = submit(sA, kA, a, placement=S.PLACE_SOLO)
        ib = submit(sA, kB, b, placement=S.PLACE_SOLO)
        qa, qb = collect(sA, ia), collect(sA, ib)
    elif name == "seq_slate_ba":
        ib = submit(sA, kB, b, placement=S.PLACE_SOLO)
        ia = submit(sA, kA, a, placement=S.PLACE_SOLO)
        qa, qb = collect(sA, ia), collect(sA, ib)
    elif name == "streams":         # plain concurrent streams: hardware leftover policy
        ia = submit(sA, kA, a, mode=S.MODE_STANDALONE)
        spin_ms(w.arrival_ms)
        ib = submit(sB, kB, b, mode=S.MODE_STANDALONE)
        qa, qb = collect(sA, ia), collect(sB, ib)
    elif name == "slate":           # Slate AUTO: selector + split + shrink on arrival + grow on completion
        ia = submit(sA, kA, a, placement=S.PLACE_AUTO)
        spin_ms(w.arrival_ms)
        ib = submit(sB, kB, b, placement=S.PLACE_AUTO)
        qa, qb = collect(sA, ia), collect(sB, ib)
    elif name == "slate_antt":      # Slate AUTO with the turnaround-aware split (reading Q41; the default is Q10's)
        sA.set_split_objective("antt", SPLIT_SLACK)
        try:
            ia = submit(sA, kA, a, placement=S.PLACE_AUTO)
            spin_ms(w.arrival_ms)
            ib = submit(sB, kB, b, placement=S.PLACE_AUTO)
            qa, qb = collect(sA, ia), collect(sB, ib)
        finally:
            sA.set_split_objective("makespan")
    elif name == "slate_table":     # Slate AUTO with the paper's Tab I alone deciding (reading Q8)
        sA.set_policy(S.POLICY_TABLE)
        try:
            ia = submit(sA, kA, a, placement=S.PLACE_AUTO)
            spin_ms(w.arrival_ms)
            ib = submit(sB, kB, b, placement=S.PLACE_AUTO)
            qa, qb = collect(sA, ia), collect(sB, ib)
        finally:
            sA.set_policy(S.POLICY_HYBRID)
    elif name == "slate_forced":    # co-run regardless of Tab I, split from the T(s) curves
        # B's first launch is placed on the top s_b SMs (A shrinks); the rest of
        # B's job queues behind it on the same range, and when A's job drains
        # the server grows B to every SM -- the AUTO co-run's shape
        n, s_b = w.n_sms, w.split
        ia = submit(sA, kA, a, placement=S.PLACE_AUTO)
        spin_ms(w.arrival_ms)
        ib = [sB.launch(kB, b.args, b.grid, placement=S.PLACE_CORUN, sm=(n - s_b, n - 1))]
        if b.reps > 1:
            ib += sB.launch_n(kB, b.args, b.grid, b.reps - 1, placement=S.PLACE_AUTO)
        qa, qb = collect(sA, ia), collect(sB, ib)
    else:
        raise ValueError(name)
    a0, a1 = span(qa)
    b0, b1 = span(qb)
    t0 = min(a0, b0)
    # (makespan, turnaround A, turnaround B, queries A, queries B, job time A, job time B):
    # a job's time is first start to last end of its own launches
    return max(a1, b1) - t0, a1 - t0, b1 - t0, qa, qb, a1 - a0, b1 - b0


def stp_antt(solo, turn):
    stp = sum(s / t for s, t in zip(solo, turn))
    antt = sum(t / s for s, t in zip(solo, turn)) / len(solo)
    return stp, antt


def flush_l2(buf):
    buf.fill_(1.0)
    import torch
    torch.cuda.synchronize()


def median_schedule(name, w, sA, sB, kA, kB, S, flush, reps, spread=None):
    rs = []
    for _ in range(reps):
        flush_l2(flush)
        rs.append(run_schedule(name, w, sA, sB, kA, kB, S))
    rs.sort(key=lambda r: r[0])
    if spread is not None:   # makespan min / max over the timed runs
        spread[name] = {"runs": len(rs), "min_ms": round(rs[0][0], 3), "max_ms": round(rs[-1][0], 3)}
    return rs[len(rs) // 2]


def resize_storm(S, sess, job, n_sms, n_resizes=200, per_launch=12, gap_us=100.0, seed=20190520 + 303):
    """SURVEY §8(d) C3 resize storm: during each GEMM launch, the host alternates a
    shrink to a random sub-range (>= 16 SMs) and a grow back to all SMs every
    gap_us, up to `per_launch` times, until n_resizes were issued; each resize's
    latency is measured by the server on the device clock (reading Q30)."""
    import random
    rng = random.Random(seed)
    k = sess.register_kernel(job.kind)
    lat = {"shrink": [], "grow": []}
    issued = superseded = 0
    while issued < n_resizes:
        lid = sess.launch(k, job.args, job.grid, placement=S.PLACE_CORUN, sm=(0, n_sms - 1))
        spin_ms(0.05)
        for i in range(min(per_launch, n_resizes - issued)):
            if i % 2 == 0:
                lo = rng.randrange(0, n_sms - 16)
                hi = rng.randrange(lo + 15, n_sms)
                if lo == 0 and hi == n_sms - 1:
                    hi -= 1
            else:
                lo, hi = 0, n_sms - 1
            st = sess.resize(lid, lo, hi)
            issued += 1
            if st == S.DONE:
                break
            spin_ms(gap_us * 1e-3)
        sess.resize(lid, 0, n_sms - 1)
        sess.sync(lid)
        q = sess.query(lid)
        for v, kind in zip(q["resize_us"], q["resize_kind"]):
            lat[kind].append(v)
        superseded += q["n_superseded"]

    def stats(v):
        return {"n": len(v), "p50": round(statistics.median(v), 2) if v else None,
                "p99": round(float(np.percentile(v, 99)), 2) if v else None, "max": round(max(v), 2) if v else None}
    return {"tenant": "gemm_bf16 8192^3, one launch per %d resizes" % per_launch, "resizes_issued": issued,
            "gap_us": gap_us, "shrink_us": stats(lat["shrink"]), "grow_us": stats(lat["grow"]),
            "shrinks_superseded": superseded,   # overtaken by the next grow before completing: not timed
            "clock": "device %globaltimer mapped to the host clock (DESIGN.md Q30)"}


def prof_view(p):
    return {"solo_ms": round(p["solo_ms"], 4), "hbm_gbps": round(p["hbm_gbps"], 1),
            "fp32_gflops": round(p["fp32_gflops"], 1), "tc_tflops": round(p["tc_tflops"], 1),
            "category": p["category_name"],
            "curve": {str(s): round(t, 4) for s, t in zip(p["curve_sms"], p["curve_ms"])}}


def evaluate(w, S, sA, sB, flush, steps, warmup, peaks, timed=None):
    """Profiles, baselines and (if `timed` is None) `steps` timed Slate co-run steps.
    Returns a dict of results; `timed(callback)` lets the caller bracket the timed loop."""
    import torch
    info = sA.info()
    kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
    pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
    pb = sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
    w.n_sms = info["num_sms"]
    # the split the server's AUTO placement takes (reading Q10 + the Q29 saturation cap)
    ca, cb = dict(zip(pa["curve_sms"], pa["curve_ms"])), dict(zip(pb["curve_sms"], pb["curve_ms"]))
    mem_a, mem_b = pa["category_name"].endswith("_M"), pb["category_name"].endswith("_M")
    frac = float(os.environ.get("SLATE_SATURATION_FRAC", "0.95"))
    cap = frac < 1.0
    lo_b = w.n_sms - S.saturation_sms(ca, w.n_sms, frac) if cap and mem_a and not mem_b else 0
    hi_b = S.saturation_sms(cb, w.n_sms, frac) if cap and mem_b and not mem_a else 0
    # job-level curves: a job is `reps` launches of its kernel
    ja = {k: v * w.a.reps for k, v in ca.items()}
    jb = {k: v * w.b.reps for k, v in cb.items()}
    w.split, _ = S.choose_split(ja, jb, w.n_sms, 2, lo_b, hi_b)
    w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
    base, spread = {}, {}
    # every schedule gets 3 warm-up runs, then 10 timed runs; the
    # median is reported with the min and max.  Each schedule starts from an
    # idle GPU (a 0.2-s pause): back to back, ~100 runs of a 1-kW GEMM pair
    # (C3) left the co-run measured last in a lower-clock state (1.86 ms
    # against 1.74 ms; tools/c3_repeat.py showed the same drift in long series)
    for name in ("seq_cuda", "seq_cuda_ba", "seq_slate", "seq_slate_ba", "streams", "slate_table", "slate_forced",
                 "slate_antt"):
        torch.cuda.synchronize()
        time.sleep(0.2)
        for _ in range(3):
            run_schedule(name, w, sA, sB, kA, kB, S)
        base[name] = median_schedule(name, w, sA, sB, kA, kB, S, flush, 10, spread)
    # every job's solo time: alone on the whole GPU, as original kernels or as
    # workers (Slate-solo), whichever is faster, in either order -- the best
    # sequential schedule is the baseline of every gain
    solo_opts = {"a": {}, "b": {}}
    for name in ("seq_cuda", "seq_cuda_ba", "seq_slate", "seq_slate_ba"):
        solo_opts["a"][name] = base[name][5]
        solo_opts["b"][name] = base[name][6]
    solo_a = min(solo_opts["a"].values())
    solo_b = min(solo_opts["b"].values())
    t_best_seq = solo_a + solo_b
    t_seq = base["seq_cuda"][0]
    arr = w.arrival_ms
    # sequential STP / ANTT in both orders from the best solo times:
    # A first (B arriving at `arr` waits for A), or B first (as if B were there at 0)
    seq_orders = {"a_first": stp_antt([solo_a, solo_b], [solo_a, max(solo_a + solo_b - arr, 1e-9)]),
                  "b_first": stp_antt([solo_a, solo_b], [solo_a + solo_b, solo_b])}
    torch.cuda.synchronize()
    time.sleep(0.2)                       # the co-run starts from an idle GPU too
    for _ in range(max(3, warmup)):
        flush_l2(flush)
        run_schedule("slate", w, sA, sB, kA, kB, S)

    def loop():
        out = []
        for _ in range(steps):
            flush_l2(flush)
            out.append(run_schedule("slate", w, sA, sB, kA, kB, S))
        return out

    steps_out = timed(loop) if timed else loop()
    med = sorted(steps_out, key=lambda r: r[0])[len(steps_out) // 2]

    def summary(r):
        mk, ta, tb = r[0], r[1], r[2]
        # B's turnaround counts from its arrival; STP / ANTT against the best solo times
        stp, antt = stp_antt([solo_a, solo_b], [ta, max(tb - w.arrival_ms, 1e-9)])
        la = [q["end_ms"] - q["start_ms"] for q in r[3]]
        lb = [q["end_ms"] - q["start_ms"] for q in r[4]]
        return {"makespan_ms": round(mk, 3), "turnaround_%s_ms" % w.a.name: round(ta, 3),
                "turnaround_%s_ms" % w.b.name: round(tb, 3), "gain_vs_seq_cuda": round(t_seq / mk, 4),
                "gain_vs_best_sequential": round(t_best_seq / mk, 4),
                "stp": round(stp, 4), "antt": round(antt, 4),
                "stp_vs_sequential": {k: round(stp / v[0], 4) for k, v in seq_orders.items()},
                "antt_vs_sequential": {k: round(antt / v[1], 4) for k, v in seq_orders.items()},
                "launch_ms_%s" % w.a.name: [round(x, 3) for x in la] if len(la) <= 8 else round(sum(la) / len(la), 4),
                "launch_ms_%s" % w.b.name: [round(x, 3) for x in lb] if len(lb) <= 8 else round(sum(lb) / len(lb), 4)}

    sched = {k: summary(v) for k, v in base.items()}
    sched["slate_corun"] = summary(med)
    for k in base:
        sched[k]["makespan_spread"] = spread[k]
    sched["slate_corun"]["makespan_spread"] = {"runs": len(steps_out), "min_ms": round(min(r[0] for r in steps_out), 3),
                                               "max_ms": round(max(r[0] for r in steps_out), 3)}
    qa, qb = med[3], med[4]
    # resize latencies of every timed step (the median step alone holds two)
    resize = [v for r in steps_out for q in r[3] + r[4] for v in q["resize_us"]]
    mk = med[0]
    peak_hbm = float(peaks.get("hbm_gbs", 6650.0))
    peak_fp32 = info["peak_fp32_gflops"] / 1e3
    # a GEMM launch of ~1 ms timed on its own: the burst figure (B200_PROFILING.md)
    peak_tc = float(peaks.get("bf16_tflops", 1662.3))
    jb = w.a.reps * w.a.bytes + w.b.reps * w.b.bytes
    jf = w.a.reps * w.a.fp32 + w.b.reps * w.b.fp32
    jt = w.a.reps * w.a.tc + w.b.reps * w.b.tc
    util = {"U_HBM": round(jb / (mk * 1e-3) / 1e9 / peak_hbm, 4),
            "U_FP32": round(jf / (mk * 1e-3) / 1e12 / peak_fp32, 4),
            "U_TC": round(jt / (mk * 1e-3) / 1e12 / peak_tc, 4),
            "hbm_gbps": round(jb / (mk * 1e-3) / 1e9, 1)}
    util["U_sum"] = round(util["U_HBM"] + util["U_FP32"] + util["U_TC"], 4)
    # roofline of the kernel with the largest summed launch time in the co-run
    # a kernel's time per launch = its job's span / its launches: the launches of
    # a batch overlap (programmatic dependent launch; SpMV's producer warps start
    # before the previous launch ends), so one launch's start-to-end overstates it
    def per_launch(qs):
        return (max(q["end_ms"] for q in qs) - min(q["start_ms"] for q in qs)) / len(qs)
    durs = {w.a.name: per_launch(qa), w.b.name: per_launch(qb)}
    job = {w.a.name: w.a, w.b.name: w.b}
    top = max(durs, key=lambda k: durs[k] * len(qa if k == w.a.name else qb))
    j, avg = job[top], durs[top]
    # the worker kernel's name as ncu prints it (the key of profiles/ncu_traffic.json)
    kname = {"blackscholes": "slate_worker<BlackScholes>", "spmv": "spmv::spmv_worker",
             "gemm_bf16": "gemm::gemm_kernel<1>", "copy": "slate_worker<Copy>"}[top]
    if j.tc:
        ach = j.tc / (avg * 1e-3) / 1e12
        roof = {"kernel": kname, "bound": "tensor", "achieved": round(ach, 2), "peak": peak_tc,
                "unit": "TFLOP/s", "frac": round(ach / peak_tc, 4),
                "peak_source": "MEASURED_PEAKS.json bf16_tflops (burst: a ~1-ms launch timed on its own)"}
    elif j.fp32 and j.fp32 / j.bytes > 1.0:
        ach = j.fp32 / (avg * 1e-3) / 1e12
        roof = {"kernel": kname, "bound": "alu", "achieved": round(ach, 3),
                "peak": round(peak_fp32, 2), "unit": "TFLOP/s", "frac": round(ach / peak_fp32, 4),
                "peak_source": "FP32 = 148 SMs x 128 lanes x 2 flop x 1.965 GHz (DESIGN.md §5)"}
    else:
        ach = j.bytes / (avg * 1e-3) / 1e9
        roof = {"kernel": kname, "bound": "hbm", "achieved": round(ach, 1), "peak": peak_hbm,
                "unit": "GB/s", "frac": round(ach / peak_hbm, 4), "peak_source": "MEASURED_PEAKS.json hbm_gbs"}
    roof["avg_launch_ms"] = round(avg, 5)
    roof["launch_time"] = "job span / launches (the launches of a batch overlap)"
    # in the co-run the kernel holds only its share of the SMs (the split): its
    # rate against that share of the peak (the job also grows to every SM once
    # its co-runner drains, so this is a lower bound on the share's use)
    share = (w.n_sms - w.split) if top == w.a.name else w.split
    roof["corun_sms"] = int(share)
    roof["frac_of_share"] = round(roof["frac"] * w.n_sms / max(share, 1), 4)
    # the same kernel solo on every SM (the Slate-sequential schedule): in the
    # co-run it holds only its share of the SMs, so its per-launch rate there
    # is not its roofline position
    solo_q = base["seq_slate"][3] if top == w.a.name else base["seq_slate"][4]
    solo_avg = per_launch(solo_q)
    roof["solo"] = {"avg_launch_ms": round(solo_avg, 5),
                    "achieved": round(roof["achieved"] * avg / solo_avg, 3 if roof["unit"] != "GB/s" else 1),
                    "frac": round(roof["frac"] * avg / solo_avg, 4)}
    if roof["kernel"] == "spmv::spmv_worker":
        # the bound per SM (profiles/r2_spmv_limits.md): the worker's compute
        # goes through the SM's shared-memory SRAM -- 0.25 LSU wavefronts (32 B)
        # per nonzero measured by ncu, plus the bulk copies' 8 B per nonzero
        # written into it -- against 128 B/clk: 3.2 nonzeros per clock, ~55 GB/s
        # of SpMV traffic per SM; on its co-run share the HBM fraction is not
        # its roofline position
        ceil_gbs = 128.0 / 40.0 * 1.965e9 * (147e6 / 16.78e6) / 1e9
        per_sm = roof["achieved"] / max(share, 1)
        roof["per_sm"] = {"achieved_gbs": round(per_sm, 1), "ceiling_gbs": round(ceil_gbs, 1),
                          "frac": round(per_sm / ceil_gbs, 4),
                          "ceiling_source": "shared-memory SRAM: 40 B per nonzero (32 B LSU wavefronts, ncu, + 8 B "
                                            "bulk-copy writes) at 128 B/clk x 1.965 GHz; 8.76 B of SpMV traffic per "
                                            "nonzero (profiles/r2_spmv_limits.md)"}
    roof["traffic"] = None
    ncu_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(ncu_path):
        roof["traffic"] = json.load(open(ncu_path)).get(roof["kernel"])
    return {"steps": steps_out, "med": med, "t_seq": t_seq, "schedules": sched,
            "gain_vs_sequential": round(t_best_seq / mk, 4), "gain_vs_seq_cuda": round(t_seq / mk, 4),
            "gain_vs_slate_sequential": round(base["seq_slate"][0] / mk, 4),
            "best_sequential": {"ms": round(t_best_seq, 3), "solo_ms": {w.a.name: round(solo_a, 3), w.b.name: round(solo_b, 3)},
                                "solo_options_ms": {w.a.name: {k: round(v, 3) for k, v in solo_opts["a"].items()},
                                                    w.b.name: {k: round(v, 3) for k, v in solo_opts["b"].items()}},
                                "stp": {k: round(v[0], 4) for k, v in seq_orders.items()},
                                "antt": {k: round(v[1], 4) for k, v in seq_orders.items()}},
            "stp_vs_sequential": sched["slate_corun"]["stp_vs_sequential"],
            "antt_vs_sequential": sched["slate_corun"]["antt_vs_sequential"],
            "resize_us": {"n": len(resize), "p50": round(statistics.median(resize), 2) if resize else None,
                          "p99": round(float(np.percentile(resize, 99)), 2) if resize else None,
                          "max": round(max(resize), 2) if resize else None,
                          "over_50us": sum(1 for v in resize if v > 50.0), "scope": "every timed step",
                          "topups": sum(q["n_topups"] for q in qa + qb)},
            "split_sms_b": w.split, "arrival_ms": round(w.arrival_ms, 3),
            "utilisation": util, "profiles": {w.a.name: prof_view(pa), w.b.name: prof_view(pb)}, "roofline": roof}


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
    sA, sB = S.Session(None, local), S.Session(None, local)
    sA.set_split_objective("makespan")   # reading Q10, the server's default (made explicit); Q41's ANTT split is the slate_antt schedule
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)   # 256 MB > L2

    # ---- C2, the headline (BASELINE configs[1]); its timed loop is the bench's timed region
    w2 = make_c2(S, dev)
    clocks = {}

    def timed(loop):
        clocks["c"] = Clocks(local)
        barrier(world)
        torch.cuda.synchronize()
        nvtx = bool(os.environ.get("SLATE_NVTX"))   # profiling only: ncu --nvtx --nvtx-include "timed/"
        if nvtx:
            torch.cuda.nvtx.range_push("timed")
        out = loop()
        if nvtx:
            torch.cuda.nvtx.range_pop()
        torch.cuda.synchronize()
        barrier(world)
        clocks["r"] = clocks["c"].stop()
        return out

    r2 = evaluate(w2, S, sA, sB, flush, args.steps, args.warmup, peaks, timed)
    total_ms = sum(s[0] for s in r2["steps"])
    total_ms_max = allmax(world, total_ms)
    value = aggregate(world, args.steps, total_ms_max)
    n_launch = sum(len(s[3]) + len(s[4]) + sum(q["n_topups"] for q in s[3] + s[4]) for s in r2["steps"])

    # ---- e2e: host buffers in, the same co-run through the public API, results out.
    # Every step copies its inputs from pinned host memory and reads its results
    # back; the copies run on a copy stream and overlap the neighbouring steps'
    # kernels (step i+1's inputs go in while step i computes, into a second
    # device set; step i's results come out while step i+1 computes).
    kA, kB = sA.register_kernel(w2.a.kind), sA.register_kernel(w2.b.kind)
    w2b = make_c2(S, dev, pinned=w2.pinned)
    w2b.arrival_ms = w2.arrival_ms
    sets = [w2, w2b]
    cs = torch.cuda.Stream()

    def h2d(w):
        with torch.cuda.stream(cs):
            for k, v in w2.pinned.items():
                w._keep[k].copy_(v, non_blocking=True)
            ev = torch.cuda.Event()
            ev.record(cs)
        return ev

    def d2h(w):
        with torch.cuda.stream(cs):
            for k in w2.out_names:
                w2.out_pinned[k].copy_(w._keep[k], non_blocking=True)
            ev = torch.cuda.Event()
            ev.record(cs)
        return ev

    def e2e_run(n):
        ev_in = h2d(sets[0])
        ev_out = [None, None]
        for i in range(n):
            cur = sets[i % 2]
            ev_in.synchronize()                      # step i's inputs are in (the server's streams do not wait)
            if ev_out[i % 2] is not None:
                ev_out[i % 2].synchronize()          # step i-2's results are out of this set
            submit(sA, kA, cur.a, placement=S.PLACE_AUTO)
            spin_ms(cur.arrival_ms)
            submit(sB, kB, cur.b, placement=S.PLACE_AUTO)
            if i + 1 < n:
                ev_in = h2d(sets[(i + 1) % 2])       # overlaps step i's kernels
            sA.sync(0)
            sB.sync(0)
            ev_out[i % 2] = d2h(cur)                 # overlaps step i+1's kernels
        cs.synchronize()

    flush_l2(flush)
    e2e_run(2)                                       # warm-up
    flush_l2(flush)
    t0 = time.perf_counter()
    e2e_run(args.steps)
    e2e_s = allmax(world, (time.perf_counter() - t0) / args.steps)
    del w2b
    h2d_bytes, d2h_bytes = w2.h2d_bytes, w2.d2h_bytes
    del w2

    # ---- C3 (configs[2]): the tensor-core + HBM pair with a resize mid-run
    c3 = None
    if not args.no_c3:
        w3 = make_c3(S, dev)
        r3 = evaluate(w3, S, sA, sB, flush, max(3, args.steps // 2), args.warmup, peaks)
        c3 = {k: r3[k] for k in ("gain_vs_sequential", "gain_vs_seq_cuda", "gain_vs_slate_sequential",
                                 "best_sequential", "stp_vs_sequential", "antt_vs_sequential", "schedules",
                                 "resize_us", "split_sms_b", "arrival_ms", "utilisation", "profiles", "roofline")}
        c3["config"] = C3
        c3["stp"] = r3["schedules"]["slate_corun"]["stp"]
        c3["antt"] = r3["schedules"]["slate_corun"]["antt"]
        c3["resize_storm"] = resize_storm(S, sA, w3.a, sA.info()["num_sms"])
        del w3

    # ---- C5 (configs[4]): the C2 pair on every GPU, aggregated over the ranks
    med = r2["med"]
    c5 = c5_aggregate(gather(world, {"t_seq_ms": r2["best_sequential"]["ms"], "makespan_ms": med[0],
                                     "stp": r2["schedules"]["slate_corun"]["stp"]}))

    # ---- C4 (configs[3]): four client processes through a slated daemon, on every rank's GPU
    c4 = None
    if not args.no_c4:
        try:
            sys.path.insert(0, os.path.join(ROOT, "tools"))
            import c4_bench
            sA.close()
            sB.close()
            sA = sB = None
            c4 = c4_bench.run(max(3, args.steps // 2), local)
        except Exception as e:   # reported, never fatal for the headline
            c4 = {"error": str(e)[:300]}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        pair_s, sample = oracle_pair_seconds(args.cpu_sample_s)
        cpu = {"value": 1.0 / pair_s, "unit": "pair-jobs/s", "cores": 1, "kind": "oracle", "sample": sample,
               "cpu_model": _cpu_model()}
        try:
            pair_all, cores = oracle_pair_seconds_all_cores(min(10.0, args.cpu_sample_s))
            cpu_all = {"value": 1.0 / pair_all, "unit": "pair-jobs/s", "cores": cores, "kind": "oracle",
                       "sample": "the same oracle with its independent blocks spread over %d worker processes "
                                 "(~%.0f s of wall clock), extrapolated to a pair-job" % (cores, min(10.0, args.cpu_sample_s)),
                       "cpu_model": _cpu_model()}
        except Exception as e:   # context only, never fatal
            cpu_all = {"error": str(e)[:200]}

    line = {
        "metric": METRIC, "value": round(value, 4), "unit": "pair-jobs/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(total_ms_max / args.steps, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": CONFIG,
        "gain_vs_sequential": r2["gain_vs_sequential"], "gain_vs_seq_cuda": r2["gain_vs_seq_cuda"],
        "gain_vs_slate_sequential": r2["gain_vs_slate_sequential"], "best_sequential": r2["best_sequential"],
        "stp": r2["schedules"]["slate_corun"]["stp"], "antt": r2["schedules"]["slate_corun"]["antt"],
        "stp_vs_sequential": r2["stp_vs_sequential"], "antt_vs_sequential": r2["antt_vs_sequential"],
        "split_objective": {"objective": "makespan", "reading": "DESIGN.md Q10/Q41",
                            "alternative": "schedules.slate_antt: ANTT within %.2f of the best makespan" % SPLIT_SLACK},
        "schedules": r2["schedules"], "forced_split_sms_spmv": r2["split_sms_b"], "resize_us": r2["resize_us"],
        "corun_utilisation": r2["utilisation"], "profiles": r2["profiles"], "roofline": r2["roofline"],
        "clocks": clocks.get("r"),
        "e2e": {"value": round(world / e2e_s, 4), "unit": "pair-jobs/s", "h2d_bytes_per_step": h2d_bytes,
                "d2h_bytes_per_step": d2h_bytes},
        "gpu_launches": n_launch,
    }
    if c3:
        line["c3"] = c3
    if c4:
        c4s = gather(world, c4)
        line["c4"] = c4s[0] if world == 1 else {"per_rank": c4s}
    line["c5"] = c5
    if cpu:
        line["cpu_baseline"] = cpu
        line["cpu_baseline_all_cores"] = cpu_all
    if rank == 0:
        print(json.dumps(line), flush=True)
    if sA:
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
