"""ncu target (SURVEY §8(d) cross-check): ONE co-run pair-job of C2 (SpMV +
Black-Scholes P=32) or C3 (bf16 GEMM 8192^3 + copy 4 GiB) under Slate AUTO,
bracketed by cudaProfilerStart/Stop, after warm-up jobs.  Run it under

    ncu --replay-mode app-range --profile-from-start off --metrics ... \\
        python tools/ncu_corun.py c2 [SPLIT]

so the counters cover the co-run as it runs (both tenants concurrently, the
split, shrink on arrival, grow on completion) -- kernel replay would
serialise it.  The co-run is the bench's `slate_forced` schedule at the split
the selector takes in the bench (68 SMs for the second tenant in C2 and C3):
under ncu the host-side selector sees perturbed solo profiles and may not
co-run at all, so the split is fixed here.  Application replay reruns the whole script once per
metric pass; each pass's co-run is a fresh run of the same schedule."""
import sys

import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
split = int(sys.argv[2]) if len(sys.argv) > 2 else 68
dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
w = {"c2": bench.make_c2, "c3": bench.make_c3}[cfg](S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
w.split = split
for _ in range(2):
    bench.run_schedule("slate_forced", w, sA, sB, kA, kB, S)
torch.cuda.synchronize()
torch.cuda.profiler.start()
mk, ta, tb = bench.run_schedule("slate_forced", w, sA, sB, kA, kB, S)[:3]
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("corun %s split %d makespan %.3f ms (A %.3f, B %.3f)" % (cfg, split, mk, ta, tb), flush=True)
sA.close()
sB.close()
