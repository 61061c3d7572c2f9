"""Development probe: one C2 pair-job under Slate AUTO (the bench's "slate"
schedule) with every launch's SM range and times, to see the scheduler's
decisions (run with SLATE_DEBUG=1 for the server's own log).

    python tools/c2_timeline.py [antt|makespan]"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

obj = sys.argv[1] if len(sys.argv) > 1 else "antt"
dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
sA.set_split_objective(obj, bench.SPLIT_SLACK)
w = bench.make_c2(S, dev)
kA, kB = sA.register_kernel(w.a.kind), sA.register_kernel(w.b.kind)
pa = sA.profile(kA, w.a.args, w.a.grid, S.PROF_CURVE)
pb = sA.profile(kB, w.b.args, w.b.grid, S.PROF_CURVE)
w.n_sms = sA.info()["num_sms"]
w.split = 0
w.arrival_ms = w.arrival_frac * pa["solo_ms"] * w.a.reps
print("profiles", json.dumps({"a": [pa["category_name"], pa["solo_ms"]], "b": [pb["category_name"], pb["solo_ms"]]}))
flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
clk = bench.Clocks(0) if os.environ.get("TL_CLOCKS") else None   # the bench's NVML sampler, as in its timed region
if os.environ.get("TL_NVML_ONLY"):   # diagnostics: one NVML call kind every 10 ms in a thread ("clock" or "reasons")
    import threading
    import pynvml as N
    N.nvmlInit()
    h = N.nvmlDeviceGetHandleByIndex(0)
    which = os.environ["TL_NVML_ONLY"]

    def _poll():
        while True:
            if which == "clock":
                N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
            else:
                N.nvmlDeviceGetCurrentClocksEventReasons(h)
            import time as _t
            _t.sleep(0.01)
    threading.Thread(target=_poll, daemon=True).start()
REPS = int(os.environ.get("TL_REPS", "3"))
for rep in range(REPS):
    bench.flush_l2(flush)
    mk, ta, tb, qa, qb, ja, jb = bench.run_schedule("slate", w, sA, sB, kA, kB, S)
    t0 = min(min(q["start_ms"] for q in qa), min(q["start_ms"] for q in qb))
    rz = [(k, round(v, 1)) for q in qa + qb for k, v in zip(q["resize_kind"], q["resize_us"])]
    print("rep %d makespan %.3f ms  turnaround A %.3f  B %.3f  resizes %s" % (rep, mk, ta, tb, rz))
    if rep < REPS - 1:
        continue
    for name, qs in (("A", qa), ("B", qb)):
        last = None
        for i, q in enumerate(qs):
            key = (q["sm_lo"], q["sm_hi"], q["n_resizes"], q["n_topups"])
            if key != last or i == len(qs) - 1:
                print("  %s[%3d] %8.3f .. %8.3f  sm %3d-%3d  resizes %d topups %d %s" %
                      (name, i, q["start_ms"] - t0, q["end_ms"] - t0, q["sm_lo"], q["sm_hi"], q["n_resizes"],
                       q["n_topups"], list(zip(q["resize_kind"], [round(v, 1) for v in q["resize_us"]]))))
                last = key
if clk:
    print("clocks", clk.stop())
