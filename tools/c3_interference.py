"""Diagnostic: where does the bf16 GEMM lose time next to the STREAM copy?
The GEMM (8192^3) runs on SMs [0, 83] with, on the other SMs, nothing / the
4 GiB copy / an L2-resident copy (no DRAM) / the 4 GiB copy on fewer SMs.
Device times from the server's events; prints one line per case."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

dev = "cuda:0"
sA, sB = S.Session(None, 0), S.Session(None, 0)
g = torch.Generator(device=dev)
g.manual_seed(1)
A = (torch.rand(8192, 8192, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
B = (torch.rand(8192, 8192, device=dev, generator=g) * 2 - 1).to(torch.bfloat16)
C = torch.zeros(8192, 8192, device=dev)
big_b, big_a = torch.rand(1 << 30, device=dev), torch.empty(1 << 30, device=dev)
small_b, small_a = torch.rand(1 << 22, device=dev), torch.empty(1 << 22, device=dev)   # 16 MiB each
torch.cuda.synchronize()
gk = sA.register_kernel(S.KIND_GEMM_BF16)
ck = sB.register_kernel(S.KIND_COPY)
gargs, ggrid = S.gemm_args(A.view(torch.int16), B.view(torch.int16), C)
big, bgrid = S.copy_args(big_a, big_b)
small, sgrid = S.copy_args(small_a, small_b)


def dur(s, i):
    q = s.query(i)
    return q["end_ms"] - q["start_ms"]


def case(name, copy=None, crange=None, reps=1, gemm_sms=(0, 83)):
    ts = []
    for _ in range(3):
        ids = []
        if copy is not None:
            args, grid = copy
            ids = [sB.launch(ck, args, grid, placement=S.PLACE_CORUN, sm=crange) for _ in range(reps)]
        gi = sA.launch(gk, gargs, ggrid, placement=S.PLACE_CORUN, sm=gemm_sms)
        sA.sync(0)
        sB.sync(0)
        c_ms = (sB.query(ids[-1])["end_ms"] - sB.query(ids[0])["start_ms"]) if ids else 0.0
        ts.append((dur(sA, gi), c_ms, sA.query(gi)["workers_started"], sA.query(gi)["n_topups"]))
    ts.sort()
    gm, cm, ws, tu = ts[1]
    print("%-38s gemm %.3f ms (%.0f TFLOP/s)  copy span %.3f ms  gemm workers %d topups %d"
          % (name, gm, 2 * 8192 ** 3 / gm / 1e9, cm, ws, tu), flush=True)


case("gemm alone on 148", gemm_sms=(0, 147))
case("gemm alone on 84")
case("gemm 84 + copy 4GiB on 64", (big, bgrid), (84, 147))
case("gemm 84 + copy 4GiB on 48", (big, bgrid), (100, 147))
case("gemm 84 + copy 4GiB on 32", (big, bgrid), (116, 147))
case("gemm 84 + copy 4GiB on 16", (big, bgrid), (132, 147))
case("gemm 84 + L2-resident copy on 64", (small, sgrid), (84, 147), reps=400)
sA.close()
sB.close()
