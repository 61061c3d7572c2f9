"""A client process for the slated tests (config C4 shape): attaches to a server
endpoint, shares its buffers by CUDA IPC, launches one tenant with AUTO
placement, checks the result against the oracle (and, with --exact, bit for bit
against the same tenant's standalone launch run through the same server).

    python tests/ipc_client.py ENDPOINT KIND SEED [--reps R] [--hang]
"""
import os
import sys
import time

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
sys.path.insert(0, HERE)

import torch  # noqa: E402

from gpu_helpers import make_bs, make_gemm, make_spmv, make_stencil, make_triad  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

MAKERS = {
    "triad": lambda seed: make_triad(1024 * 300 + 7, seed),
    "spmv": lambda seed: make_spmv(32 * 2000 + 5, seed, band=512),
    "stencil": lambda seed: make_stencil(8 * 200 + 3, 32 * 40 + 1, seed),
    "gemm": lambda seed: make_gemm(512, 512, 1024, seed, "int"),
    "bs": lambda seed: make_bs(1024 * 64, seed, n_scen=4),
}


def main():
    endpoint, kind, seed = sys.argv[1], sys.argv[2], int(sys.argv[3])
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 3
    t = MAKERS[kind](seed)
    s = S.Session(endpoint)
    info = s.info()
    assert info["server_pid"] != os.getpid() and info["server_pid"] > 0, info
    for ten in list(t.outputs) + list(t._keep):
        s.share_buffer(ten)
    k_std = s.register_kernel(t.kind)
    s.sync(s.launch(k_std, t.args, t.grid, mode=S.MODE_STANDALONE))
    ref = t.snapshot()
    if "--hang" in sys.argv:      # die with launches in flight (the server must clean up)
        k = s.register_kernel(t.kind)
        for _ in range(50):
            s.launch(k, t.args, t.grid)
        print("READY", flush=True)
        time.sleep(60)
        return
    k = s.register_kernel(t.kind, flags=S.KFLAG_COVERAGE)
    for r in range(reps):
        t.zero_outputs()
        cov = torch.zeros(int(t.grid[0] * t.grid[1] * t.grid[2]), dtype=torch.int32, device="cuda:0")
        torch.cuda.synchronize()
        s.share_buffer(cov)
        lid = s.launch(k, t.args, t.grid, placement=S.PLACE_AUTO, coverage=cov)
        s.sync(lid)
        q = s.query(lid)
        assert q["coverage_ok"] == 1 and q["blocks_done"] == q["total_blocks"], q
        out = t.snapshot()
        assert all(torch.equal(a, b) for a, b in zip(out, ref)), "slate != standalone"
    ok, err = t.check(out)
    assert ok, err
    s.close()
    print("OK", kind, flush=True)


if __name__ == "__main__":
    main()
