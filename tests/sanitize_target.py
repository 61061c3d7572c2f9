"""Tiny launches of every worker for compute-sanitizer (tests/test_gpu_sanitizer.py).

    compute-sanitizer --tool memcheck|racecheck|synccheck python tests/sanitize_target.py [GROUP]

Every tenant kind's slate worker -- the generic worker (triad, copy with its
bulk-copy ring, naive SGEMM, Black-Scholes in both variants, stencil, the Tab II
apps), the warp-specialised SpMV worker, the tcgen05 GEMM CTA pair and a
runtime-compiled user kernel -- runs once on a sub-range of the SMs with a
resize in flight, once on the whole chip, and once as the original kernel;
outputs are checked against the oracle so a run that is clean but wrong
fails too.  Sizes are a few blocks per worker: sanitizer runs are ~100x slower.
"""
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
sys.path.insert(0, HERE)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gpu_helpers as G  # noqa: E402
from paper_conf_ipps_allenf019_b200 import slate as S  # noqa: E402

GROUPS = {
    "generic": [lambda: G.make_triad(1024 * 40 + 5, 901, "int"), lambda: G.make_copy(4096 * 24 + 3, 902),
                lambda: G.make_sgemm(48, 40, 32, 903, "int"), lambda: G.make_bs(1024 * 6 + 3, 904, n_scen=2),
                lambda: G.make_bs(1024 * 3, 905, n_scen=33), lambda: G.make_stencil(8 * 5 + 1, 32 * 3 + 5, 906, "int")],
    "apps": [lambda: G.make_transpose(70, 45, 907), lambda: G.make_qrng(3000, 2, 908),
             lambda: G.make_sgemm_tiled(40, 70, 33, 909, "int"), lambda: G.make_gauss_fan1(100, 3, 910),
             lambda: G.make_gauss_fan2(100, 3, 911)],
    "spmv": [lambda: G.make_spmv(32 * 90 + 7, 912, "int", band=256)],
    "gemm": [lambda: G.make_gemm(512, 512, 256, 913, "int")],
}


def run(s, t, n_sms):
    k_std = s.register_kernel(t.kind)
    t.zero_outputs()
    s.sync(s.launch(k_std, t.args, t.grid, mode=S.MODE_STANDALONE))
    torch.cuda.synchronize()
    ok, err = t.check(t.snapshot())
    assert ok, ("standalone", t.kind, err)
    iters = 2 if t.kind != S.KIND_GEMM_BF16 else 1
    k = s.register_kernel(t.kind, iters=iters, flags=S.KFLAG_COVERAGE | S.KFLAG_RANKLOG)
    for sm, resize in (((2, 2 + n_sms // 4), (n_sms // 2, n_sms - 1)), ((0, n_sms - 1), None)):
        t.zero_outputs()
        B = int(np.prod(t.grid))
        cov = torch.zeros(2 * B, dtype=torch.int32, device="cuda:0")
        torch.cuda.synchronize()
        lid = s.launch(k, t.args, t.grid, placement=S.PLACE_CORUN, sm=sm, coverage=cov)
        if resize:
            s.resize(lid, *resize)
        s.sync(lid)
        torch.cuda.synchronize()
        q = s.query(lid)
        assert q["coverage_ok"] == 1 and q["blocks_done"] == B, (t.kind, q)
        ok, err = t.check(t.snapshot())
        assert ok, ("slate", t.kind, sm, err)


def run_user(s, n_sms):
    from oracle import tenants as OT
    from test_user_kernels import PROBE3D_SRC, Args3D
    shape, block = (5, 9, 21), (8, 4, 2)
    grid = OT.probe3d_grid(shape, block)
    x = np.arange(np.prod(shape), dtype=np.float32).reshape(shape) % 97
    xd, yd = torch.from_numpy(x).cuda(), torch.zeros(shape, device="cuda:0")
    torch.cuda.synchronize()
    k = s.register_source(PROBE3D_SRC, "probe3d", Args3D, block=block, iters=3)
    s.sync(s.launch(k, Args3D(xd.data_ptr(), yd.data_ptr(), shape[2], shape[1], shape[0]), grid,
                    placement=S.PLACE_CORUN, sm=(1, n_sms // 3)))
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().numpy().astype(np.float64), OT.probe3d(x, block))


def run_fused(s, n_sms):
    """NEXT-1: a fused pair (triad + naive SGEMM, integer inputs) with a resize in flight."""
    sb = S.Session(None, 0)
    try:
        ta, tb = G.make_triad(1024 * 30 + 5, 914, "int"), G.make_sgemm(64, 48, 40, 915, "int")
        ka = s.register_kernel(ta.kind, iters=3, flags=S.KFLAG_COVERAGE | S.KFLAG_RANKLOG)
        kb = sb.register_kernel(tb.kind, iters=2, flags=S.KFLAG_COVERAGE | S.KFLAG_RANKLOG)
        Ba, Bb = int(np.prod(ta.grid)), int(np.prod(tb.grid))
        ca = torch.zeros(2 * Ba, dtype=torch.int32, device="cuda:0")
        cb = torch.zeros(2 * Bb, dtype=torch.int32, device="cuda:0")
        ta.zero_outputs()
        tb.zero_outputs()
        la, lb = S.launch_fused(s, ka, ta.args, ta.grid, sb, kb, tb.args, tb.grid, n_sms // 3, ca, cb)
        s.resize(la, 0, n_sms // 2 - 1)
        sb.resize(lb, n_sms // 2, n_sms - 1)
        s.sync(la)
        sb.sync(lb)
        torch.cuda.synchronize()
        assert ta.check(ta.snapshot())[0] and tb.check(tb.snapshot())[0]
        assert s.query(la)["coverage_ok"] == 1 and sb.query(lb)["coverage_ok"] == 1
    finally:
        sb.close()


def main():
    import atexit
    import faulthandler
    if os.environ.get("SLATE_EXIT_TRACE"):
        atexit.register(lambda: print("PY-ATEXIT", flush=True))
    groups = sys.argv[1:] or list(GROUPS) + ["user", "fused"]
    faulthandler.dump_traceback_later(float(os.environ.get("SANITIZE_DUMP_S", "600")), exit=True)
    with S.Session(None, 0) as s:
        n = s.info()["num_sms"]
        for g in groups:
            if g == "user":
                run_user(s, n)
            elif g == "fused":
                run_fused(s, n)
            else:
                for mk in GROUPS[g]:
                    run(s, mk(), n)
            print("SANITIZE-OK", g, flush=True)
    print("SANITIZE-CLOSED", flush=True)
    # Leave without the interpreter's and the CUDA runtimes' teardown: under
    # compute-sanitizer about one process exit in ten hung there (after every
    # check passed, every session closed, the server threads joined and all of
    # its streams idle -- tools/san_exit_probe.sh); with os._exit 0 hangs in 30
    # runs, and the tool still prints its summary.  SANITIZE_FAST_EXIT=0 keeps
    # the normal exit.
    if os.environ.get("SANITIZE_FAST_EXIT", "1") != "0":
        torch.cuda.synchronize()
        sys.stdout.flush()
        sys.stderr.flush()
        os._exit(0)


if __name__ == "__main__":
    main()
