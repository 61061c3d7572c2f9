"""C2 at BASELINE.json's full size, in the launch configuration bench.py times
(-m gpu): the SpMV job (2^20 rows x 16 nnz, banded) and the Black-Scholes job
(2^23 options x 32 scenarios) submitted as slate_launch_n jobs from two
sessions with AUTO placement, so the selector co-runs them, splits the SMs,
re-splits and grows the survivor.  Checked: the outputs equal the original
kernels' bit for bit; sampled blocks equal the fp64 oracle (exact for the
integer-valued SpMV, Q17 for Black-Scholes); the SpMV column-sum invariant
holds exactly over all rows; every launch's counters are exact."""
import numpy as np
import pytest
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import inputs as I
from paper_conf_ipps_allenf019_b200 import slate as S

from gpu_helpers import within

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def test_c2_full_size_corun():
    n_rows, n_opt, P = 1 << 20, 1 << 23, 32
    rp, col, val, x = I.spmv_inputs(n_rows, I.seed_for(2, 0), mode="int")
    Sx, X, T, r = I.bs_inputs(n_opt, I.seed_for(2, 1))
    sig = I.bs_sigmas(P)
    d = {k: torch.from_numpy(v).to(DEV) for k, v in
         {"rp": rp, "col": col, "val": val, "x": x, "S": Sx, "X": X, "T": T, "sig": sig}.items()}
    y = torch.zeros(n_rows, device=DEV)
    call, put = torch.zeros(n_opt, device=DEV), torch.zeros(n_opt, device=DEV)
    torch.cuda.synchronize()
    sp_args, sp_grid = S.spmv_args(d["rp"], d["col"], d["val"], d["x"], y)
    bs_args, bs_grid = S.bs_args(d["S"], d["X"], d["T"], call, put, d["sig"], float(r))
    with S.Session(None, 0) as sA, S.Session(None, 0) as sB:
        kbs, ksp = sA.register_kernel(S.KIND_BLACKSCHOLES), sB.register_kernel(S.KIND_SPMV_CSR)
        # the original kernels: the reference outputs
        sA.sync(sA.launch(kbs, bs_args, bs_grid, mode=S.MODE_STANDALONE))
        sB.sync(sB.launch(ksp, sp_args, sp_grid, mode=S.MODE_STANDALONE))
        torch.cuda.synchronize()
        y_ref, c_ref, p_ref = y.clone(), call.clone(), put.clone()
        # profiles, as bench.py takes them (the selector needs the classes and curves)
        sA.profile(kbs, bs_args, bs_grid, S.PROF_CURVE)
        sB.profile(ksp, sp_args, sp_grid, S.PROF_CURVE)
        y.zero_(), call.zero_(), put.zero_()
        torch.cuda.synchronize()
        ia = sA.launch_n(kbs, bs_args, bs_grid, 4, placement=S.PLACE_AUTO)
        ib = sB.launch_n(ksp, sp_args, sp_grid, 40, placement=S.PLACE_AUTO)
        sA.sync(0)
        sB.sync(0)
        torch.cuda.synchronize()
        for s, ids, grid in ((sA, ia, bs_grid), (sB, ib, sp_grid)):
            B = grid[0] * grid[1] * grid[2]
            for i in ids:
                q = s.query(i)
                ex = OT.expected_counters(B, q["iters"])
                assert q["state"] == 2 and q["blocks_done"] == B and q["tasks_done"] == ex["tasks_done"]
                assert q["next_clamped"] == ex["next_clamped"]
        overlap = max(sA.query(i)["end_ms"] for i in ia) > min(sB.query(i)["start_ms"] for i in ib)
    assert torch.equal(y, y_ref) and torch.equal(call, c_ref) and torch.equal(put, p_ref)
    assert overlap, "the selector did not co-run the pair"
    yg = y.cpu().numpy().astype(np.float64)
    # SpMV: sampled blocks exact against the oracle; the column-sum invariant over every row
    rng = np.random.default_rng(171)
    blocks = sorted(set([0, sp_grid[0] - 1] + list(rng.integers(0, sp_grid[0], 300))))
    ref = OT.spmv_csr(rp, col, val, x, blocks=blocks)
    rows = np.concatenate([np.arange(b * 32, b * 32 + 32) for b in blocks])
    assert np.array_equal(yg[rows], ref[rows])
    colsum = np.bincount(col, weights=val.astype(np.int64), minlength=n_rows).astype(np.int64)
    assert int(yg.sum()) == int((colsum * x.astype(np.int64)).sum())
    # Black-Scholes: sampled blocks within Q17 of the fp64 oracle
    bblocks = sorted(set([0, bs_grid[0] - 1] + list(rng.integers(0, bs_grid[0], 12))))
    cr, pr = OT.blackscholes(Sx, X, T, r, sig, blocks=bblocks)
    idx = np.concatenate([np.arange(b * 1024, b * 1024 + 1024) for b in bblocks])
    scale = Sx[idx].astype(np.float64)
    assert within(call.cpu().numpy()[idx], cr[idx], scale)[0]
    assert within(put.cpu().numpy()[idx], pr[idx], scale)[0]
