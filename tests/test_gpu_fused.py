"""NEXT-1, the fused co-run worker (-m gpu): two launches from two sessions run
as ONE persistent kernel whose CTAs pick a tenant at every task boundary from
the two queues' resize words (P:L123-127 shrink on arrival / "seamlessly
claims" on completion; P:L237-245 exit conditions).  Checked against the
oracle (config C1's pair, integer inputs: exact), bit for bit against the
original kernels under random resize storms, with exactly-once coverage, the
exact counters, the rank log (every task ran on a rank inside the range in
force) and no top-up launch."""
import random
import time

import numpy as np
import pytest
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import slate as S

from gpu_helpers import make_bs, make_sgemm, make_stencil, make_transpose, make_triad

pytestmark = pytest.mark.gpu
FLAGS = S.KFLAG_COVERAGE | S.KFLAG_RANKLOG


def _log(cov, B):
    c = cov.cpu().numpy().view(np.uint32)
    counts, log = c[:B], c[B:]
    return counts, log & 0xff, (log >> 8) & 0xff, (log >> 16) & 0xff, (log >> 24) & 0x81


def _fused(ta, tb, sm_b, iters_a=0, iters_b=0, storm=None):
    sa, sb = S.Session(None, 0), S.Session(None, 0)
    try:
        n = sa.info()["num_sms"]
        ka = sa.register_kernel(ta.kind, iters=iters_a, flags=FLAGS)
        kb = sb.register_kernel(tb.kind, iters=iters_b, flags=FLAGS)
        Ba, Bb = int(np.prod(ta.grid)), int(np.prod(tb.grid))
        ca = torch.zeros(2 * Ba, dtype=torch.int32, device="cuda:0")
        cb = torch.zeros(2 * Bb, dtype=torch.int32, device="cuda:0")
        ta.zero_outputs()
        tb.zero_outputs()
        torch.cuda.synchronize()
        la, lb = S.launch_fused(sa, ka, ta.args, ta.grid, sb, kb, tb.args, tb.grid, sm_b, ca, cb)
        requested = {(0, n - sm_b - 1), (n - sm_b, n - 1), (0, n - 1)}
        if storm:
            rng = random.Random(storm)
            for _ in range(30):
                k = rng.randrange(8, n - 8)
                requested |= {(0, k - 1), (k, n - 1)}
                ra, rb = sa.resize(la, 0, k - 1), sb.resize(lb, k, n - 1)
                if ra == S.DONE or rb == S.DONE:
                    break
                time.sleep(100e-6)
        sa.sync(la)
        sb.sync(lb)
        torch.cuda.synchronize()
        return sa.query(la), sb.query(lb), ca, cb, Ba, Bb, requested, n
    finally:
        sa.close()
        sb.close()


def _check_log(cov, B, requested, iters):
    counts, rank, lo, hi, flags = _log(cov, B)
    ex = OT.expected_counters(B, iters)
    assert np.array_equal(counts, ex["coverage"])                       # every block exactly once
    assert np.all(flags == 0x80)                                         # logged, never outside its range
    assert np.all((rank >= lo) & (rank <= hi))
    assert set(zip(lo.tolist(), hi.tolist())) <= requested
    return rank, lo, hi


def test_fused_c1_pair_matches_the_oracle():
    """Config C1 (triad + naive SGEMM) as one fused kernel: exact on integer inputs."""
    ta = make_triad(1 << 20, 501, "int")
    tb = make_sgemm(256, 256, 256, 502, "int")
    qa, qb, ca, cb, Ba, Bb, req, n = _fused(ta, tb, 40, 10, 1)
    ok_a, _ = ta.check(ta.snapshot())
    ok_b, err_b = tb.check(tb.snapshot())
    assert ok_a and ok_b, err_b
    for q, B, it in ((qa, Ba, 10), (qb, Bb, 1)):
        ex = OT.expected_counters(B, it)
        assert (q["blocks_done"], q["tasks_done"], q["next_clamped"]) == \
            (ex["blocks_done"], ex["tasks_done"], ex["next_clamped"])
        assert q["coverage_ok"] == 1 and q["n_topups"] == 0
    ra, la_, ha = _check_log(ca, Ba, req, 10)
    rb, lb_, hb = _check_log(cb, Bb, req, 1)
    # while both ran, their rank sets were disjoint (entries under the initial ranges)
    own_a = set(ra[(la_ == 0) & (ha == n - 41)].tolist())
    own_b = set(rb[(lb_ == n - 40) & (hb == n - 1)].tolist())
    assert own_a and own_b and not (own_a & own_b)


@pytest.mark.parametrize("pair", ["bs+stencil", "bs+stencil_ragged", "transpose+sgemm"])
def test_fused_resize_storm_exactly_once(pair):
    if pair == "bs+stencil":
        ta, tb, ia, ib = make_bs(1 << 21, 503, n_scen=64), make_stencil(8192, 4096, 504), 1, 4
    elif pair == "bs+stencil_ragged":
        # the fused stencil body pairs x-neighbouring blocks: 33 blocks a row band
        # (the last one ragged, w % 128 = 4) and 3 blocks a task, so pairs start at
        # both parities and tasks straddle row bands; h % 8 = 1
        ta, tb, ia, ib = make_bs(1 << 20, 509, n_scen=32), make_stencil(1001, 4100, 510), 1, 3
    else:
        ta, tb, ia, ib = make_transpose(4096, 4096, 505), make_sgemm(512, 512, 512, 506), 4, 2
    refs = []
    s = S.Session(None, 0)
    for t in (ta, tb):
        k = s.register_kernel(t.kind)
        t.zero_outputs()
        s.sync(s.launch(k, t.args, t.grid, mode=S.MODE_STANDALONE))
        torch.cuda.synchronize()
        refs.append(t.snapshot())
    s.close()
    qa, qb, ca, cb, Ba, Bb, req, n = _fused(ta, tb, 60, ia, ib, storm=11)
    for t, ref in zip((ta, tb), refs):
        for x, y in zip(t.snapshot(), ref):
            assert torch.equal(x, y), pair
    if pair == "bs+stencil_ragged":
        ok, err = tb.check(tb.snapshot())
        assert ok, err
    _check_log(ca, Ba, req, ia)
    _check_log(cb, Bb, req, ib)
    for q, B, it in ((qa, Ba, ia), (qb, Bb, ib)):
        ex = OT.expected_counters(B, it)
        assert (q["blocks_done"], q["tasks_done"]) == (ex["blocks_done"], ex["tasks_done"])
        assert q["n_topups"] == 0 and q["n_resizes"] >= 1


def test_fused_grow_on_drain_claims_the_partners_sms():
    """when the short tenant drains, the long one runs on its SMs at
    once -- the same kernel, no launch; its log shows tasks under the whole-chip
    range on the short tenant's former ranks."""
    ta = make_triad(1 << 18, 507)
    tb = make_bs(1 << 21, 508, n_scen=32)
    qa, qb, ca, cb, Ba, Bb, req, n = _fused(ta, tb, n_b := 74, 10, 1)
    rb, lb_, hb = _check_log(cb, Bb, req, 1)
    grown = (lb_ == 0) & (hb == n - 1)
    assert grown.any()
    assert set(rb[grown].tolist()) & set(range(0, n - n_b))             # on A's former ranks
    assert qb["n_topups"] == 0
    ok_a, _ = ta.check(ta.snapshot())
    ok_b, err_b = tb.check(tb.snapshot())
    assert ok_a and ok_b, err_b
