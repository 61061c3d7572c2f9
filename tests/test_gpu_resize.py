"""GPU tests of dynamic resizing (-m gpu): random resize storms from the host
while a launch runs must keep every original block executed exactly once
(coverage log all ones, exact counters) and the output bit-identical to the
standalone launch (P:L127 progress carried in slateIdx; P:L243-245 exit
conditions); shrink and grow latencies are observed."""
import random
import time

import numpy as np
import pytest
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import slate as S

from gpu_helpers import make_bs, make_copy, make_gemm, make_spmv, make_stencil, make_triad, within

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sess():
    s = S.Session(None, 0)
    yield s
    s.close()


def _storm(sess, t, iters, n_resizes, seed, gap_us):
    n = sess.info()["num_sms"]
    k_std = sess.register_kernel(t.kind)
    t.zero_outputs()
    torch.cuda.synchronize()
    sess.sync(sess.launch(k_std, t.args, t.grid, mode=S.MODE_STANDALONE))
    ref = t.snapshot()
    k = sess.register_kernel(t.kind, iters=iters, flags=S.KFLAG_COVERAGE)
    t.zero_outputs()
    B = int(np.prod(t.grid))
    cov = torch.zeros(B, dtype=torch.int32, device="cuda:0")
    torch.cuda.synchronize()   # the server's streams do not wait for torch's stream
    rng = random.Random(seed)
    lid = sess.launch(k, t.args, t.grid, placement=S.PLACE_CORUN, sm=(0, n - 1), coverage=cov)
    done = 0
    for _ in range(n_resizes):
        lo = rng.randrange(0, n)
        hi = rng.randrange(lo, n)
        st = sess.resize(lid, lo, hi)
        done += 1
        if st == S.DONE:
            break
        t0 = time.perf_counter()
        while (time.perf_counter() - t0) * 1e6 < gap_us:
            pass
    sess.sync(lid)
    torch.cuda.synchronize()
    q = sess.query(lid)
    ex = OT.expected_counters(B, iters)
    assert q["coverage_ok"] == 1 and np.array_equal(cov.cpu().numpy(), ex["coverage"].astype(np.int32))
    assert (q["blocks_done"], q["tasks_done"], q["next_clamped"]) == \
        (ex["blocks_done"], ex["tasks_done"], ex["next_clamped"])
    for a, b in zip(t.snapshot(), ref):
        assert torch.equal(a, b)
    return q, done


def test_resize_storm_bs(sess):
    t = make_bs(1 << 21, 201, n_scen=64)
    q, done = _storm(sess, t, 1, 30, 1, 100)
    assert done >= 3 and q["n_resizes"] >= 2
    # the launch really ran on sub-ranges: a sampled block matches the oracle
    S_, X_, T_ = (x.cpu().numpy() for x in t._keep[:3])
    sig = t._keep[3].cpu().numpy()
    blocks = [0, 777, int(np.prod(t.grid)) - 1]
    c_ref, p_ref = OT.blackscholes(S_, X_, T_, 0.02, sig, blocks=blocks)
    out = t.snapshot()[0].cpu().numpy()
    idx = np.concatenate([np.arange(b * 1024, min((b + 1) * 1024, len(S_))) for b in blocks])
    assert within(out[idx], c_ref[idx], S_[idx].astype(np.float64))[0]


def test_resize_storm_cta_tenant(sess):
    t = make_stencil(8192, 8192, 202)
    q, done = _storm(sess, t, 10, 30, 2, 20)
    assert done >= 3


def test_resize_storm_spmv_warp_specialised(sess):
    """The SpMV worker's task warp fetches up to two tasks ahead of its compute
    warps; a CTA that leaves the range still finishes what it fetched, so
    coverage stays exactly-once under a storm."""
    t = make_spmv(1 << 22, 207)
    q, done = _storm(sess, t, 1, 30, 4, 20)
    assert done >= 3


def test_resize_storm_iters1_copy(sess):
    t = make_copy(1 << 30, 203)
    q, done = _storm(sess, t, 1, 40, 3, 10)
    assert done >= 4          # the 8-GiB copy lasts ~1.5 ms: a handful of resizes land while it runs
    assert len(q["resize_us"]) >= 3, q


def test_shrink_then_grow_latency(sess):
    n = sess.info()["num_sms"]
    t = make_triad(1 << 28, 204)
    k = sess.register_kernel(t.kind, iters=1)
    lid = sess.launch(k, t.args, t.grid, placement=S.PLACE_CORUN, sm=(0, n - 1))
    time.sleep(0.0002)
    sess.resize(lid, 0, n // 2 - 1)      # shrink: workers on the upper half retire
    time.sleep(0.0002)
    sess.resize(lid, 0, n - 1)           # grow: a top-up launch adds workers
    sess.sync(lid)
    q = sess.query(lid)
    assert q["blocks_done"] == q["total_blocks"]
    assert q["n_topups"] >= 1
    lat = q["resize_us"]
    assert len(lat) == 2 and all(0 < v < 5000 for v in lat), lat


def test_shrink_latency_inside_a_batch(sess):
    """Resize accounting in a batched job (reading Q50 era fix): the finished
    members of a batch stay issued until the batch's end event, and a shrink
    used to be 'resolved' by the end stamp of one that had finished before the
    resize (0 us).  Shrink the queue in the middle of a 200-launch triad job:
    the shrink is timed from the call to the out-of-range workers' retirement
    -- above 0, and well under a launch of the job."""
    n = sess.info()["num_sms"]
    t = make_triad(1 << 24, 208)
    k = sess.register_kernel(t.kind)
    ids = sess.launch_n(k, t.args, t.grid, 200, placement=S.PLACE_CORUN, sm=(0, n - 1))
    time.sleep(0.003)                     # well into the job: many members already finished
    st = sess.resize(ids[0], 0, n // 2 - 1)
    sess.sync(0)
    lats = [v for i in ids for kd, v in zip(sess.query(i)["resize_kind"], sess.query(i)["resize_us"]) if kd == "shrink"]
    if st == S.DONE or not lats:
        pytest.skip("the job ended before the resize landed")
    assert all(0 < v < 200 for v in lats), lats


def test_resize_storm_gemm_abandons_tiles(sess):
    """tcgen05 GEMM under a resize storm: workers leaving the range abandon their
    tile mid-K and give it back (Q28); every tile is still stored exactly once,
    bit-identical to the standalone launch (integer inputs: exact vs the oracle
    on sampled tiles)."""
    t = make_gemm(4096, 4096, 8192, 205, "int")
    q, done = _storm(sess, t, 1, 40, 4, 30)
    assert done >= 5
    ok, err = t.check(t.snapshot(), rows=[(0, 0), (15, 31), (7, 3)])
    assert ok


def test_resize_storm_gemm_ragged(sess):
    """The same storm on a GEMM ragged in m, n and k (partial last tile row,
    column and K slice: zero-filled TMA loads, clipped TMA stores): abandoned
    and retaken tiles still store every element exactly once, exact against the
    oracle on sampled tiles including the ragged corner."""
    m, n, k = 2048 + 77, 2048 + 132, 4096 + 24
    t = make_gemm(m, n, k, 207, "int")
    q, done = _storm(sess, t, 1, 30, 5, 30)
    assert done >= 5
    last_x, last_y = (n - 1) // 128, (m - 1) // 128
    ok, err = t.check(t.snapshot(), rows=[(0, 0), (last_x, last_y), (last_x, 3), (5, last_y)])
    assert ok


def test_gemm_shrink_latency(sess):
    n = sess.info()["num_sms"]
    t = make_gemm(8192, 8192, 8192, 206)
    k = sess.register_kernel(t.kind)
    lats = []
    for _ in range(3):
        lid = sess.launch(k, t.args, t.grid, placement=S.PLACE_CORUN, sm=(0, n - 1))
        time.sleep(0.0003)
        sess.resize(lid, 0, n // 2 - 1)
        time.sleep(0.0002)
        sess.resize(lid, 0, n - 1)
        sess.sync(lid)
        q = sess.query(lid)
        assert q["blocks_done"] == q["total_blocks"]
        lats += q["resize_us"]
    assert lats and max(lats) < 200, lats


def test_dependent_chain_with_topups(sess):
    """Stream order under grows: a chain of triads where each launch reads the
    previous one's output (ping-pong x <- x + 1), all queued at once on a
    quarter of the SMs, then a storm of grows and shrinks.  A grow tops up the
    RUNNING launch while the rest of the chain is queued behind it; its last
    main CTA waits for the top-up's blocks before the kernel ends, so the next
    launch reads finished data: the result must be exactly x0 + K."""
    n_sms = sess.info()["num_sms"]
    n, K = 1 << 25, 60
    x0 = torch.arange(n, dtype=torch.float32, device="cuda:0") % 1000
    bufs = [x0.clone(), torch.zeros(n, device="cuda:0")]
    ones = torch.ones(n, device="cuda:0")
    torch.cuda.synchronize()
    k = sess.register_kernel(S.KIND_TRIAD, iters=2)
    ids = []
    for i in range(K):
        args, grid = S.triad_args(bufs[(i + 1) % 2], bufs[i % 2], ones, 1.0)
        ids.append(sess.launch(k, args, grid, placement=S.PLACE_CORUN, sm=(0, n_sms // 4 - 1)))
    rng = random.Random(205)
    for i in range(4000):
        lo, hi = (0, n_sms - 1) if i % 2 == 0 else (0, rng.randrange(n_sms // 8, n_sms // 2))
        if sess.resize(ids[-1], lo, hi) == S.DONE:
            break
        time.sleep(0.00015)
    sess.sync(0)
    torch.cuda.synchronize()
    topups = sum(sess.query(i)["n_topups"] for i in ids)
    for i in ids:
        q = sess.query(i)
        assert q["blocks_done"] == q["total_blocks"] and q["tasks_done"] == -(-q["total_blocks"] // 2)
    assert torch.equal(bufs[K % 2], x0 + K)
    assert topups >= 1, "no grow landed on a running launch"
