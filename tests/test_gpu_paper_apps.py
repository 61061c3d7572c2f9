"""GPU parity of the paper's Gaussian elimination (GS, Tab II) as a whole job
(-m gpu): n-1 steps, each a Fan1 and a Fan2 launch through the C ABI on one
session (FIFO), against the oracle's elimination and against the same
job run as standalone kernels.

Integer systems (a = L U with small integer factors) are exact in fp32, so the
slate job must reproduce the oracle bit for bit.  On Rodinia's SPD matrix the
fp32 elimination is compared with the fp64 oracle under the standard forward
error bound of Gaussian elimination: |g - o| <= c n u max|a| with u = 2^-24
(c = 4, Q36); the slate job equals the standalone job bit for bit
(the same fmaf sequence per element)."""
import numpy as np
import pytest
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import inputs as I
from paper_conf_ipps_allenf019_b200 import slate as S

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


@pytest.fixture(scope="module")
def sess():
    s = S.Session(None, 0)
    yield s
    s.close()


def _eliminate(sess, a0, b0, mode, iters=0, placement=S.PLACE_AUTO, sm=None, many=False):
    n = a0.shape[0]
    a = torch.from_numpy(a0).to(DEV)
    b = torch.from_numpy(b0).to(DEV)
    m = torch.zeros(n, n, device=DEV)
    torch.cuda.synchronize()
    k1 = sess.register_kernel(S.KIND_GAUSS_FAN1, iters=iters)
    k2 = sess.register_kernel(S.KIND_GAUSS_FAN2, iters=iters)
    ids, items = [], []
    for t in range(n - 1):
        items.append((k1,) + S.gauss_fan1_args(a, b, m, t))
        items.append((k2,) + S.gauss_fan2_args(a, b, m, t))
    if many:    # one slate_launch_many call: one batch (no events between kernels, PDL)
        ids = sess.launch_many(items, placement=placement, sm=sm, mode=mode)
    else:
        ids = [sess.launch(k, args, grid, placement=placement, sm=sm, mode=mode) for k, args, grid in items]
    sess.sync(0)
    torch.cuda.synchronize()
    for i in ids[-4:]:
        q = sess.query(i)
        assert q["state"] == 2 and q["blocks_done"] == q["total_blocks"]
    return a.cpu().numpy(), b.cpu().numpy(), m.cpu().numpy()


@pytest.mark.parametrize("n,iters,many", [(256, 0, False), (129, 1, False), (300, 0, True)])
def test_gaussian_int_exact(sess, n, iters, many):
    a0, b0 = I.gauss_inputs(n, 140 + n, mode="int")
    ra, rb, rm = OT.gaussian(a0, b0)
    ga, gb, gm = _eliminate(sess, a0, b0, S.MODE_SLATE, iters=iters, many=many)
    assert np.array_equal(ga.astype(np.float64), ra)
    assert np.array_equal(gb.astype(np.float64), rb)
    assert np.array_equal(gm.astype(np.float64), rm)


def test_gaussian_rodinia_matrix(sess):
    n = 384
    a0, b0 = I.gauss_inputs(n)
    ra, rb, rm = OT.gaussian(a0, b0)
    ga, gb, gm = _eliminate(sess, a0, b0, S.MODE_SLATE, many=True)
    sa, sb, sm_ = _eliminate(sess, a0, b0, S.MODE_STANDALONE, many=True)
    assert np.array_equal(ga, sa) and np.array_equal(gb, sb) and np.array_equal(gm, sm_)
    tol = 4 * n * 2.0 ** -24 * float(np.abs(a0).max())
    assert np.abs(np.triu(ga).astype(np.float64) - np.triu(ra)).max() <= tol
    assert np.abs(gm.astype(np.float64) - rm).max() <= tol
    assert np.abs(gb.astype(np.float64) - rb).max() <= tol * max(1.0, float(np.abs(rb).max()))


def test_gaussian_under_resize_storm(sess):
    """A dependent job under shrinks and grows: every Fan2 reads what the Fan1
    and Fan2 before it wrote, and a grow tops up the RUNNING launch while the
    rest of the job is already queued behind it (its last main CTA waits for
    the top-up's blocks, so stream order holds).  Integer system: the result
    must be the oracle's bit for bit; every launch's counters exact."""
    import random
    import time
    n_sms = sess.info()["num_sms"]
    n = 512
    a0, b0 = I.gauss_inputs(n, 150, mode="int")
    ra, rb, rm = OT.gaussian(a0, b0)
    a = torch.from_numpy(a0).to(DEV)
    b = torch.from_numpy(b0).to(DEV)
    m = torch.zeros(n, n, device=DEV)
    torch.cuda.synchronize()
    k1 = sess.register_kernel(S.KIND_GAUSS_FAN1, iters=1)
    k2 = sess.register_kernel(S.KIND_GAUSS_FAN2, iters=1)
    # a long Black-Scholes launch at the head of the queue: the whole job is
    # queued behind it before the storm starts (submission is slower than the GPU)
    Sx, X, T, r = I.bs_inputs(1 << 22, 152)
    bs = [torch.from_numpy(v).to(DEV) for v in (Sx, X, T, I.bs_sigmas(2048))]
    call, put = torch.zeros(1 << 22, device=DEV), torch.zeros(1 << 22, device=DEV)
    torch.cuda.synchronize()
    bargs, bgrid = S.bs_args(bs[0], bs[1], bs[2], call, put, bs[3], float(r))
    kb = sess.register_kernel(S.KIND_BLACKSCHOLES)
    ids = [sess.launch(kb, bargs, bgrid, placement=S.PLACE_CORUN, sm=(0, n_sms // 4 - 1))]
    for t in range(n - 1):
        args, grid = S.gauss_fan1_args(a, b, m, t)
        ids.append(sess.launch(k1, args, grid, placement=S.PLACE_CORUN, sm=(0, n_sms // 4 - 1)))
        args, grid = S.gauss_fan2_args(a, b, m, t)
        ids.append(sess.launch(k2, args, grid, placement=S.PLACE_CORUN, sm=(0, n_sms // 4 - 1)))
    rng = random.Random(151)
    for i in range(2000):                     # alternate grows to the full chip and shrinks
        lo, hi = (0, n_sms - 1) if i % 2 == 0 else (rng.randrange(0, n_sms // 2), n_sms - 1)
        if sess.resize(ids[-1], lo, hi) == S.DONE:
            break
        time.sleep(0.0001)
    sess.sync(0)
    torch.cuda.synchronize()
    for i in ids[1:]:
        q = sess.query(i)
        assert q["state"] == 2 and q["blocks_done"] == q["total_blocks"] and q["tasks_done"] == q["total_blocks"], q
    assert sess.query(ids[0])["blocks_done"] == int(np.prod(bgrid))
    assert np.array_equal(a.cpu().numpy().astype(np.float64), ra)
    assert np.array_equal(b.cpu().numpy().astype(np.float64), rb)
    assert np.array_equal(m.cpu().numpy().astype(np.float64), rm)
