"""GPU parity of the slate path (-m gpu): every tenant through the C ABI,
  * slate worker output == the same tenant's standalone launch, bit for bit;
  * output == oracle (exact on integer inputs, Q17 tolerance on floats);
  * coverage log all ones and counters == oracle.expected_counters
    (blocks_done, tasks_done, next_clamped), for iters in {1, 10}, on the full
    GPU and on a sub-range of SMs.
Sizes span several tiles and a ragged tail."""
import numpy as np
import pytest
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import slate as S

from gpu_helpers import (make_bs, make_copy, make_gauss_fan1, make_gauss_fan2, make_gemm, make_qrng, make_sgemm,
                         make_sgemm_tiled, make_spmv, make_stencil, make_transpose, make_triad)

pytestmark = pytest.mark.gpu

CASES = {
    "triad_float": lambda: make_triad(1024 * 37 + 517, 101),
    "triad_int": lambda: make_triad(1024 * 50 + 4, 102, "int"),
    "copy": lambda: make_copy(4096 * 21 + 999, 103),
    "sgemm_float": lambda: make_sgemm(200, 232, 96, 104),
    "sgemm_int": lambda: make_sgemm(256, 256, 256, 105, "int"),
    "spmv_float": lambda: make_spmv(32 * 300 + 7, 106, band=512),
    "spmv_int": lambda: make_spmv(32 * 128, 107, "int", band=64),
    # irregular rows (empty ones included): chunks over the staging slot's
    # capacity take the global-memory path
    "spmv_ragged": lambda: make_spmv(32 * 200 + 13, 115, band=3000, ragged=dict(lengths=(0, 48))),
    # a non-square matrix with columns spread over all of x: the x window misses
    "spmv_wide": lambda: make_spmv(32 * 150 + 5, 116, band=None, ragged=dict(lengths=(16, 16), n_cols=50001)),
    # a few very long rows between short ones
    "spmv_long_rows": lambda: make_spmv(32 * 100 + 31, 117, "int", band=None,
                                        ragged=dict(lengths=(0, 4), n_cols=20000, long_rows=3, long_len=3000)),
    "bs": lambda: make_bs(1024 * 12 + 4 * 33 + 2, 108, n_scen=5),
    "stencil_float": lambda: make_stencil(8 * 37 + 3, 32 * 9 + 5, 109),
    "stencil_int": lambda: make_stencil(77, 130, 110, "int"),
    # width a multiple of 4: the float4 path, a ragged last block of 64 columns
    "stencil_vec_float": lambda: make_stencil(8 * 13 + 5, 128 * 3 + 64, 113),
    "stencil_vec_int": lambda: make_stencil(8 * 5 + 2, 128 * 2 + 4, 114, "int"),
    "gemm_int": lambda: make_gemm(256, 512, 512, 113, "int"),
    "gemm_float": lambda: make_gemm(768, 512, 1024, 114),
    # ragged in all three: a partial last tile row (m), column (n) and K slice (k)
    "gemm_ragged_int": lambda: make_gemm(256 * 2 + 77, 256 + 132, 64 * 5 + 24, 131, "int"),
    "gemm_ragged_float": lambda: make_gemm(300, 260, 520, 132),
    # the paper's Tab II apps (NEXT-2)
    "tr": lambda: make_transpose(32 * 11 + 7, 32 * 9 + 19, 120),
    "tr_row": lambda: make_transpose(1, 32 * 40 + 1, 121),
    "mm_float": lambda: make_sgemm_tiled(32 * 7 + 5, 32 * 6 + 31, 32 * 3 + 9, 122),
    "mm_int": lambda: make_sgemm_tiled(256, 192, 160, 123, "int"),
    "rg": lambda: make_qrng(1024 * 13 + 4 * 17 + 2, 3, 124, qseed=5),
    "rg_wrap": lambda: make_qrng(1024 * 3, 2, 125, qseed=2 ** 32 - 1500),   # k wraps past 2^31 and 2^32
    "bs_textbook": lambda: make_bs(1024 * 9 + 3, 130, n_scen=1),
    "gs_fan1": lambda: make_gauss_fan1(700, 37, 126, "rodinia"),
    "gs_fan2_int": lambda: make_gauss_fan2(300, 11, 127, "int"),
    "gs_fan2_float": lambda: make_gauss_fan2(500, 23, 128, "rodinia"),
    "gs_fan2_last": lambda: make_gauss_fan2(200, 198, 129, "int"),
}


@pytest.fixture(scope="module")
def sess():
    s = S.Session(None, 0)
    yield s
    s.close()


def _run(sess, t, kernel, **kw):
    t.zero_outputs()
    cov = torch.zeros(int(np.prod(t.grid)), dtype=torch.int32, device="cuda:0")
    torch.cuda.synchronize()   # the server's streams do not wait for torch's stream
    lid = sess.launch(kernel, t.args, t.grid, coverage=cov if kw.pop("cov", True) else None, **kw)
    sess.sync(lid)
    torch.cuda.synchronize()
    return lid, t.snapshot(), cov


@pytest.mark.parametrize("name", sorted(CASES))
def test_tenant_parity(sess, name):
    t = CASES[name]()
    k_std = sess.register_kernel(t.kind)
    lid, ref_outs, _ = _run(sess, t, k_std, mode=S.MODE_STANDALONE, cov=False)
    ok, err = t.check(ref_outs)
    assert ok, "standalone vs oracle: %s (worst %.3g of tolerance)" % (name, err)
    B = int(np.prod(t.grid))
    n = sess.info()["num_sms"]
    for iters in ((1, 10, 32) if t.kind == S.KIND_SPMV_CSR else (1, 10)):
        k = sess.register_kernel(t.kind, iters=iters, flags=S.KFLAG_COVERAGE)
        for sm in [(0, n - 1), (3, 3 + n // 3)]:
            lid, outs, cov = _run(sess, t, k, placement=S.PLACE_CORUN, sm=sm)
            for a, b in zip(outs, ref_outs):
                assert torch.equal(a, b), "slate vs standalone not bit-exact: %s iters=%d sm=%s" % (name, iters, sm)
            q = sess.query(lid)
            ex = OT.expected_counters(B, iters)
            assert q["state"] == 2 and q["coverage_ok"] == 1
            assert np.array_equal(cov.cpu().numpy(), ex["coverage"].astype(np.int32))
            assert (q["blocks_done"], q["tasks_done"], q["next_clamped"]) == \
                (ex["blocks_done"], ex["tasks_done"], ex["next_clamped"]), (name, iters, q)
            assert q["live_workers"] == 0


def test_empty_and_single_block(sess):
    t = make_triad(3, 111)          # one block, 3 elements (ragged inside a float4)
    k = sess.register_kernel(t.kind, iters=10, flags=S.KFLAG_COVERAGE)
    lid, outs, cov = _run(sess, t, k, placement=S.PLACE_CORUN, sm=(0, 0))
    assert t.check(outs)[0]
    assert sess.query(lid)["tasks_done"] == 1
    with pytest.raises(S.SlateError):
        args, grid = S.triad_args(torch.zeros(0, device="cuda:0"), torch.zeros(0, device="cuda:0"),
                                  torch.zeros(0, device="cuda:0"), 1.0)
        sess.launch(k, args, grid)
    with pytest.raises(S.SlateError):          # grid inconsistent with args
        sess.launch(k, t.args, (2, 1, 1))
    with pytest.raises(S.SlateError):          # bad SM range
        sess.launch(k, t.args, t.grid, placement=S.PLACE_CORUN, sm=(5, 4))


def test_auto_solo_path(sess):
    t = make_stencil(8 * 64, 32 * 64, 112)
    k = sess.register_kernel(t.kind)
    lid = sess.launch(k, t.args, t.grid, placement=S.PLACE_AUTO)
    sess.sync(lid)
    assert t.check(t.snapshot())[0]
    q = sess.query(lid)
    assert q["blocks_done"] == q["total_blocks"] and q["end_ms"] >= q["start_ms"] > 0


def test_gemm_full_size_sampled(sess):
    """bf16 GEMM 8192^3 (BASELINE config 3) in the bench's launch configuration:
    slate == standalone bit for bit, exact counters, and 24 sampled 128x128
    tiles against the fp64 oracle; integer inputs in [-2, 2] keep every partial
    sum below 2^24, so those tiles must match exactly."""
    import random
    for mode in ("int", "float"):
        t = make_gemm(8192, 8192, 8192, 115, mode)
        k_std = sess.register_kernel(t.kind)
        _, ref, _ = _run(sess, t, k_std, mode=S.MODE_STANDALONE, cov=False)
        k = sess.register_kernel(t.kind, flags=S.KFLAG_COVERAGE)
        lid, outs, cov = _run(sess, t, k, placement=S.PLACE_AUTO)
        assert torch.equal(outs[0], ref[0])
        q = sess.query(lid)
        B = int(np.prod(t.grid))
        assert q["coverage_ok"] == 1 and q["blocks_done"] == B and q["tasks_done"] == B
        rng = random.Random(116)
        tiles = [(0, 0), (63, 63)] + [(rng.randrange(64), rng.randrange(64)) for _ in range(22)]
        ok, err = t.check(outs, rows=tiles)
        assert ok, (mode, err)


def test_launch_n_job(sess):
    """slate_launch_n: a job of n launches in one call -- consecutive ids, every
    launch complete with exact counters, the output the oracle's."""
    t = make_triad(1024 * 40 + 3, 118, "int")
    k = sess.register_kernel(t.kind, iters=4)
    t.zero_outputs()
    torch.cuda.synchronize()
    ids = sess.launch_n(k, t.args, t.grid, 5)
    assert ids == list(range(ids[0], ids[0] + 5))
    sess.sync(0)
    torch.cuda.synchronize()
    B = int(np.prod(t.grid))
    for i in ids:
        q = sess.query(i)
        assert q["state"] == 2 and q["blocks_done"] == B and q["tasks_done"] == -(-B // 4)
    assert t.check(t.snapshot())[0]
