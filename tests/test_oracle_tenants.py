"""Pins for oracle/tenants.py (CPU only): each tenant body against closed forms,
special cases that reduce to a library routine, invariants and textbook values.
None of these re-types the oracle's own formula."""
import math
import os

import numpy as np
import scipy.signal
import scipy.sparse

from oracle import tenants as T
from paper_conf_ipps_allenf019_b200 import inputs as I

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ triad / copy
def test_triad_special_cases_and_linearity():
    n = 5000                                     # 5 blocks, ragged tail
    b, c, s = I.triad_inputs(n, 1, mode="int")
    a = T.triad(b, c, s)
    # s = 0 reduces to copy; c = 0 reduces to copy; b = 0, s = 1 gives c
    assert np.array_equal(T.triad(b, c, 0.0), b.astype(np.float64))
    assert np.array_equal(T.triad(b, np.zeros_like(c), s), b.astype(np.float64))
    assert np.array_equal(T.triad(np.zeros_like(b), c, 1.0), c.astype(np.float64))
    # exact sum identity on integer inputs: sum a = sum b + s sum c
    assert a.sum() == b.astype(np.int64).sum() + 3 * c.astype(np.int64).sum()
    # integer inputs: every fp32 result is exact, so the float32 cast round-trips
    assert np.array_equal(a.astype(np.float32).astype(np.float64), a)


def test_copy_is_bytes():
    b = I.copy_inputs(4096 * 3 + 17, 2)
    assert T.copy(b).tobytes() == b.tobytes()


def test_block_subset_covers_only_those_blocks():
    b, c, s = I.triad_inputs(4096, 3)
    a = T.triad(b, c, s, blocks=[1, 3])
    assert np.all(a[:1024] == 0) and np.all(a[2048:3072] == 0)
    assert np.any(a[1024:2048] != 0) and np.any(a[3072:] != 0)


# ------------------------------------------------------------------ sgemm
def test_sgemm_identity_and_library():
    A, B = I.sgemm_inputs(40, 56, 24, 4, mode="int")   # ragged 16x16 tiles
    C = T.sgemm_naive(A, B)
    assert np.array_equal(C, A.astype(np.int64) @ B.astype(np.int64))
    eye = np.eye(24, dtype=np.float32)
    assert np.array_equal(T.sgemm_naive(A, eye), A.astype(np.float64))
    A2, B2 = I.sgemm_inputs(33, 17, 65, 5)
    np.testing.assert_allclose(T.sgemm_naive(A2, B2), np.matmul(A2.astype(np.float64), B2.astype(np.float64)),
                               rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------ spmv
def test_spmv_identity_library_and_invariant():
    n = 1000
    rp = np.arange(n + 1, dtype=np.int32)
    col = np.arange(n, dtype=np.int32)
    x = I.copy_inputs(n, 6)
    assert np.array_equal(T.spmv_csr(rp, col, np.ones(n, np.float32), x), x.astype(np.float64))
    rp, col, val, x = I.spmv_inputs(2000, 7, mode="int", band=64)
    y = T.spmv_csr(rp, col, val, x)
    A = scipy.sparse.csr_matrix((val.astype(np.int64), col, rp), shape=(2000, 2000))
    assert np.array_equal(y, A @ x.astype(np.int64))
    # sum_i y_i = sum_j x_j * colsum_j(A), exact in int64
    colsum = np.bincount(col, weights=val.astype(np.int64), minlength=2000).astype(np.int64)
    assert int(y.sum()) == int((colsum * x.astype(np.int64)).sum())


def test_spmv_generator_structure():
    rp, col, val, x = I.spmv_inputs(10000, 8, band=4096)
    assert rp[0] == 0 and np.all(np.diff(rp) == 16)
    for i in [0, 1, 5000, 9999]:
        c = col[rp[i]:rp[i + 1]]
        assert np.all(np.diff(c) > 0) and c.min() >= max(0, i - 4096) and c.max() <= min(9999, i + 4096)


# ------------------------------------------------------------------ Black-Scholes
def _bs_golden():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "bs_textbook.txt")) if l.strip() and l[0] != "#"]
    return [tuple(float(v) for v in r) for r in rows]


def test_bs_textbook_values():
    for S, X, Tm, r, sg, call, put, d1, d2 in _bs_golden():
        c, p = T.bs_option(np.array([S]), np.array([X]), np.array([Tm]), r, sg)
        assert round(float(c[0]), 2) == call and round(float(p[0]), 2) == put


def test_bs_put_call_parity_and_limits():
    S, X, Tm, r = I.bs_inputs(3000, 9)
    sig = I.bs_sigmas(4)
    call, put = T.blackscholes(S, X, Tm, r, sig)
    S64, X64, T64 = (v.astype(np.float64) for v in (S, X, Tm))
    # put-call parity holds for every scenario, hence for the mean: C - P = S - X e^{-rT}
    np.testing.assert_allclose(call - put, S64 - X64 * np.exp(-float(r) * T64), rtol=0, atol=1e-9 * S64.max())
    # sigma sqrt T -> 0: C -> max(S - X e^{-rT}, 0)
    c0, _ = T.bs_option(S64, X64, T64, float(r), 1e-9)
    np.testing.assert_allclose(c0, np.maximum(S64 - X64 * np.exp(-float(r) * T64), 0), atol=1e-6)
    # Phi(x) + Phi(-x) = 1, Phi(0) = 1/2, Phi(1.96) = 0.975002 (normal table)
    xs = np.linspace(-6, 6, 101)
    np.testing.assert_allclose(T.phi(xs) + T.phi(-xs), 1.0, atol=1e-15)
    assert T.phi(0.0) == 0.5 and abs(T.phi(1.96) - 0.9750021) < 1e-7
    # bounds: max(S - X e^{-rT}, 0) <= C <= S
    assert np.all(call <= S64 + 1e-9) and np.all(call >= np.maximum(S64 - X64 * np.exp(-float(r) * T64), 0) - 1e-9)


def test_bs_mean_over_scenarios():
    S, X, Tm, r = I.bs_inputs(1024 + 5, 10)
    sig = I.bs_sigmas(3)
    call, put = T.blackscholes(S, X, Tm, r, sig)
    one = [T.blackscholes(S, X, Tm, r, sig[i:i + 1]) for i in range(3)]
    np.testing.assert_allclose(call, sum(o[0] for o in one) / 3, rtol=1e-14)
    np.testing.assert_allclose(put, sum(o[1] for o in one) / 3, rtol=1e-14)


# ------------------------------------------------------------------ stencil
def test_stencil_fixed_points_and_library():
    h, w = 37, 70                                    # ragged 32x8 blocks
    const = np.full((h, w), 0.3, np.float32)
    assert np.array_equal(T.stencil2d(const), const.astype(np.float64))
    lin = I.stencil_inputs(h, w, 11, mode="int")     # a*i + b*j + c is harmonic
    assert np.array_equal(T.stencil2d(lin), lin.astype(np.float64))
    f = I.stencil_inputs(h, w, 12).astype(np.float64)
    k = np.array([[0, .25, 0], [.25, 0, .25], [0, .25, 0]])
    ref = f.copy()
    ref[1:-1, 1:-1] = scipy.signal.convolve2d(f, k, mode="valid")
    np.testing.assert_allclose(T.stencil2d(f.astype(np.float32)), ref, rtol=1e-15, atol=1e-15)
    tiny = I.stencil_inputs(2, 5, 13)
    assert np.array_equal(T.stencil2d(tiny), tiny.astype(np.float64))


# ------------------------------------------------------------------ bf16 GEMM
def test_bf16_decoding():
    bits = np.array([0x3F80, 0xC000, 0x0000, 0x8000, 0x3F00, 0x4049, 0x7F80], dtype=np.uint16)
    vals = T.bf16_to_f64(bits)
    assert list(vals[:5]) == [1.0, -2.0, 0.0, -0.0, 0.5] and vals[5] == 3.140625 and math.isinf(vals[6])
    import torch
    x = torch.randn(1000, dtype=torch.float32).to(torch.bfloat16)
    assert np.array_equal(T.bf16_to_f64(x.view(torch.int16).numpy().view(np.uint16)),
                          x.to(torch.float64).numpy())


def test_gemm_bf16_int_exact_and_sums():
    A, B = I.gemm_inputs(200, 136, 96, 14, mode="int")   # ragged 128x128 tiles
    C = T.gemm_bf16(A, B)
    Ai = T.bf16_to_f64(A).astype(np.int64)
    Bi = T.bf16_to_f64(B).astype(np.int64)
    assert np.array_equal(C, Ai @ Bi.T)
    # row-sum identity C 1 = A (B^T 1) and column-sum identity 1^T C = (1^T A) B^T
    assert np.array_equal(C.sum(axis=1).astype(np.int64), Ai @ Bi.sum(axis=0))
    assert np.array_equal(C.sum(axis=0).astype(np.int64), Bi @ Ai.sum(axis=0))
    Af, Bf = I.gemm_inputs(130, 129, 64, 15)
    np.testing.assert_allclose(T.gemm_bf16(Af, Bf),
                               T.bf16_to_f64(Af) @ T.bf16_to_f64(Bf).T, rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------ probe3d (3-D grid of 3-D blocks)
def test_probe3d_block_ids_and_linearity():
    """With a zero input each element holds the id term of the block that
    wrote it: the block is the element's coordinates integer-divided by the
    block shape (not decode(): an independent route), and every element of the
    ragged 3-D field is written exactly once; the input term is linear."""
    shape, block = (7, 11, 37), (8, 4, 2)          # (nz, ny, nx), (bx, by, bz): ragged in all three
    assert T.probe3d_grid(shape, block) == (5, 3, 4)
    z = T.probe3d(np.zeros(shape, np.float32), block)
    k, j, i = np.meshgrid(np.arange(7), np.arange(11), np.arange(37), indexing="ij")
    assert np.array_equal(z, (i // 8) + 3 * (j // 4) + 7 * (k // 2))
    rng = np.random.default_rng(3)
    x = rng.integers(-50, 50, size=shape).astype(np.float32)
    assert np.array_equal(T.probe3d(x, block) - z, 2.0 * x.astype(np.float64))
    # a subset of blocks writes only the elements of those blocks
    part = T.probe3d(np.ones(shape, np.float32), block, blocks=[17])   # block 17 = (2, 0, 1)
    nz_ = np.argwhere(part != 0)
    assert nz_.size and set(map(tuple, (nz_ // [2, 4, 8]).tolist())) == {(1, 0, 2)}
