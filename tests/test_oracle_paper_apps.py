"""Pins for the oracle of the paper's own applications (Tab II, P:L277-285;
NEXT-2): transpose (TR), tiled matrixMul (MM), quasirandom generator (RG),
Gaussian elimination (GS).  CPU only; each pin comes from a library routine,
a closed form or an invariant, never from re-typing the oracle's formula."""
import numpy as np
import scipy.linalg

from oracle import tenants as T
from paper_conf_ipps_allenf019_b200 import inputs as I


# ------------------------------------------------------------------ TR
def test_transpose_library_and_involution():
    A = I.transpose_inputs(70, 45, 21)                 # ragged 32x32 tiles both ways
    out = T.transpose(A)
    assert out.shape == (45, 70) and out.tobytes() == np.ascontiguousarray(A.T).tobytes()
    assert T.transpose(out).tobytes() == A.tobytes()
    one = T.transpose(np.arange(5, dtype=np.float32).reshape(1, 5))
    assert one.shape == (5, 1) and list(one[:, 0]) == [0, 1, 2, 3, 4]


def test_transpose_block_subset():
    A = I.transpose_inputs(64, 64, 22)
    out = T.transpose(A, blocks=[1])                   # block (x=1, y=0): input rows 0..31, cols 32..63
    assert np.array_equal(out[32:, :32], A[:32, 32:].T)
    assert not out[:32].any() and not out[32:, 32:].any()


# ------------------------------------------------------------------ MM
def test_sgemm_tiled_integer_exact_and_identity():
    A, B = I.sgemm_inputs(70, 40, 50, 23, mode="int")    # ragged 32x32 tiles
    assert np.array_equal(T.sgemm_tiled(A, B), A.astype(np.int64) @ B.astype(np.int64))
    assert np.array_equal(T.sgemm_tiled(A, np.eye(50, dtype=np.float32)), A.astype(np.float64))
    A2, B2 = I.sgemm_inputs(33, 35, 31, 24)
    np.testing.assert_allclose(T.sgemm_tiled(A2, B2), A2.astype(np.float64) @ B2.astype(np.float64),
                               rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------ RG
def _radical_inverse_2(k, bits=31):
    """van der Corput radical inverse by repeated division by 2 (digit expansion)."""
    r, f = 0.0, 0.5
    while k:
        k, d = divmod(k, 2)
        r += d * f
        f /= 2
    return r


def test_qrng_van_der_corput_dimension():
    table = I.qrng_table(3, 25)
    n = 3000
    out = T.qrng(table, n, 0)
    # dimension 0 is the van der Corput sequence: (q + 1) 2^-31 = phi_2(k) + 2^-31
    ref = np.array([_radical_inverse_2(k) + 2.0 ** -31 for k in range(n)]).astype(np.float32)
    assert np.array_equal(out[0], ref)
    assert out[0, 1] == np.float32(0.5 + 2.0 ** -31) and out[0, 3] == np.float32(0.75 + 2.0 ** -31)


def test_qrng_digital_net_properties():
    table = I.qrng_table(3, 26)
    # GF(2) linearity: q(a ^ b) = q(a) ^ q(b)
    for a, b in [(5, 9), (1023, 77), (2 ** 30 + 3, 12345)]:
        for d in range(3):
            assert T.qrng_point(table[d], a ^ b) == T.qrng_point(table[d], a) ^ T.qrng_point(table[d], b)
    # unit-triangular generator: the leading m bits of the first 2^m points are a permutation
    m = 10
    for d in range(3):
        lead = [T.qrng_point(table[d], k) >> (31 - m) for k in range(2 ** m)]
        assert sorted(lead) == list(range(2 ** m))
    # the seed offsets the index; every value lies in (0, 1]
    out = T.qrng(table, 1500, 7)
    ref = T.qrng(table, 1507, 0)
    assert np.array_equal(out, ref[:, 7:])
    assert out.min() > 0 and out.max() <= 1.0


# ------------------------------------------------------------------ GS
def test_gaussian_matches_cholesky_factorisation():
    n = 97                                            # ragged Fan1/Fan2 blocks
    a0, b0 = I.gauss_inputs(n)
    a, b, m = T.gaussian(a0, b0)
    A = a0.astype(np.float64)
    # SPD: A = L D L^T with L = C diag(C)^-1 (C = Cholesky factor); elimination
    # without pivoting gives multipliers L and the upper factor U = D L^T
    C = np.linalg.cholesky(A)
    L = C / np.diag(C)[None, :]
    U = (np.diag(C)[:, None] * C.T)
    np.testing.assert_allclose(np.tril(m, -1), np.tril(L, -1), rtol=1e-10, atol=1e-10)
    np.testing.assert_allclose(np.triu(a), U, rtol=1e-10, atol=1e-9)
    assert np.abs(np.tril(a, -1)).max() < 1e-9       # eliminated entries are rounding residue
    # forward-substituted right-hand side and the solution by back substitution
    np.testing.assert_allclose(b, scipy.linalg.solve_triangular(L, b0.astype(np.float64), lower=True,
                                                                unit_diagonal=True), rtol=1e-10, atol=1e-10)
    x = scipy.linalg.solve_triangular(np.triu(a), b)
    np.testing.assert_allclose(x, np.linalg.solve(A, b0.astype(np.float64)), rtol=1e-8, atol=1e-10)


def test_gaussian_integer_factors_recovered_exactly():
    n = 60
    a0, b0 = I.gauss_inputs(n, 27, mode="int")
    a, b, m = T.gaussian(a0, b0)
    # a0 = L U built from integer factors: elimination recovers them exactly
    Lm = np.tril(m, -1) + np.eye(n)
    assert np.array_equal(Lm @ np.triu(a), a0.astype(np.float64))
    assert np.array_equal(np.tril(a, -1), np.zeros((n, n)))
    assert np.all(np.diag(a) == 1.0) and np.all(m == np.round(m))
    assert np.array_equal(Lm @ b, b0.astype(np.float64))


def test_gaussian_steps_compose_and_grids():
    n = 40
    a0, b0 = I.gauss_inputs(n, 28, mode="int")
    a5, b5, m5 = T.gaussian(a0, b0, steps=5)
    # the first 5 columns are eliminated and the trailing block is the Schur complement
    A = a0.astype(np.float64)
    S = A[5:, 5:] - A[5:, :5] @ np.linalg.solve(A[:5, :5], A[:5, 5:])
    np.testing.assert_allclose(a5[5:, 5:], S, rtol=1e-12, atol=1e-9)
    assert T.gauss_fan2_grid(n, 0) == (1, 3, 1) and T.gauss_fan2_grid(300, 10) == (3, 19, 1)
    assert T.gauss_fan1_grid(n, n - 2) == (1, 1, 1)
