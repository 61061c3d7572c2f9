"""Seeded synthetic inputs for the tenant kernels.

This module is the ONLY code shared by the CUDA path's harness (tests, bench)
and the CPU oracle's harness: it draws random numbers and lays out arrays, and
holds none of the method's arithmetic.  Recipes follow
SURVEY.md §8(d): numpy PCG64, seed = 20190520 + 100*cfg + tenant; every tenant
has an ``int`` mode (small integers: every fp32 result is exact, so GPU and
oracle agree bit for bit) and a ``float`` mode (realistic values, tolerance).
"""
import numpy as np

BASE_SEED = 20190520


def seed_for(cfg, tenant):
    return BASE_SEED + 100 * cfg + tenant


def rng(seed):
    return np.random.Generator(np.random.PCG64(seed))


def _vec(g, n, mode, int_lo, int_hi):
    if mode == "int":
        return g.integers(int_lo, int_hi + 1, size=n).astype(np.float32)
    return g.uniform(-1.0, 1.0, size=n).astype(np.float32)


def triad_inputs(n, seed, mode="float"):
    """b, c in U[-1,1) (float) or integers in [-2^10, 2^10] (int); s = 3."""
    g = rng(seed)
    return _vec(g, n, mode, -1024, 1024), _vec(g, n, mode, -1024, 1024), np.float32(3.0)


def copy_inputs(n, seed, mode="float"):
    return _vec(rng(seed), n, mode, -1024, 1024)


def sgemm_inputs(m, n, k, seed, mode="float"):
    """A (m x k), B (k x n) row-major fp32; U[-1,1) or integers in [-4, 4]."""
    g = rng(seed)
    A = _vec(g, m * k, mode, -4, 4).reshape(m, k)
    B = _vec(g, k * n, mode, -4, 4).reshape(k, n)
    return A, B


def spmv_inputs(n_rows, seed, mode="float", nnz_per_row=16, band=4096, n_cols=None):
    """CSR with ``nnz_per_row`` distinct sorted columns per row drawn from the
    band [i - band, i + band] clipped to [0, n_cols) (fewer when the clipped band
    is narrower than nnz_per_row).  int32 rowptr/col, fp32 val and x:
    U[-1,1) or integers in [-2, 2]."""
    n_cols = n_rows if n_cols is None else n_cols
    g = rng(seed)
    i = np.arange(n_rows, dtype=np.int64)
    start = np.clip(i - band, 0, n_cols)
    stop = np.clip(i + band + 1, 0, n_cols)
    width = stop - start
    per_row = np.minimum(width, nnz_per_row)
    # k distinct sorted offsets in [0, width): sorted draws with replacement from
    # [0, width - k] plus 0..k-1 (strictly increasing by construction)
    k = nnz_per_row
    draws = np.sort(g.integers(0, 1 << 62, size=(n_rows, k)) % np.maximum(width - per_row + 1, 1)[:, None], axis=1)
    offs = draws + np.arange(k)[None, :]
    mask = np.arange(k)[None, :] < per_row[:, None]
    cols = (start[:, None] + offs)[mask].astype(np.int32)
    rowptr = np.zeros(n_rows + 1, dtype=np.int64)
    rowptr[1:] = np.cumsum(per_row)
    nnz = int(rowptr[-1])
    val = _vec(g, nnz, mode, -2, 2)
    x = _vec(g, n_cols, mode, -2, 2)
    return rowptr.astype(np.int32), cols, val, x


def spmv_ragged_inputs(n_rows, seed, mode="float", lengths=(0, 48), band=None, n_cols=None, long_rows=0,
                       long_len=2000):
    """CSR with irregular rows: each row's length uniform in ``lengths`` (empty
    rows included), plus ``long_rows`` rows of ``long_len`` nonzeros at random
    positions; distinct sorted columns uniform in [i - band, i + band] clipped to
    [0, n_cols), or over all columns when ``band`` is None.  Same dtypes and
    value ranges as spmv_inputs."""
    n_cols = n_rows if n_cols is None else n_cols
    g = rng(seed)
    per_row = g.integers(lengths[0], lengths[1] + 1, size=n_rows)
    if long_rows:
        per_row[g.choice(n_rows, size=long_rows, replace=False)] = long_len
    cols = []
    for i in range(n_rows):
        lo, hi = (0, n_cols) if band is None else (max(0, i - band), min(n_cols, i + band + 1))
        k = min(int(per_row[i]), hi - lo)
        per_row[i] = k
        cols.append(np.sort(g.choice(hi - lo, size=k, replace=False)) + lo)
    rowptr = np.zeros(n_rows + 1, dtype=np.int64)
    rowptr[1:] = np.cumsum(per_row)
    nnz = int(rowptr[-1])
    col = np.concatenate(cols).astype(np.int32) if nnz else np.zeros(0, np.int32)
    val = _vec(g, nnz, mode, -2, 2)
    x = _vec(g, n_cols, mode, -2, 2)
    return rowptr.astype(np.int32), col, val, x


def bs_inputs(n, seed):
    """Option batch in the CUDA SDK BlackScholes sample's ranges: stock price
    S ~ U[5, 30], strike X ~ U[1, 100], expiry T ~ U[0.25, 10] years; SoA fp32.
    The riskless rate r = 0.02 is a constant of the workload."""
    g = rng(seed)
    S = g.uniform(5.0, 30.0, size=n).astype(np.float32)
    X = g.uniform(1.0, 100.0, size=n).astype(np.float32)
    T = g.uniform(0.25, 10.0, size=n).astype(np.float32)
    return S, X, T, np.float32(0.02)


def bs_sigmas(p_count, sigma0=0.30, dsigma=0.01):
    """Volatility scenarios sigma_p = sigma0 + p*dsigma, p = 0..P-1 (reading Q16),
    as float32: the values both the kernel and the oracle are given."""
    return (np.float32(sigma0) + np.float32(dsigma) * np.arange(p_count, dtype=np.float32)).astype(np.float32)


def stencil_inputs(h, w, seed, mode="float"):
    """HxW fp32 field: U[0,1) (float) or a random integer linear field
    f = a*i + b*j + c with small integer a, b, c (int)."""
    g = rng(seed)
    if mode == "int":
        a, b, c = (int(v) for v in g.integers(-3, 4, size=3))
        i = np.arange(h, dtype=np.int64)[:, None]
        j = np.arange(w, dtype=np.int64)[None, :]
        return (a * i + b * j + c).astype(np.float32)
    return g.uniform(0.0, 1.0, size=(h, w)).astype(np.float32)


def to_bf16_bits(x):
    """Round-toward-zero fp32 -> bf16 bit patterns (uint16): the input
    distribution only; exact for values already representable in bf16."""
    return (np.ascontiguousarray(x, dtype=np.float32).view(np.uint32) >> np.uint32(16)).astype(np.uint16)


def gemm_inputs(m, n, k, seed, mode="float"):
    """A (m x k) and B (n x k), both K-major bf16 bit patterns (uint16):
    U[-1,1) or integers in [-2, 2]."""
    g = rng(seed)
    A = _vec(g, m * k, mode, -2, 2).reshape(m, k)
    B = _vec(g, n * k, mode, -2, 2).reshape(n, k)
    return to_bf16_bits(A), to_bf16_bits(B)


# ---------------------------------------------------------------- the paper's Tab II apps (NEXT-2)
def transpose_inputs(h, w, seed, mode="float"):
    """h x w fp32 matrix: U[-1,1) or integers in [-2^10, 2^10]."""
    return _vec(rng(seed), h * w, mode, -1024, 1024).reshape(h, w)


def qrng_table(dims, seed, bits=31):
    """dims x bits uint32 generator table of a digital (0,1)-style sequence:
    entry b of a dimension has its leading bit at position bits-1-b and random
    bits below it (an upper unit-triangular generator matrix over GF(2)), so
    every dimension is a permutation-preserving digital sequence.  Dimension 0
    is the van der Corput sequence (no bits below the leading one)."""
    g = rng(seed)
    t = np.zeros((dims, bits), dtype=np.uint32)
    for d in range(dims):
        for b in range(bits):
            lead = 1 << (bits - 1 - b)
            low = 0 if d == 0 else int(g.integers(0, lead))
            t[d, b] = lead | low
    return t


def gauss_inputs(n, seed=None, mode="rodinia"):
    """Linear system a (n x n fp32) and right-hand side b (n fp32).

    ``rodinia``: Rodinia gaussian's generated matrix (``-s n``):
    a[i][j] = 10 exp(-0.01 |i - j|) (symmetric positive definite, so no pivoting
    is needed), b = 1.  ``int``: a = L U with L unit lower triangular, entries
    in {-1, 0, 1}, and U upper triangular with unit diagonal and entries in
    [-2, 2], and b = L y with y integers in [-4, 4]: after step t every
    trailing entry is sum_{k >= t} L_ik U_kj (resp. L_ik y_k), so every
    multiplier and every intermediate value of the elimination is a small
    integer, exact in fp32."""
    if mode == "rodinia":
        i = np.arange(n)
        a = (10.0 * np.exp(-0.01 * np.abs(i[:, None] - i[None, :]))).astype(np.float32)
        return a, np.ones(n, dtype=np.float32)
    g = rng(seed)
    L = np.tril(g.integers(-1, 2, size=(n, n)), -1) + np.eye(n, dtype=np.int64)
    U = np.triu(g.integers(-2, 3, size=(n, n)), 1) + np.eye(n, dtype=np.int64)
    a = (L @ U).astype(np.float32)
    y = g.integers(-4, 5, size=n)
    b = (L @ y).astype(np.float32)
    return a, b
