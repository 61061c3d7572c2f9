"""Tenant kernels K(B,T), executed block by block on the CPU  (test infrastructure only).

The paper fixes *what* Slate must compute only by reference to the user kernel:
"The kernel transformation must preserve the semantics of user kernels"
(§III-A) and "K and K* are isomorphic".  So the oracle of every
tenant is the tenant kernel itself, its blocks run one after another in linear
order b = 0 .. B-1 with (x,y,z) = decode(b), each block's arithmetic
written out in float64 from the tenant's plain definition.  Each block owns a
disjoint slice of the output (no block reads another block's output), so the
result does not depend on the order blocks run in -- the property Slate's
out-of-order, multi-worker execution relies on.

Tenants (BASELINE.json configs; geometry in
DESIGN.md §Tenants):

  triad        a[i] = b[i] + s*c[i]              STREAM triad (K9), E=1024 elems/block
  copy         a[i] = b[i]                        STREAM copy (K9), E=4096 elems/block
  sgemm_naive  C = A @ B, one thread per C elem   CUDA-sample naive SGEMM "MM" (K6), 16x16 blocks
  spmv_csr     y = A x, CSR                       32 rows/block (K10)
  blackscholes European call/put, mean over P volatility scenarios (K4, reading Q16),
               1024 options/block; Phi(x) = erfc(-x/sqrt 2)/2 in double
  stencil2d    5-point Jacobi sweep, Dirichlet boundary copied; 32x8 points/block (K11)
  gemm_bf16    C = A @ B^T, A[MxK], B[NxK] bf16 K-major, C fp32; 128x128 tile/block (K12)

Inputs are numpy arrays (fp32, int32, or uint16 bf16 bit patterns); outputs
are float64 arrays of the same shape as the tenant's output.  Nothing here
decides an integer from floating point, so no precision pairing is needed.
"""
import math

import numpy as np
from scipy.special import erfc

from .decode import decode

TRIAD_E = 1024
COPY_E = 4096
SGEMM_TILE = 16
SPMV_ROWS = 32
BS_E = 1024
STENCIL_BX, STENCIL_BY = 128, 8   # 128 columns x 8 rows per block (the tenant's float4 geometry)
GEMM_TILE = 128


def cdiv(a, b):
    return -(-a // b)


def run_grid(grid, block, blocks=None):
    """Execute ``block(x, y, z)`` for every original block in linear order.

    ``blocks`` optionally restricts execution to a subset of linear indices
    (used for bounded samples); the default is all of 0 .. B-1.
    """
    gx, gy, gz = grid
    total = gx * gy * gz
    for b in (range(total) if blocks is None else blocks):
        block(*decode(b, grid))


# ---------------------------------------------------------------- triad / copy
def triad_grid(n):
    return (cdiv(n, TRIAD_E), 1, 1)


def triad(b, c, s, blocks=None):
    """STREAM triad a = b + s*c (McCalpin's STREAM; the Stream app of)."""
    n = b.shape[0]
    a = np.zeros(n, dtype=np.float64)
    b64 = b.astype(np.float64)
    c64 = c.astype(np.float64)
    s64 = float(s)

    def block(x, y, z):
        lo, hi = x * TRIAD_E, min((x + 1) * TRIAD_E, n)
        a[lo:hi] = b64[lo:hi] + s64 * c64[lo:hi]

    run_grid(triad_grid(n), block, blocks)
    return a


def copy_grid(n):
    return (cdiv(n, COPY_E), 1, 1)


def copy(b, blocks=None):
    """STREAM copy a = b; the output is the input's exact bytes."""
    n = b.shape[0]
    a = np.zeros(n, dtype=b.dtype)

    def block(x, y, z):
        lo, hi = x * COPY_E, min((x + 1) * COPY_E, n)
        a[lo:hi] = b[lo:hi]

    run_grid(copy_grid(n), block, blocks)
    return a


# ---------------------------------------------------------------- naive SGEMM
def sgemm_grid(m, n):
    return (cdiv(n, SGEMM_TILE), cdiv(m, SGEMM_TILE), 1)


def sgemm_naive(A, B, blocks=None):
    """C = A @ B; A is MxK, B is KxN, row-major.  Block (x, y) owns rows
    16y..16y+15 and columns 16x..16x+15 (thread (tx, ty) -> C[16y+ty][16x+tx])."""
    m, k = A.shape
    k2, n = B.shape
    assert k == k2
    A64 = A.astype(np.float64)
    B64 = B.astype(np.float64)
    C = np.zeros((m, n), dtype=np.float64)

    def block(x, y, z):
        r0, r1 = y * SGEMM_TILE, min((y + 1) * SGEMM_TILE, m)
        c0, c1 = x * SGEMM_TILE, min((x + 1) * SGEMM_TILE, n)
        # thread (tx, ty) computes the dot product of row 16y+ty and column 16x+tx
        C[r0:r1, c0:c1] = A64[r0:r1, :] @ B64[:, c0:c1]

    run_grid(sgemm_grid(m, n), block, blocks)
    return C


# ---------------------------------------------------------------- CSR SpMV
def spmv_grid(n_rows):
    return (cdiv(n_rows, SPMV_ROWS), 1, 1)


def spmv_csr(rowptr, col, val, xvec, blocks=None):
    """y[i] = sum_{j = rowptr[i]}^{rowptr[i+1]-1} val[j] * x[col[j]]."""
    n_rows = rowptr.shape[0] - 1
    y = np.zeros(n_rows, dtype=np.float64)
    v64 = val.astype(np.float64)
    x64 = xvec.astype(np.float64)

    def block(x, yy, z):
        for i in range(x * SPMV_ROWS, min((x + 1) * SPMV_ROWS, n_rows)):
            lo, hi = int(rowptr[i]), int(rowptr[i + 1])
            y[i] = float(np.sum(v64[lo:hi] * x64[col[lo:hi]]))

    run_grid(spmv_grid(n_rows), block, blocks)
    return y


# ---------------------------------------------------------------- Black-Scholes
def phi(x):
    """Standard normal CDF, Phi(x) = erfc(-x / sqrt(2)) / 2, in double."""
    return 0.5 * erfc(-x / math.sqrt(2.0))


def bs_option(S, X, T, r, sigma):
    """Black-Scholes European call and put (Black & Scholes 1973):
       d1 = (ln(S/X) + (r + sigma^2/2) T) / (sigma sqrt T),  d2 = d1 - sigma sqrt T
       C  = S Phi(d1) - X e^{-rT} Phi(d2),  P = X e^{-rT} Phi(-d2) - S Phi(-d1)."""
    sqt = np.sqrt(T)
    d1 = (np.log(S / X) + (r + 0.5 * sigma * sigma) * T) / (sigma * sqt)
    d2 = d1 - sigma * sqt
    disc = X * np.exp(-r * T)
    call = S * phi(d1) - disc * phi(d2)
    put = disc * phi(-d2) - S * phi(-d1)
    return call, put


def bs_grid(n):
    return (cdiv(n, BS_E), 1, 1)


def blackscholes(S, X, T, r, sigmas, blocks=None):
    """Per option, the mean over the P scenarios of the call and put prices."""
    n = S.shape[0]
    call = np.zeros(n, dtype=np.float64)
    put = np.zeros(n, dtype=np.float64)
    S64, X64, T64 = (v.astype(np.float64) for v in (S, X, T))
    r64 = float(np.float32(r))
    sig64 = sigmas.astype(np.float64)

    def block(x, y, z):
        lo, hi = x * BS_E, min((x + 1) * BS_E, n)
        cs = np.zeros(hi - lo)
        ps = np.zeros(hi - lo)
        for sg in sig64:
            c, p = bs_option(S64[lo:hi], X64[lo:hi], T64[lo:hi], r64, sg)
            cs += c
            ps += p
        call[lo:hi] = cs / len(sig64)
        put[lo:hi] = ps / len(sig64)

    run_grid(bs_grid(n), block, blocks)
    return call, put


# ---------------------------------------------------------------- 2-D stencil
def stencil_grid(h, w):
    return (cdiv(w, STENCIL_BX), cdiv(h, STENCIL_BY), 1)


def stencil2d(field, blocks=None):
    """One 5-point Jacobi sweep of an HxW field:
       out[i][j] = (in[i-1][j] + in[i+1][j] + in[i][j-1] + in[i][j+1]) / 4
    on the interior; boundary points (Dirichlet) are copied."""
    h, w = field.shape
    f = field.astype(np.float64)
    out = np.zeros((h, w), dtype=np.float64)

    def block(x, y, z):
        i0, i1 = y * STENCIL_BY, min((y + 1) * STENCIL_BY, h)
        j0, j1 = x * STENCIL_BX, min((x + 1) * STENCIL_BX, w)
        i = np.arange(i0, i1)[:, None]
        j = np.arange(j0, j1)[None, :]
        boundary = (i == 0) | (j == 0) | (i == h - 1) | (j == w - 1)
        if h < 3 or w < 3:      # every point is a boundary point
            out[i0:i1, j0:j1] = f[i0:i1, j0:j1]
            return
        ic, jc = np.clip(i, 1, h - 2), np.clip(j, 1, w - 2)   # neighbour indices, valid for interior points
        interior = 0.25 * (f[ic - 1, jc] + f[ic + 1, jc] + f[ic, jc - 1] + f[ic, jc + 1])
        out[i0:i1, j0:j1] = np.where(boundary, f[i0:i1, j0:j1], interior)

    run_grid(stencil_grid(h, w), block, blocks)
    return out


# ---------------------------------------------------------------- bf16 GEMM
def bf16_to_f64(bits):
    """bfloat16 bit patterns (uint16) -> float64.  A bf16 value is the float32
    whose upper 16 bits are the pattern and whose lower 16 bits are zero."""
    return (bits.astype(np.uint32) << np.uint32(16)).view(np.float32).astype(np.float64)


def gemm_grid(m, n):
    return (cdiv(n, GEMM_TILE), cdiv(m, GEMM_TILE), 1)


def gemm_bf16_tile(A_bits, B_bits, x, y):
    """One 128x128 output tile (x = column tile, y = row tile) of C = A @ B^T."""
    m, _ = A_bits.shape
    n, _ = B_bits.shape
    r0, r1 = y * GEMM_TILE, min((y + 1) * GEMM_TILE, m)
    c0, c1 = x * GEMM_TILE, min((x + 1) * GEMM_TILE, n)
    return bf16_to_f64(A_bits[r0:r1]) @ bf16_to_f64(B_bits[c0:c1]).T


def gemm_bf16(A_bits, B_bits, blocks=None):
    """C[m][n] = sum_k A[m][k] * B[n][k], inputs bf16 widened exactly, summed in double."""
    m, k = A_bits.shape
    n, k2 = B_bits.shape
    assert k == k2
    C = np.zeros((m, n), dtype=np.float64)

    def block(x, y, z):
        r0, c0 = y * GEMM_TILE, x * GEMM_TILE
        t = gemm_bf16_tile(A_bits, B_bits, x, y)
        C[r0:r0 + t.shape[0], c0:c0 + t.shape[1]] = t

    run_grid(gemm_grid(m, n), block, blocks)
    return C


# ---------------------------------------------------------------- probe3d (a 3-D grid of 3-D blocks)
# The user kernel of the NEXT-3 / 3-D-grid parity test (tests/test_user_kernels.py):
#   i = blockIdx.x*blockDim.x + threadIdx.x (and j, k on y, z); inside the field
#   out[k][j][i] = 2*in[k][j][i] + (blockIdx.x + 3*blockIdx.y + 7*blockIdx.z)
# so every element records which original block wrote it: the block's (x,y,z)
# comes from decode() of its linear index (reading Q18 for z), the
# threads of a block are enumerated x-fastest (CUDA's threadIdx order).
def probe3d_grid(shape, block):
    nz, ny, nx = shape
    bx, by, bz = block
    return (cdiv(nx, bx), cdiv(ny, by), cdiv(nz, bz))


def probe3d(inp, block, blocks=None):
    nz, ny, nx = inp.shape
    bx, by, bz = block
    out = np.zeros(inp.shape, dtype=np.float64)
    src = inp.astype(np.float64)

    def body(x, y, z):
        for tz in range(bz):
            for ty in range(by):
                for tx in range(bx):
                    i, j, k = x * bx + tx, y * by + ty, z * bz + tz
                    if i < nx and j < ny and k < nz:
                        out[k, j, i] = 2.0 * src[k, j, i] + (x + 3 * y + 7 * z)

    run_grid(probe3d_grid(inp.shape, block), body, blocks)
    return out


# ---------------------------------------------------------------- coverage
def expected_counters(total_blocks, iters):
    """Deterministic counters of one complete slate launch.

    Every original block runs exactly once (P:L79 isomorphism; P:L127 progress
    carried in slateIdx), tasks are ``iters`` consecutive blocks, so
    the task starts are 0, iters, 2*iters, ... < B and the last task is clamped
    (P:L210).  ``next_clamped`` is the counter value once every task start has
    been handed out, clamped to the first start >= B.
    """
    tasks = cdiv(total_blocks, iters)
    return {
        "coverage": np.ones(total_blocks, dtype=np.uint32),
        "blocks_done": total_blocks,
        "tasks_done": tasks,
        "task_starts": list(range(0, total_blocks, iters)),
        "next_clamped": tasks * iters,
    }


# ================================================================ the paper's own workload (Tab II)
# NEXT-2: the five applications of Tab II ("from the
# NVIDIA CUDA 8.0 samples and the Rodinia benchmark suite") as tenants.
# Black-Scholes (BS) is ``blackscholes`` above with one scenario (P = 1, the
# SDK kernel).  The other four follow.  Readings (Q33-Q36): TR is the
# SDK's tiled transpose, MM the SDK's shared-memory tiled matrixMul, RG the
# SDK's quasirandomGenerator kernel (the Niederreiter-style XOR generator, the
# inverse-CND pass not included), GS Rodinia's Gaussian elimination as its two
# kernels Fan1 (multipliers of column t) and Fan2 (rank-1 update of the
# trailing rows), one pair of launches per elimination step t.

TR_TILE = 32          # 32x32 input tile per block
MM_TILE = 32          # 32x32 C tile per block
QRNG_E = 1024         # points per block (one dimension)
QRNG_BITS = 31        # QRNG_RESOLUTION of the SDK sample
GS_FAN1_E = 256       # rows per Fan1 block
GS_FAN2_R, GS_FAN2_C = 16, 128   # rows x columns of the trailing submatrix per Fan2 block


# ---------------------------------------------------------------- TR: transpose
def transpose_grid(h, w):
    return (cdiv(w, TR_TILE), cdiv(h, TR_TILE), 1)


def transpose(inp, blocks=None):
    """out[j][i] = in[i][j]; ``inp`` is h x w row-major, the output w x h.
    Block (x, y) moves the input tile rows 32y.., columns 32x.."""
    h, w = inp.shape
    out = np.zeros((w, h), dtype=inp.dtype)

    def block(x, y, z):
        r0, r1 = y * TR_TILE, min((y + 1) * TR_TILE, h)
        c0, c1 = x * TR_TILE, min((x + 1) * TR_TILE, w)
        for i in range(r0, r1):
            out[c0:c1, i] = inp[i, c0:c1]

    run_grid(transpose_grid(h, w), block, blocks)
    return out


# ---------------------------------------------------------------- MM: tiled SGEMM
def sgemm_tiled_grid(m, n):
    return (cdiv(n, MM_TILE), cdiv(m, MM_TILE), 1)


def sgemm_tiled(A, B, blocks=None):
    """C = A @ B (A m x k, B k x n, row-major), the SDK matrixMul: block (x, y)
    owns the 32x32 C tile rows 32y.., columns 32x..; every C element is the dot
    product of its row of A and column of B (k ascending; summed here in double)."""
    m, k = A.shape
    k2, n = B.shape
    assert k == k2
    A64 = A.astype(np.float64)
    B64 = B.astype(np.float64)
    C = np.zeros((m, n), dtype=np.float64)

    def block(x, y, z):
        r0, r1 = y * MM_TILE, min((y + 1) * MM_TILE, m)
        c0, c1 = x * MM_TILE, min((x + 1) * MM_TILE, n)
        for r in range(r0, r1):
            for c in range(c0, c1):
                C[r, c] = float(np.dot(A64[r, :], B64[:, c]))

    run_grid(sgemm_tiled_grid(m, n), block, blocks)
    return C


# ---------------------------------------------------------------- RG: quasirandom generator
def qrng_grid(n, dims):
    return (cdiv(n, QRNG_E), dims, 1)


def qrng_point(table_row, k):
    """q(k) = XOR of table_row[b] over the set bits b < 31 of k (the generator
    matrix applied to the binary digits of k over GF(2))."""
    r = 0
    for b in range(QRNG_BITS):
        if (k >> b) & 1:
            r ^= int(table_row[b])
    return r


def qrng(table, n, seed, blocks=None):
    """out[d][i] = float32(q_d(seed + i) + 1) * 2^-31 for i < n, d < dims: the
    SDK kernel's ``(float)(result + 1) * INT_SCALE`` (INT_SCALE = 2^-31, the
    float nearest 1/0x80000001).  ``table`` is dims x 31 uint32 (< 2^31).  The
    integer -> float conversion rounds to nearest (fp32, as the kernel does);
    the scaling by a power of two is exact.  Block (x, d) makes points
    1024x .. of dimension d."""
    dims = table.shape[0]
    out = np.zeros((dims, n), dtype=np.float32)

    def block(x, d, z):
        for i in range(x * QRNG_E, min((x + 1) * QRNG_E, n)):
            q = qrng_point(table[d], (seed + i) & 0xFFFFFFFF)
            out[d, i] = np.float32(q + 1) * np.float32(2.0 ** -31)

    run_grid(qrng_grid(n, dims), block, blocks)
    return out


# ---------------------------------------------------------------- GS: Gaussian elimination
def gauss_fan1_grid(n, t):
    return (max(cdiv(n - 1 - t, GS_FAN1_E), 1), 1, 1)


def gauss_fan2_grid(n, t):
    return (max(cdiv(n - t, GS_FAN2_C), 1), max(cdiv(n - 1 - t, GS_FAN2_R), 1), 1)


def gauss_fan1(a, m, t, blocks=None):
    """Rodinia Fan1 at step t: m[i][t] = a[i][t] / a[t][t] for rows i = t+1 .. n-1.
    ``a`` and ``m`` are n x n float64 arrays, ``m`` updated in place."""
    n = a.shape[0]

    def block(x, y, z):
        for i in range(t + 1 + x * GS_FAN1_E, min(t + 1 + (x + 1) * GS_FAN1_E, n)):
            m[i, t] = a[i, t] / a[t, t]

    run_grid(gauss_fan1_grid(n, t), block, blocks)


def gauss_fan2(a, b, m, t, blocks=None):
    """Rodinia Fan2 at step t: a[i][j] -= m[i][t] * a[t][j] for rows i = t+1 .. n-1
    and columns j = t .. n-1 (column t included: it becomes ~0), and
    b[i] -= m[i][t] * b[t].  In place on float64 arrays.  Block (x, y) owns rows
    t+1+16y .., columns t+128x ..; the blocks with x = 0 update b."""
    n = a.shape[0]

    def block(x, y, z):
        r0, r1 = t + 1 + y * GS_FAN2_R, min(t + 1 + (y + 1) * GS_FAN2_R, n)
        c0, c1 = t + x * GS_FAN2_C, min(t + (x + 1) * GS_FAN2_C, n)
        for i in range(r0, r1):
            a[i, c0:c1] -= m[i, t] * a[t, c0:c1]
            if x == 0:
                b[i] -= m[i, t] * b[t]

    run_grid(gauss_fan2_grid(n, t), block, blocks)


def gaussian(a, b, steps=None):
    """Forward elimination without pivoting (Rodinia ``ForwardSub``): for
    t = 0 .. n-2, Fan1 then Fan2.  Returns (a, b, m) in float64: a upper
    triangular below the diagonal up to rounding (column entries ~0), m the
    unit-lower factor's multipliers below the diagonal (zero elsewhere)."""
    n = a.shape[0]
    a = a.astype(np.float64).copy()
    b = b.astype(np.float64).copy()
    m = np.zeros((n, n), dtype=np.float64)
    for t in range(n - 1 if steps is None else steps):
        gauss_fan1(a, m, t)
        gauss_fan2(a, b, m, t)
    return a, b, m
