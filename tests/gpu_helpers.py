"""Shared helpers for the -m gpu tests: tenant setup on the device, the
tolerance rule (reading Q17) and oracle comparisons.  Inputs come from
paper_conf_ipps_allenf019_b200.inputs (seeded); expected values from oracle/."""
import numpy as np
import torch

from oracle import tenants as OT
from paper_conf_ipps_allenf019_b200 import inputs as I
from paper_conf_ipps_allenf019_b200 import slate as S

DEV = "cuda:0"


def within(g, o, scale, rel=1e-5):
    """Q17: |g - o| <= rel * max(|o|, scale) element-wise (north star: 1e-5 relative)."""
    g = np.asarray(g, dtype=np.float64)
    o = np.asarray(o, dtype=np.float64)
    bound = rel * np.maximum(np.abs(o), scale)
    bad = np.abs(g - o) > bound
    return (not bad.any()), (float(np.max(np.abs(g - o) / np.maximum(bound, 1e-300))) if g.size else 0.0)


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


class Tenant:
    """A tenant instance: device buffers, args, grid, and the oracle check."""

    def __init__(self, kind, args, grid, outputs, check, keep, initial=None):
        self.kind, self.args, self.grid, self.outputs, self.check, self._keep = kind, args, grid, outputs, check, keep
        # in-place tenants (GS Fan2 updates a and b): every run restarts from these
        self._initial = None if initial is None else [t.clone() for t in initial]
        torch.cuda.synchronize()   # inputs are written on torch's stream; the server's streams do not wait

    def zero_outputs(self):
        for i, t in enumerate(self.outputs):
            if self._initial is None:
                t.zero_()
            else:
                t.copy_(self._initial[i])
        torch.cuda.synchronize()

    def snapshot(self):
        return [t.clone() for t in self.outputs]


def make_triad(n, seed, mode="float"):
    b, c, s = I.triad_inputs(n, seed, mode)
    a_d, b_d, c_d = torch.zeros(n, device=DEV), dev(b), dev(c)
    args, grid = S.triad_args(a_d, b_d, c_d, s)

    def check(outs, rows=None):
        ref = OT.triad(b, c, s)
        g = outs[0].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(g, ref), 0.0
        return within(g, ref, np.abs(b) + abs(float(s)) * np.abs(c))

    return Tenant(S.KIND_TRIAD, args, grid, [a_d], check, (b_d, c_d))


def make_copy(n, seed):
    b = I.copy_inputs(n, seed)
    a_d, b_d = torch.zeros(n, device=DEV), dev(b)
    args, grid = S.copy_args(a_d, b_d)

    def check(outs, rows=None):
        return outs[0].cpu().numpy().tobytes() == OT.copy(b).tobytes(), 0.0

    return Tenant(S.KIND_COPY, args, grid, [a_d], check, (b_d,))


def make_sgemm(m, n, k, seed, mode="float"):
    A, B = I.sgemm_inputs(m, n, k, seed, mode)
    A_d, B_d, C_d = dev(A), dev(B), torch.zeros(m, n, device=DEV)
    args, grid = S.sgemm_args(A_d, B_d, C_d)

    def check(outs, rows=None):
        ref = OT.sgemm_naive(A, B)
        g = outs[0].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(g, ref), 0.0
        return within(g, ref, np.abs(A.astype(np.float64)) @ np.abs(B.astype(np.float64)))

    return Tenant(S.KIND_SGEMM_NAIVE, args, grid, [C_d], check, (A_d, B_d))


def make_spmv(n_rows, seed, mode="float", band=4096, ragged=None):
    if ragged is None:
        rp, col, val, x = I.spmv_inputs(n_rows, seed, mode, band=band)
    else:
        rp, col, val, x = I.spmv_ragged_inputs(n_rows, seed, mode, band=band, **ragged)
    rp_d, col_d, val_d, x_d = dev(rp), dev(col), dev(val), dev(x)
    y_d = torch.zeros(n_rows, device=DEV)
    args, grid = S.spmv_args(rp_d, col_d, val_d, x_d, y_d)

    def check(outs, rows=None):
        ref = OT.spmv_csr(rp, col, val, x)
        g = outs[0].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(g, ref), 0.0
        scale = OT.spmv_csr(rp, col, np.abs(val), np.abs(x))
        return within(g, ref, scale)

    return Tenant(S.KIND_SPMV_CSR, args, grid, [y_d], check, (rp_d, col_d, val_d, x_d))


def make_bs(n, seed, n_scen=4):
    Sx, X, T, r = I.bs_inputs(n, seed)
    sig = I.bs_sigmas(n_scen)
    S_d, X_d, T_d, sig_d = dev(Sx), dev(X), dev(T), dev(sig)
    call_d, put_d = torch.zeros(n, device=DEV), torch.zeros(n, device=DEV)
    args, grid = S.bs_args(S_d, X_d, T_d, call_d, put_d, sig_d, r)

    def check(outs, rows=None):
        c_ref, p_ref = OT.blackscholes(Sx, X, T, r, sig)
        ok1, e1 = within(outs[0].cpu().numpy(), c_ref, Sx.astype(np.float64))
        ok2, e2 = within(outs[1].cpu().numpy(), p_ref, Sx.astype(np.float64))
        return ok1 and ok2, max(e1, e2)

    return Tenant(S.KIND_BLACKSCHOLES, args, grid, [call_d, put_d], check, (S_d, X_d, T_d, sig_d))


def make_stencil(h, w, seed, mode="float"):
    f = I.stencil_inputs(h, w, seed, mode)
    in_d, out_d = dev(f), torch.zeros(h, w, device=DEV)
    args, grid = S.stencil_args(in_d, out_d)

    def check(outs, rows=None):
        ref = OT.stencil2d(f)
        g = outs[0].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(g, ref), 0.0
        return within(g, ref, float(np.abs(f).max()))

    return Tenant(S.KIND_STENCIL2D, args, grid, [out_d], check, (in_d,))


def make_gemm(m, n, k, seed, mode="float"):
    A, B = I.gemm_inputs(m, n, k, seed, mode)
    A_d = torch.from_numpy(A.view(np.int16)).to(DEV)
    B_d = torch.from_numpy(B.view(np.int16)).to(DEV)
    C_d = torch.zeros(m, n, device=DEV)
    args, grid = S.gemm_args(A_d, B_d, C_d)

    def check(outs, rows=None):
        C = outs[0].cpu().numpy().astype(np.float64)
        if rows is None:
            ref = OT.gemm_bf16(A, B)
            if mode == "int":
                return np.array_equal(C, ref), 0.0
            return within(C, ref, np.abs(OT.bf16_to_f64(A)) @ np.abs(OT.bf16_to_f64(B)).T)
        # sampled 128 x 128 tiles (x, y) at full size (the oracle's tiling, independent of the kernel's)
        worst, ok = 0.0, True
        for (x, y) in rows:
            ref = OT.gemm_bf16_tile(A, B, x, y)
            g = C[y * 128:(y + 1) * 128, x * 128:(x + 1) * 128]
            if mode == "int":
                ok &= np.array_equal(g, ref)
            else:
                scale = np.abs(OT.bf16_to_f64(A[y * 128:(y + 1) * 128])) @ np.abs(OT.bf16_to_f64(B[x * 128:(x + 1) * 128])).T
                o, e = within(g, ref, scale)
                ok &= o
                worst = max(worst, e)
        return ok, worst

    return Tenant(S.KIND_GEMM_BF16, args, grid, [C_d], check, (A_d, B_d))


# ------------------------------------------------------------------ the paper's Tab II apps (NEXT-2)
def make_transpose(h, w, seed):
    A = I.transpose_inputs(h, w, seed)
    in_d, out_d = dev(A), torch.zeros(w, h, device=DEV)
    args, grid = S.transpose_args(in_d, out_d)

    def check(outs, rows=None):
        return outs[0].cpu().numpy().tobytes() == OT.transpose(A).tobytes(), 0.0

    return Tenant(S.KIND_TRANSPOSE, args, grid, [out_d], check, (in_d,))


def make_sgemm_tiled(m, n, k, seed, mode="float"):
    A, B = I.sgemm_inputs(m, n, k, seed, mode)
    A_d, B_d, C_d = dev(A), dev(B), torch.zeros(m, n, device=DEV)
    args, grid = S.sgemm_tiled_args(A_d, B_d, C_d)

    def check(outs, rows=None):
        ref = OT.sgemm_tiled(A, B)
        g = outs[0].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(g, ref), 0.0
        return within(g, ref, np.abs(A.astype(np.float64)) @ np.abs(B.astype(np.float64)))

    return Tenant(S.KIND_SGEMM_TILED, args, grid, [C_d], check, (A_d, B_d))


def make_qrng(n, dims, seed, qseed=0):
    table = I.qrng_table(dims, seed)
    t_d = dev(table.view(np.int32))
    out_d = torch.zeros(dims, n, device=DEV)
    args, grid = S.qrng_args(t_d, out_d, qseed)

    def check(outs, rows=None):
        return np.array_equal(outs[0].cpu().numpy(), OT.qrng(table, n, qseed)), 0.0

    return Tenant(S.KIND_QRNG, args, grid, [out_d], check, (t_d,))


def gauss_state(n, t, seed, mode):
    """The system after t elimination steps of the oracle, as fp32 inputs (exact
    in int mode), and the oracle's multipliers of column t (Fan1 of step t)."""
    a0, b0 = I.gauss_inputs(n, seed, mode)
    a, b, m = OT.gaussian(a0, b0, steps=t)
    return a.astype(np.float32), b.astype(np.float32), m.astype(np.float32)


def make_gauss_fan1(n, t, seed, mode="int"):
    a, b, m = gauss_state(n, t, seed, mode)
    a_d, b_d, m_d = dev(a), dev(b), torch.zeros(n, n, device=DEV)
    args, grid = S.gauss_fan1_args(a_d, b_d, m_d, t)

    def check(outs, rows=None):
        ref = np.zeros((n, n))
        OT.gauss_fan1(a.astype(np.float64), ref, t)
        g = outs[0].cpu().numpy().astype(np.float64)
        # fp32 division is correctly rounded; so is the fp64 quotient rounded to fp32
        return np.array_equal(g, ref.astype(np.float32).astype(np.float64)), 0.0

    return Tenant(S.KIND_GAUSS_FAN1, args, grid, [m_d], check, (a_d, b_d))


def make_gauss_fan2(n, t, seed, mode="int"):
    a, b, m = gauss_state(n, t, seed, mode)
    mt = np.zeros((n, n))
    OT.gauss_fan1(a.astype(np.float64), mt, t)
    m[:, t] = mt[:, t].astype(np.float32)
    a_d, b_d, m_d = dev(a), dev(b), dev(m)
    args, grid = S.gauss_fan2_args(a_d, b_d, m_d, t)

    def check(outs, rows=None):
        ra, rb = a.astype(np.float64), b.astype(np.float64)
        OT.gauss_fan2(ra, rb, m.astype(np.float64), t)
        ga = outs[0].cpu().numpy().astype(np.float64)
        gb = outs[1].cpu().numpy().astype(np.float64)
        if mode == "int":
            return np.array_equal(ga, ra) and np.array_equal(gb, rb), 0.0
        # one fmaf per element: Q17 with scale |a| + |m p|
        m64 = m[:, t].astype(np.float64)
        sa = np.abs(a.astype(np.float64)) + np.abs(m64)[:, None] * np.abs(a[t].astype(np.float64))[None, :]
        sb = np.abs(b.astype(np.float64)) + np.abs(m64) * abs(float(b[t]))
        ok1, e1 = within(ga, ra, sa)
        ok2, e2 = within(gb, rb, sb)
        return ok1 and ok2, max(e1, e2)

    return Tenant(S.KIND_GAUSS_FAN2, args, grid, [a_d, b_d], check, (m_d,), initial=[a_d, b_d])
