"""Thin ctypes binding of libslate (include/slate.h) -- argument marshalling only.

Every step of the slate path runs in the CUDA library; this module only packs
C structs and raises on error status.  PyTorch tensors may be passed wherever a
device pointer is expected (their ``data_ptr()`` is used); torch is plumbing.
There is no fallback: if ``libslate.so`` is missing, importing this module
raises.
"""
import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("SLATE_LIB", os.path.join(_PKG, "libslate.so"))
if not os.path.exists(_LIB_PATH):
    raise ImportError("libslate.so not built (run `python -m paper_conf_ipps_allenf019_b200.build`): %s" % _LIB_PATH)
_lib = ctypes.CDLL(_LIB_PATH)
LIB_PATH = _LIB_PATH

c_u32, c_u64, c_i32, c_i64, c_f32, c_f64 = (ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32, ctypes.c_int64,
                                            ctypes.c_float, ctypes.c_double)

ABI_VERSION = 1
OK, DONE = 0, 1
EINVAL, ENOMEM, ECUDA, EIPC, ETIMEDOUT, ENOTFOUND, ESTATE, EUNSUPPORTED = -1, -2, -3, -4, -5, -6, -7, -8

KIND_TRIAD, KIND_COPY, KIND_SGEMM_NAIVE, KIND_SPMV_CSR, KIND_BLACKSCHOLES, KIND_STENCIL2D, KIND_GEMM_BF16 = range(1, 8)
# the paper's Tab II apps (TR, MM, RG, GS = Fan1 + Fan2; BS is KIND_BLACKSCHOLES with one scenario)
KIND_TRANSPOSE, KIND_SGEMM_TILED, KIND_QRNG, KIND_GAUSS_FAN1, KIND_GAUSS_FAN2 = range(8, 13)
KIND_USER = 13   # a user kernel compiled at run time (register_source, NEXT-3)
KFLAG_COVERAGE = 1
KFLAG_RANKLOG = 2   # with KFLAG_COVERAGE: the coverage log is u32[2B], cov[B + b] = who took block b (slate.h)
PLACE_AUTO, PLACE_SOLO, PLACE_CORUN = 0, 1, 2
MODE_SLATE, MODE_STANDALONE = 0, 1
PROF_CURVE, PROF_FORCE = 1, 2
CATEGORIES = ("L_C", "M_C", "H_C", "M_M", "H_M")


class SlateError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__("%s: %s" % (status_string(status), msg))
        self.status = status


# ------------------------------------------------------------------ structs
class ArgsTriad(ctypes.Structure):
    _fields_ = [("a", c_u64), ("b", c_u64), ("c", c_u64), ("n", c_u64), ("s", c_f32), ("pad_", c_u32)]


class ArgsCopy(ctypes.Structure):
    _fields_ = [("a", c_u64), ("b", c_u64), ("n", c_u64)]


class ArgsSgemm(ctypes.Structure):
    _fields_ = [("A", c_u64), ("B", c_u64), ("C", c_u64), ("m", c_u32), ("n", c_u32), ("k", c_u32), ("pad_", c_u32)]


class ArgsSpmv(ctypes.Structure):
    _fields_ = [("rowptr", c_u64), ("col", c_u64), ("val", c_u64), ("x", c_u64), ("y", c_u64),
                ("n_rows", c_u32), ("n_cols", c_u32)]


class ArgsBS(ctypes.Structure):
    _fields_ = [("S", c_u64), ("X", c_u64), ("T", c_u64), ("call", c_u64), ("put", c_u64), ("sigmas", c_u64),
                ("n", c_u64), ("r", c_f32), ("n_scen", c_u32)]


class ArgsStencil(ctypes.Structure):
    _fields_ = [("inp", c_u64), ("out", c_u64), ("h", c_u32), ("w", c_u32)]


class ArgsGemm(ctypes.Structure):
    _fields_ = [("A", c_u64), ("B", c_u64), ("C", c_u64), ("m", c_u32), ("n", c_u32), ("k", c_u32), ("pad_", c_u32)]


class ArgsTranspose(ctypes.Structure):
    _fields_ = [("inp", c_u64), ("out", c_u64), ("h", c_u32), ("w", c_u32)]


class ArgsQrng(ctypes.Structure):
    _fields_ = [("table", c_u64), ("out", c_u64), ("n", c_u32), ("dims", c_u32), ("seed", c_u32), ("pad_", c_u32)]


class ArgsGauss(ctypes.Structure):
    _fields_ = [("a", c_u64), ("b", c_u64), ("m", c_u64), ("n", c_u32), ("t", c_u32)]


class SourceDesc(ctypes.Structure):
    _fields_ = [("abi_version", c_u32), ("block_threads", c_u32), ("smem_bytes", c_u32), ("args_size", c_u32),
                ("iters", c_u32), ("flags", c_u32), ("source", ctypes.c_char_p), ("kernel_name", ctypes.c_char_p),
                ("bytes_per_block", c_f64), ("flops_per_block", c_f64), ("block_y", c_u32), ("block_z", c_u32)]


class Info(ctypes.Structure):
    _fields_ = [("abi_version", c_u32), ("num_sms", c_u32), ("max_smid", c_u32), ("device", c_u32),
                ("server_pid", c_u64), ("peak_hbm_gbps", c_f64), ("peak_fp32_gflops", c_f64),
                ("peak_tc_tflops", c_f64)]


class KernelDesc(ctypes.Structure):
    _fields_ = [("abi_version", c_u32), ("kind", c_u32), ("iters", c_u32), ("flags", c_u32)]


class LaunchDesc(ctypes.Structure):
    _fields_ = [("grid", c_u32 * 3), ("placement", c_u32), ("sm_lo", c_u32), ("sm_hi", c_u32), ("mode", c_u32),
                ("args_size", c_u32), ("args", ctypes.c_void_p), ("coverage", c_u64)]


class Profile(ctypes.Structure):
    _fields_ = [("solo_ms", c_f64), ("hbm_gbps", c_f64), ("fp32_gflops", c_f64), ("tc_tflops", c_f64),
                ("hbm_frac", c_f64), ("fp32_frac", c_f64), ("tc_frac", c_f64), ("c_level", c_u32),
                ("m_level", c_u32), ("category", c_u32), ("n_curve", c_u32), ("curve_sms", c_u32 * 8),
                ("curve_ms", c_f64 * 8), ("bytes", c_f64), ("flops", c_f64)]

    def as_dict(self):
        d = {f[0]: getattr(self, f[0]) for f in self._fields_}
        d["curve_sms"] = list(self.curve_sms)[:self.n_curve]
        d["curve_ms"] = list(self.curve_ms)[:self.n_curve]
        d["category_name"] = CATEGORIES[self.category]
        return d


class LaunchInfo(ctypes.Structure):
    _fields_ = [("state", c_u32), ("blocks_done", c_u32), ("tasks_done", c_u32), ("total_blocks", c_u32),
                ("next_clamped", c_u32), ("next_raw", c_u32), ("live_workers", c_u32), ("iters", c_u32),
                ("sm_lo", c_u32), ("sm_hi", c_u32), ("n_resizes", c_u32), ("n_topups", c_u32),
                ("workers_started", c_u32), ("coverage_ok", c_u32), ("epoch", c_u32), ("shrink_epoch", c_u32),
                ("join_epoch", c_u32), ("pad_", c_u32), ("t_first_ns", c_u64), ("t_last_ns", c_u64),
                ("start_ms", c_f64), ("end_ms", c_f64), ("resize_us", c_f64 * 16), ("resize_kind", ctypes.c_uint8 * 16),
                ("t_enter_ns", c_u64), ("t_exit_ns", c_u64), ("n_superseded", c_u32), ("pad2_", c_u32)]

    def as_dict(self):
        d = {f[0]: getattr(self, f[0]) for f in self._fields_}
        d["resize_us"] = [v for v in self.resize_us if v >= 0]
        d["resize_kind"] = [("shrink", "grow")[k - 1] for v, k in zip(self.resize_us, self.resize_kind)
                            if v >= 0 and k in (1, 2)]
        return d


# ------------------------------------------------------------------ prototypes
_P = ctypes.POINTER
_lib.slate_status_string.restype = ctypes.c_char_p
_lib.slate_status_string.argtypes = [c_i32]
_lib.slate_last_error.restype = ctypes.c_char_p
_lib.slate_last_error.argtypes = [ctypes.c_void_p]
for _name, _args in [
    ("slate_attach", [ctypes.c_char_p, ctypes.c_int, _P(ctypes.c_void_p)]),
    ("slate_detach", [ctypes.c_void_p]),
    ("slate_get_info", [ctypes.c_void_p, _P(Info)]),
    ("slate_share_buffer", [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, _P(c_u64)]),
    ("slate_unshare_buffer", [ctypes.c_void_p, c_u64]),
    ("slate_register_kernel", [ctypes.c_void_p, _P(KernelDesc), _P(c_u64)]),
    ("slate_launch", [ctypes.c_void_p, c_u64, _P(LaunchDesc), _P(c_u64)]),
    ("slate_resize", [ctypes.c_void_p, c_u64, c_u32, c_u32]),
    ("slate_sync", [ctypes.c_void_p, c_u64, c_i64]),
    ("slate_profile", [ctypes.c_void_p, c_u64, _P(LaunchDesc), c_u32, _P(Profile)]),
    ("slate_query", [ctypes.c_void_p, c_u64, _P(LaunchInfo)]),
    ("slate_serve", [ctypes.c_char_p, ctypes.c_int, c_u32]),
    ("slate_kind_geometry", [c_u32, _P(c_u32), _P(c_u32)]),
    ("slate_set_policy", [ctypes.c_void_p, c_u32]),
    ("slate_launch_n", [ctypes.c_void_p, c_u64, _P(LaunchDesc), c_u32, _P(c_u64)]),
    ("slate_launch_many", [ctypes.c_void_p, c_u32, _P(c_u64), _P(LaunchDesc), _P(c_u64)]),
    ("slate_register_source", [ctypes.c_void_p, _P(SourceDesc), _P(c_u64)]),
    ("slate_transform_source", [ctypes.c_char_p, ctypes.c_char_p, c_u32, c_u32, c_u32, c_u32, ctypes.c_char_p,
                                ctypes.c_size_t, _P(ctypes.c_size_t)]),
]:
    getattr(_lib, _name).restype = c_i32
    getattr(_lib, _name).argtypes = _args
_lib.slate_classify.restype = c_u32
_lib.slate_classify.argtypes = [c_f64, c_f64, c_f64, _P(c_u32), _P(c_u32)]
_lib.slate_policy.restype = ctypes.c_int
_lib.slate_policy.argtypes = [c_u32, c_u32, ctypes.c_int]
_lib.slate_select.restype = ctypes.c_int
_lib.slate_select.argtypes = [c_u32, _P(c_u32), _P(c_u32), c_u32, c_u32, ctypes.c_int]
_lib.slate_choose_split.restype = c_u32
_lib.slate_choose_split.argtypes = [_P(c_u32), _P(c_f64), c_u32, _P(c_u32), _P(c_f64), c_u32, c_u32, c_u32, c_u32,
                                    c_u32, _P(c_f64)]
_lib.slate_saturation_sms.restype = c_u32
_lib.slate_saturation_sms.argtypes = [_P(c_u32), _P(c_f64), c_u32, c_u32, c_f64]
_lib.slate_corun_makespan_k.restype = c_f64
_lib.slate_corun_makespan_k.argtypes = [ctypes.c_void_p, ctypes.c_void_p, _P(c_u32), c_u32, _P(c_u32)]
_lib.slate_choose_split_k.restype = c_f64
_lib.slate_choose_split_k.argtypes = [ctypes.c_void_p, ctypes.c_void_p, _P(c_u32), c_u32, c_u32, c_u32, _P(c_u32)]
_lib.slate_kway_admit.restype = ctypes.c_int
_lib.slate_kway_admit.argtypes = [ctypes.c_void_p, ctypes.c_void_p, _P(c_u32), _P(c_u32), c_u32, _P(c_u32), c_u32, c_u32,
                                  c_f64, _P(c_u32), _P(c_f64)]
_lib.slate_choose_iters.restype = c_u32
_lib.slate_choose_iters.argtypes = [c_f64, c_u32, c_u32, c_u32, c_u32, c_f64]
_lib.slate_choose_split_obj.restype = c_u32
_lib.slate_choose_split_obj.argtypes = [_P(c_u32), _P(c_f64), c_u32, _P(c_u32), _P(c_f64), c_u32, c_u32, c_u32, c_u32,
                                        c_u32, c_u32, c_f64, _P(c_f64), _P(c_f64)]
_lib.slate_fluid_corun_obj.restype = ctypes.c_int
_lib.slate_fluid_corun_obj.argtypes = [_P(c_u32), _P(c_f64), c_u32, c_f64, _P(c_u32), _P(c_f64), c_u32, c_f64, c_u32,
                                       c_u32, c_u32, c_u32, c_f64, c_u32, c_f64, _P(c_u32), _P(c_f64)]
_lib.slate_launch_fused.restype = c_i32
_lib.slate_launch_fused.argtypes = [ctypes.c_void_p, c_u64, ctypes.c_void_p, ctypes.c_void_p, c_u64, ctypes.c_void_p,
                                    c_u32, _P(c_u64), _P(c_u64)]
_lib.slate_set_split_objective.restype = c_i32
_lib.slate_set_split_objective.argtypes = [ctypes.c_void_p, c_u32, c_f64]
_lib.slate_fluid_corun.restype = ctypes.c_int
_lib.slate_fluid_corun.argtypes = [_P(c_u32), _P(c_f64), c_u32, c_f64, _P(c_u32), _P(c_f64), c_u32, c_f64, c_u32,
                                   c_u32, c_u32, c_u32, c_f64, _P(c_u32), _P(c_f64)]
_lib.slate_rtc_stats.restype = None
_lib.slate_rtc_stats.argtypes = [_P(c_u64), _P(c_u64), _P(c_u64)]
POLICY_TABLE, POLICY_LITERAL, POLICY_HYBRID = 0, 1, 2

EXPORTED = ["slate_attach", "slate_detach", "slate_get_info", "slate_share_buffer", "slate_unshare_buffer",
            "slate_register_kernel", "slate_launch", "slate_resize", "slate_sync", "slate_profile", "slate_query",
            "slate_status_string", "slate_last_error", "slate_classify", "slate_policy", "slate_select",
            "slate_choose_split", "slate_serve", "slate_kind_geometry", "slate_saturation_sms",
            "slate_fluid_corun", "slate_set_policy", "slate_launch_n", "slate_launch_many", "slate_choose_iters",
            "slate_register_source", "slate_transform_source", "slate_corun_makespan_k", "slate_choose_split_k",
            "slate_rtc_stats", "slate_choose_split_obj", "slate_fluid_corun_obj", "slate_set_split_objective", "slate_launch_fused", "slate_kway_admit"]
DAEMON = os.path.join(_PKG, "bin", "slated")


def status_string(st):
    return _lib.slate_status_string(st).decode()


def _ptr(x):
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    return int(x.data_ptr())


# ------------------------------------------------------------------ sessions
class Session:
    """One client session.  ``endpoint=None`` -> in-process server."""

    def __init__(self, endpoint=None, device=0):
        h = ctypes.c_void_p()
        st = _lib.slate_attach(endpoint.encode() if endpoint else None, device, ctypes.byref(h))
        if st != OK:
            raise SlateError(st, "slate_attach(%r, %d) failed" % (endpoint, device))
        self._h = h

    def _check(self, st, what):
        if st < 0:
            raise SlateError(st, "%s: %s" % (what, _lib.slate_last_error(self._h).decode()))
        return st

    def close(self):
        if self._h:
            st = _lib.slate_detach(self._h)
            self._h = None
            if st < 0:
                raise SlateError(st, "slate_detach")

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def info(self):
        i = Info()
        self._check(_lib.slate_get_info(self._h, ctypes.byref(i)), "slate_get_info")
        return {f[0]: getattr(i, f[0]) for f in Info._fields_}

    def share_buffer(self, t, nbytes=None):
        h = c_u64()
        nb = nbytes if nbytes is not None else t.numel() * t.element_size()
        self._check(_lib.slate_share_buffer(self._h, _ptr(t), nb, ctypes.byref(h)), "slate_share_buffer")
        return h.value

    def share_tensors(self, *tensors):
        return [self.share_buffer(t) for t in tensors]

    def unshare_buffer(self, handle):
        self._check(_lib.slate_unshare_buffer(self._h, handle), "slate_unshare_buffer")

    def register_source(self, source, name, args_struct, threads=256, smem=0, iters=0, bytes_per_block=0.0,
                        flops_per_block=0.0, flags=0, block=None):
        """A user CUDA kernel compiled at run time (NEXT-3); `args_struct` is the
        ctypes Structure type of its parameters, in declaration order; `block`
        an (x, y, z) block shape (default (threads, 1, 1))."""
        bx, by, bz = block if block is not None else (threads, 1, 1)
        d = SourceDesc(ABI_VERSION, bx, smem, ctypes.sizeof(args_struct), iters, flags, source.encode(), name.encode(),
                       bytes_per_block, flops_per_block, by, bz)
        k = c_u64()
        self._check(_lib.slate_register_source(self._h, ctypes.byref(d), ctypes.byref(k)), "slate_register_source")
        return k.value

    def register_kernel(self, kind, iters=0, flags=0):
        d = KernelDesc(ABI_VERSION, kind, iters, flags)
        k = c_u64()
        self._check(_lib.slate_register_kernel(self._h, ctypes.byref(d), ctypes.byref(k)), "slate_register_kernel")
        return k.value

    @staticmethod
    def _desc(args, grid, placement=PLACE_AUTO, sm=None, mode=MODE_SLATE, coverage=None):
        d = LaunchDesc()
        g = tuple(grid) + (1,) * (3 - len(grid))
        d.grid[0], d.grid[1], d.grid[2] = g
        d.placement = placement
        d.sm_lo, d.sm_hi = sm if sm is not None else (0, 0)
        d.mode = mode
        d.args_size = ctypes.sizeof(args)
        d.args = ctypes.cast(ctypes.pointer(args), ctypes.c_void_p)
        d.coverage = _ptr(coverage)
        return d

    def launch(self, kernel, args, grid, placement=PLACE_AUTO, sm=None, mode=MODE_SLATE, coverage=None):
        d = self._desc(args, grid, placement, sm, mode, coverage)
        lid = c_u64()
        self._check(_lib.slate_launch(self._h, kernel, ctypes.byref(d), ctypes.byref(lid)), "slate_launch")
        return lid.value

    def launch_n(self, kernel, args, grid, n, placement=PLACE_AUTO, sm=None, mode=MODE_SLATE, coverage=None):
        """n launches of one kernel as one job; returns their ids."""
        d = self._desc(args, grid, placement, sm, mode, coverage)
        first = c_u64()
        self._check(_lib.slate_launch_n(self._h, kernel, ctypes.byref(d), n, ctypes.byref(first)), "slate_launch_n")
        return list(range(first.value, first.value + n))

    def launch_many(self, items, placement=PLACE_AUTO, sm=None, mode=MODE_SLATE):
        """Launches [(kernel, args, grid), ...] in order as one job (one batch); returns their ids."""
        n = len(items)
        ks = (c_u64 * n)(*[k for k, _, _ in items])
        ds = (LaunchDesc * n)()
        for i, (_, args, grid) in enumerate(items):
            ds[i] = self._desc(args, grid, placement, sm, mode)
        first = c_u64()
        self._check(_lib.slate_launch_many(self._h, n, ks, ds, ctypes.byref(first)), "slate_launch_many")
        return list(range(first.value, first.value + n))

    def resize(self, launch_id, lo, hi):
        return self._check(_lib.slate_resize(self._h, launch_id, lo, hi), "slate_resize")

    def set_policy(self, policy):
        """Selector policy of the server (POLICY_TABLE / LITERAL / HYBRID; reading Q31)."""
        return self._check(_lib.slate_set_policy(self._h, policy), "slate_set_policy")

    def set_split_objective(self, objective="makespan", slack=0.05):
        """The split objective of the server's co-runs (reading Q41): "makespan" or "antt"."""
        return self._check(_lib.slate_set_split_objective(self._h, _OBJ[objective], slack), "slate_set_split_objective")

    def sync(self, launch_id=0, timeout_us=-1):
        return self._check(_lib.slate_sync(self._h, launch_id, timeout_us), "slate_sync")

    def profile(self, kernel, args, grid, flags=0):
        d = self._desc(args, grid)
        p = Profile()
        self._check(_lib.slate_profile(self._h, kernel, ctypes.byref(d), flags, ctypes.byref(p)), "slate_profile")
        return p.as_dict()

    def query(self, launch_id):
        i = LaunchInfo()
        self._check(_lib.slate_query(self._h, launch_id, ctypes.byref(i)), "slate_query")
        return i.as_dict()


# ------------------------------------------------------------------ host logic (no GPU)
def classify(hbm_frac, fp32_frac, tc_frac):
    c, m = c_u32(), c_u32()
    cat = _lib.slate_classify(hbm_frac, fp32_frac, tc_frac, ctypes.byref(c), ctypes.byref(m))
    return "LMH"[c.value], "LMH"[m.value], CATEGORIES[cat]


def policy(a, b, literal=False):
    return "corun" if _lib.slate_policy(CATEGORIES.index(a), CATEGORIES.index(b), int(literal)) else "solo"


def select(active, queue, bypassed=None, max_bypass=4, literal=False):
    n = len(queue)
    cats = (c_u32 * max(n, 1))(*[CATEGORIES.index(q) for q in queue])
    byp = (c_u32 * max(n, 1))(*(bypassed or [0] * n)) if bypassed is not None else None
    r = _lib.slate_select(CATEGORIES.index(active), cats, byp, n, max_bypass, int(literal))
    return None if r < 0 else r


def _curve(c):
    k = sorted(c)
    return (c_u32 * len(k))(*k), (c_f64 * len(k))(*[c[x] for x in k]), len(k)


SPLIT_MAKESPAN, SPLIT_ANTT = 0, 1
_OBJ = {"makespan": SPLIT_MAKESPAN, "antt": SPLIT_ANTT}


def choose_split(curve_a, curve_b, n_sms, step=2, lo_b=0, hi_b=0, objective="makespan", slack=0.05, with_antt=False):
    sa, ta, na = _curve(curve_a)
    sb, tb, nb = _curve(curve_b)
    t, a = c_f64(), c_f64()
    s = _lib.slate_choose_split_obj(sa, ta, na, sb, tb, nb, n_sms, step, lo_b, hi_b, _OBJ[objective], slack,
                                    ctypes.byref(t), ctypes.byref(a))
    return (s, t.value, a.value) if with_antt else (s, t.value)


def fluid_corun(curve_a, work_a, curve_b, work_b, n_sms, step=2, lo_b=0, hi_b=0, min_gain=1.05,
                objective="makespan", slack=0.05):
    sa, ta, na = _curve(curve_a)
    sb, tb, nb = _curve(curve_b)
    s, g = c_u32(), c_f64()
    r = _lib.slate_fluid_corun_obj(sa, ta, na, work_a, sb, tb, nb, work_b, n_sms, step, lo_b, hi_b, min_gain,
                                   _OBJ[objective], slack, ctypes.byref(s), ctypes.byref(g))
    return bool(r), s.value, g.value


def _curves_k(curves):
    keep = [_curve(c) for c in curves]
    sms = (ctypes.POINTER(c_u32) * len(curves))(*[ctypes.cast(a, ctypes.POINTER(c_u32)) for a, _, _ in keep])
    ms = (ctypes.POINTER(c_f64) * len(curves))(*[ctypes.cast(b, ctypes.POINTER(c_f64)) for _, b, _ in keep])
    npts = (c_u32 * len(curves))(*[n for _, _, n in keep])
    return keep, sms, ms, npts


def corun_makespan_k(curves, shares):
    keep, sms, ms, npts = _curves_k(curves)
    return _lib.slate_corun_makespan_k(ctypes.cast(sms, ctypes.c_void_p), ctypes.cast(ms, ctypes.c_void_p), npts,
                                       len(curves), (c_u32 * len(shares))(*shares))


def choose_split_k(curves, n_sms, step=2):
    keep, sms, ms, npts = _curves_k(curves)
    out = (c_u32 * len(curves))()
    t = _lib.slate_choose_split_k(ctypes.cast(sms, ctypes.c_void_p), ctypes.cast(ms, ctypes.c_void_p), npts,
                                  len(curves), n_sms, step, out)
    return list(out), t


def launch_fused(sa, ka, args_a, grid_a, sb, kb, args_b, grid_b, sm_b, coverage_a=None, coverage_b=None):
    """NEXT-1: launches A (session sa) and B (session sb) as one fused co-run
    kernel, B on the top sm_b SM ranks; returns (id_a, id_b)."""
    da = sa._desc(args_a, grid_a, coverage=coverage_a)
    db = sb._desc(args_b, grid_b, coverage=coverage_b)
    la, lb = c_u64(), c_u64()
    st = _lib.slate_launch_fused(sa._h, ka, ctypes.byref(da), sb._h, kb, ctypes.byref(db), sm_b, ctypes.byref(la),
                                 ctypes.byref(lb))
    if st < 0:
        raise SlateError(st, "slate_launch_fused: " + _lib.slate_last_error(sa._h).decode())
    return la.value, lb.value


def kway_admit(curves, cats, shares_cur, n_sms, step=2, min_gain=1.05):
    keep, sms, ms, npts = _curves_k(curves)
    out = (c_u32 * len(curves))()
    g = c_f64()
    r = _lib.slate_kway_admit(ctypes.cast(sms, ctypes.c_void_p), ctypes.cast(ms, ctypes.c_void_p), npts,
                              (c_u32 * len(cats))(*cats), len(shares_cur), (c_u32 * len(shares_cur))(*shares_cur),
                              n_sms, step, min_gain, out, ctypes.byref(g))
    return bool(r), list(out), g.value


def transform_source(source, name, threads=256, smem=0, block=None):
    """The generated worker source for a user kernel (no GPU needed)."""
    bx, by, bz = block if block is not None else (threads, 1, 1)
    n = ctypes.c_size_t()
    st = _lib.slate_transform_source(source.encode(), name.encode(), bx, by, bz, smem, None, 0, ctypes.byref(n))
    if st != OK:
        raise SlateError(st, "slate_transform_source")
    buf = ctypes.create_string_buffer(n.value + 1)
    _lib.slate_transform_source(source.encode(), name.encode(), bx, by, bz, smem, buf, n.value + 1, ctypes.byref(n))
    return buf.value.decode()


def rtc_stats():
    """(NVRTC compiles, in-process cache hits, on-disk cache hits) of this process."""
    a, b, c = c_u64(), c_u64(), c_u64()
    _lib.slate_rtc_stats(ctypes.byref(a), ctypes.byref(b), ctypes.byref(c))
    return a.value, b.value, c.value


def choose_iters(solo_ms, occ, n_sms, blocks, cap, budget_us=20.0):
    return _lib.slate_choose_iters(solo_ms, occ, n_sms, blocks, cap, budget_us)


def saturation_sms(curve, n_sms, frac=0.9):
    sc, tc, nc = _curve(curve)
    return _lib.slate_saturation_sms(sc, tc, nc, n_sms, frac)


# ------------------------------------------------------------------ per-kind marshalling
def cdiv(a, b):
    return -(-a // b)


def triad_args(a, b, c, s):
    n = a.numel()
    return ArgsTriad(_ptr(a), _ptr(b), _ptr(c), n, float(s), 0), (cdiv(n, 1024), 1, 1)


def copy_args(a, b):
    n = a.numel()
    return ArgsCopy(_ptr(a), _ptr(b), n), (cdiv(n, 4096), 1, 1)


def sgemm_args(A, B, C):
    m, k = A.shape
    _, n = B.shape
    return ArgsSgemm(_ptr(A), _ptr(B), _ptr(C), m, n, k, 0), (cdiv(n, 16), cdiv(m, 16), 1)


def spmv_args(rowptr, col, val, x, y):
    n_rows = rowptr.numel() - 1
    return ArgsSpmv(_ptr(rowptr), _ptr(col), _ptr(val), _ptr(x), _ptr(y), n_rows, x.numel()), (cdiv(n_rows, 32), 1, 1)


def bs_args(S, X, T, call, put, sigmas, r):
    n = S.numel()
    return ArgsBS(_ptr(S), _ptr(X), _ptr(T), _ptr(call), _ptr(put), _ptr(sigmas), n, float(r),
                  sigmas.numel()), (cdiv(n, 1024), 1, 1)


def stencil_args(inp, out):
    h, w = inp.shape
    return ArgsStencil(_ptr(inp), _ptr(out), h, w), (cdiv(w, 128), cdiv(h, 8), 1)


def kind_geometry(kind):
    tm, tn = c_u32(), c_u32()
    st = _lib.slate_kind_geometry(kind, ctypes.byref(tm), ctypes.byref(tn))
    if st != OK:
        raise SlateError(st, "slate_kind_geometry(%d)" % kind)
    return tm.value, tn.value


GEMM_TILE_M, GEMM_TILE_N = kind_geometry(KIND_GEMM_BF16)


def gemm_args(A, B, C):
    m, k = A.shape
    n, _ = B.shape
    return ArgsGemm(_ptr(A), _ptr(B), _ptr(C), m, n, k, 0), (cdiv(n, GEMM_TILE_N), cdiv(m, GEMM_TILE_M), 1)


def transpose_args(inp, out):
    h, w = inp.shape
    return ArgsTranspose(_ptr(inp), _ptr(out), h, w), (cdiv(w, 32), cdiv(h, 32), 1)


def sgemm_tiled_args(A, B, C):
    m, k = A.shape
    _, n = B.shape
    return ArgsSgemm(_ptr(A), _ptr(B), _ptr(C), m, n, k, 0), (cdiv(n, 32), cdiv(m, 32), 1)


def qrng_args(table, out, seed=0):
    dims, n = out.shape
    return ArgsQrng(_ptr(table), _ptr(out), n, dims, seed & 0xFFFFFFFF, 0), (cdiv(n, 1024), dims, 1)


def gauss_fan1_args(a, b, m, t):
    n = a.shape[0]
    return ArgsGauss(_ptr(a), _ptr(b), _ptr(m), n, t), (cdiv(n - 1 - t, 256), 1, 1)


def gauss_fan2_args(a, b, m, t):
    n = a.shape[0]
    return ArgsGauss(_ptr(a), _ptr(b), _ptr(m), n, t), (cdiv(n - t, 128), cdiv(n - 1 - t, 16), 1)
