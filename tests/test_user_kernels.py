"""NEXT-3, the runtime kernel transformation: a user's CUDA kernel
source is scanned, turned into a device body, wrapped into the slate worker
and the original kernel, and compiled with NVRTC; compiled images are cached
("A compiled kernel image can be further cached").  CPU tests check the
transformation and that NVRTC compiles its output for sm_100a (no GPU needed).
The -m gpu tests run user kernels through the worker against their original
kernel (bit-exact), the oracle or numpy (exact: integer inputs), the exact
counters and the coverage log (every original block exactly once):
  * a 2-D grid of 1-D blocks,
  * a 3-D grid of 3-D blocks (gz > 1) whose tasks straddle the x->y and y->z
    rollovers of the decode (north star "(x,y,z)", reading Q18),
    compared with oracle.tenants.probe3d, with the rank log checked,
  * a kernel that broadcasts through shared memory, at tasks of several blocks
    (the worker's barrier between blocks),
and the image cache (in process and on disk)."""
import ctypes
import os
import subprocess
import sys
import tempfile

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

USER_SRC = r"""
// a user kernel as written for plain CUDA: 2-D grid, blockIdx, gridDim, blockDim
__device__ float shift(int row) { return (float)(row % 3); }
__global__ void axpb2d(const float* __restrict__ x, float* y, float a, float b, int w, int h) {
  int col = blockIdx.x * blockDim.x + threadIdx.x;
  int row = blockIdx.y;
  if (col >= w || row >= h || blockIdx.x >= gridDim.x) return;
  y[row * w + col] = fmaf(a, x[row * w + col], b) + shift(row);
}
"""

# 3-D grid, 3-D blocks: the element (i, j, k) of an nz x ny x nx field
PROBE3D_SRC = r"""
__global__ void probe3d(const float* __restrict__ in, float* out, int nx, int ny, int nz) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  int j = blockIdx.y * blockDim.y + threadIdx.y;
  int k = blockIdx.z * blockDim.z + threadIdx.z;
  if (i >= nx || j >= ny || k >= nz) return;
  size_t e = ((size_t)k * ny + j) * nx + i;
  out[e] = in[e] * 2.0f + (float)(blockIdx.x + 3 * blockIdx.y + 7 * blockIdx.z);
}
"""

# thread 0 writes a shared value, the block reads it after a barrier
BCAST_SRC = r"""
__global__ void bcast(const float* in, float* out, int n) {
  __shared__ float s[2];
  if (threadIdx.x == 0) { s[0] = in[blockIdx.x]; s[1] = (float)blockIdx.x; }
  __syncthreads();
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  for (int r = 0; r < 64; ++r) __nanosleep(threadIdx.x & 63);   // slow lanes: a race would show
  if (i < n) out[i] = s[0] * 4.0f + s[1] + (float)threadIdx.x;
}
"""


class Args2D(ctypes.Structure):
    _fields_ = [("x", ctypes.c_uint64), ("y", ctypes.c_uint64), ("a", ctypes.c_float), ("b", ctypes.c_float),
                ("w", ctypes.c_int32), ("h", ctypes.c_int32)]


class Args3D(ctypes.Structure):
    _fields_ = [("inp", ctypes.c_uint64), ("out", ctypes.c_uint64), ("nx", ctypes.c_int32), ("ny", ctypes.c_int32),
                ("nz", ctypes.c_int32)]


class ArgsBcast(ctypes.Structure):
    _fields_ = [("inp", ctypes.c_uint64), ("out", ctypes.c_uint64), ("n", ctypes.c_int32)]


@pytest.fixture(scope="module")
def S():
    from paper_conf_ipps_allenf019_b200 import build
    build.build()
    from paper_conf_ipps_allenf019_b200 import slate
    return slate


def test_transform_renames_and_wraps(S):
    g = S.transform_source(USER_SRC, "axpb2d", threads=128)
    body = g[g.index("slate_user_body("):g.index("// ---- generated")]
    for tok in ("blockIdx", "gridDim", "threadIdx", "blockDim"):
        assert tok not in body                                         # renamed inside the body
    assert "slate_bidx.x" in body and "slate_gdim.x" in body and "slate_bdim.x" in body and "slate_tidx.x" in body
    assert "__global__ void axpb2d" not in g                          # the kernel became a device body
    assert "__device__ float shift(int row)" in g                     # the rest of the source is kept
    assert "struct SlateUserArgs {" in g and "float a;" in g and "int h;" in g
    assert ", a.x, a.y, a.a, a.b, a.w, a.h)" in g
    assert "slate::worker_body<SlateUserTenant>(p)" in g and "slate_user_original(" in g
    assert "kThreads = 128" in g
    # the pointer parameters x and y, for the server's pointer rewriting behind an endpoint
    assert "slate_user_layout[4] = {(unsigned int)sizeof(SlateUserArgs), 2u" in g
    assert "offsetof(SlateUserArgs, x)" in g and "offsetof(SlateUserArgs, y)" in g
    assert "__syncthreads();   // the previous block" not in g         # no shared memory: no barrier
    with pytest.raises(S.SlateError):
        S.transform_source(USER_SRC, "no_such_kernel")


def test_transform_3d_block_and_shared_barrier(S):
    g = S.transform_source(PROBE3D_SRC, "probe3d", block=(8, 4, 2))
    assert "kThreads = 64" in g
    assert "make_uint3(t % 8u, (t / 8u) % 4u, t / (8u * 4u)), dim3(8, 4, 2)" in g   # x-fastest linearisation
    b = S.transform_source(BCAST_SRC, "bcast", threads=128)
    assert "__syncthreads();   // the previous block" in b               # shared memory: a barrier between blocks
    assert "__syncthreads();   // the previous block" in S.transform_source(USER_SRC, "axpb2d", threads=64, smem=256)
    with pytest.raises(S.SlateError):
        S.transform_source(PROBE3D_SRC, "probe3d", block=(64, 32, 1))  # 2048 threads


@pytest.mark.parametrize("src,name,block", [(USER_SRC, "axpb2d", (128, 1, 1)), (PROBE3D_SRC, "probe3d", (8, 4, 2)),
                                            (BCAST_SRC, "bcast", (128, 1, 1))])
def test_generated_source_compiles_with_nvrtc(S, src, name, block):
    """NVRTC (the server's compiler) builds the generated worker for sm_100a."""
    try:
        nv = ctypes.CDLL("libnvrtc.so")
    except OSError:
        nv = ctypes.CDLL("/usr/local/cuda/lib64/libnvrtc.so")
    g = S.transform_source(src, name, block=block).encode()
    prog = ctypes.c_void_p()
    assert nv.nvrtcCreateProgram(ctypes.byref(prog), g, b"user.cu", 0, None, None) == 0
    opts = [b"--gpu-architecture=sm_100a", b"-std=c++17",
            ("-I" + os.path.join(ROOT, "paper_conf_ipps_allenf019_b200", "csrc")).encode(), b"-I/usr/local/cuda/include"]
    rc = nv.nvrtcCompileProgram(prog, len(opts), (ctypes.c_char_p * len(opts))(*opts))
    n = ctypes.c_size_t()
    nv.nvrtcGetProgramLogSize(prog, ctypes.byref(n))
    log = ctypes.create_string_buffer(n.value)
    nv.nvrtcGetProgramLog(prog, log)
    assert rc == 0, log.value.decode()
    nv.nvrtcGetCUBINSize(prog, ctypes.byref(n))
    cubin = ctypes.create_string_buffer(n.value)
    nv.nvrtcGetCUBIN(prog, cubin)
    assert b"slate_user_worker" in cubin.raw and b"slate_user_original" in cubin.raw
    assert b"slate_user_layout" in cubin.raw


def _check_counters(q, B, iters, cov_counts):
    from oracle import tenants as OT
    ex = OT.expected_counters(B, iters)
    assert (q["blocks_done"], q["tasks_done"], q["next_clamped"]) == \
        (ex["blocks_done"], ex["tasks_done"], ex["next_clamped"])
    assert q["coverage_ok"] == 1 and np.array_equal(cov_counts, ex["coverage"].astype(np.int32))


@pytest.mark.gpu
def test_user_kernel_through_the_worker(S):
    import torch

    w, h, T = 1000, 37, 128
    rng = np.random.default_rng(160)
    x = rng.integers(-100, 100, size=(h, w)).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(h, w, device="cuda:0")
    grid = (-(-w // T), h, 1)
    args = Args2D(xd.data_ptr(), yd.data_ptr(), 2.0, 1.0, w, h)
    expect = 2.0 * x.astype(np.float64) + 1.0 + (np.arange(h) % 3)[:, None]   # exact on these integers
    with S.Session(None, 0) as s:
        k_std = s.register_source(USER_SRC, "axpb2d", Args2D, threads=T)
        torch.cuda.synchronize()
        s.sync(s.launch(k_std, args, grid, mode=S.MODE_STANDALONE))
        torch.cuda.synchronize()
        ref = yd.clone()
        assert np.array_equal(ref.cpu().numpy().astype(np.float64), expect)
        n = s.info()["num_sms"]
        B = grid[0] * grid[1]
        for iters in (1, 3):
            k = s.register_source(USER_SRC, "axpb2d", Args2D, threads=T, iters=iters, flags=S.KFLAG_COVERAGE)
            for sm in [(0, n - 1), (5, 5 + n // 4)]:
                yd.zero_()
                cov = torch.zeros(B, dtype=torch.int32, device="cuda:0")
                torch.cuda.synchronize()
                lid = s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=sm, coverage=cov)
                s.sync(lid)
                torch.cuda.synchronize()
                assert torch.equal(yd, ref), (iters, sm)
                _check_counters(s.query(lid), B, iters, cov.cpu().numpy())


@pytest.mark.gpu
def test_3d_grid_of_3d_blocks_matches_the_oracle(S):
    """gz > 1: tasks of 4 and 7 blocks straddle the x->y and y->z rollovers of
    the per-task decode (Lst2 (4), Q18); output equals oracle.probe3d exactly
    and the original kernel bit for bit; every task ran on a rank inside the
    range in force (rank log)."""
    import torch
    from oracle import tenants as OT

    shape, block = (7, 11, 37), (8, 4, 2)
    grid = OT.probe3d_grid(shape, block)                   # (5, 3, 4): 60 blocks
    B = grid[0] * grid[1] * grid[2]
    rng = np.random.default_rng(3)
    x = rng.integers(-1000, 1000, size=shape).astype(np.float32)
    expect = OT.probe3d(x, block)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(shape, device="cuda:0")
    args = Args3D(xd.data_ptr(), yd.data_ptr(), shape[2], shape[1], shape[0])
    with S.Session(None, 0) as s:
        n = s.info()["num_sms"]
        k0 = s.register_source(PROBE3D_SRC, "probe3d", Args3D, block=block)
        torch.cuda.synchronize()
        s.sync(s.launch(k0, args, grid, mode=S.MODE_STANDALONE))
        torch.cuda.synchronize()
        ref = yd.clone()
        assert np.array_equal(ref.cpu().numpy().astype(np.float64), expect)
        for iters in (1, 4, 7):
            k = s.register_source(PROBE3D_SRC, "probe3d", Args3D, block=block, iters=iters,
                                  flags=S.KFLAG_COVERAGE | S.KFLAG_RANKLOG)
            for sm in [(0, n - 1), (3, 3 + n // 5)]:
                yd.zero_()
                cov = torch.zeros(2 * B, dtype=torch.int32, device="cuda:0")
                torch.cuda.synchronize()
                lid = s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=sm, coverage=cov)
                s.sync(lid)
                torch.cuda.synchronize()
                assert torch.equal(yd, ref), (iters, sm)
                c = cov.cpu().numpy().view(np.uint32)
                _check_counters(s.query(lid), B, iters, c[:B].astype(np.int32))
                log = c[B:]
                assert np.all(log >> 31 == 1)
                rank, lo, hi = log & 0xff, (log >> 8) & 0xff, (log >> 16) & 0xff
                assert np.all((lo == sm[0]) & (hi == sm[1])), (iters, sm)
                assert np.all((rank >= lo) & (rank <= hi)), (iters, sm)


@pytest.mark.gpu
def test_shared_memory_broadcast_at_multi_block_tasks(S):
    import torch
    T, nb = 128, 300
    n = T * nb - 17
    rng = np.random.default_rng(5)
    x = rng.integers(-64, 64, size=nb).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(n, device="cuda:0")
    args = ArgsBcast(xd.data_ptr(), yd.data_ptr(), n)
    i = np.arange(n)
    expect = x[i // T].astype(np.float64) * 4 + (i // T) + (i % T)
    with S.Session(None, 0) as s:
        nsm = s.info()["num_sms"]
        for iters in (5, 8):
            k = s.register_source(BCAST_SRC, "bcast", ArgsBcast, threads=T, iters=iters)
            yd.zero_()
            torch.cuda.synchronize()
            s.sync(s.launch(k, args, (nb, 1, 1), placement=S.PLACE_CORUN, sm=(0, nsm // 8)))
            torch.cuda.synchronize()
            assert np.array_equal(yd.cpu().numpy().astype(np.float64), expect), iters


@pytest.mark.gpu
def test_image_cache_in_process_and_on_disk(S):
    """A second registration of the same source (another task size) reuses the
    loaded image; a fresh process with the same cache directory loads the
    cubin from disk instead of running NVRTC; a wrong args_size is EINVAL."""
    with S.Session(None, 0) as s:
        c0, m0, _ = S.rtc_stats()
        s.register_source(BCAST_SRC, "bcast", ArgsBcast, threads=96, iters=2)
        c1, m1, _ = S.rtc_stats()
        s.register_source(BCAST_SRC, "bcast", ArgsBcast, threads=96, iters=3)
        c2, m2, _ = S.rtc_stats()
        assert c2 == c1 and m2 == m1 + 1
        with pytest.raises(S.SlateError) as e:
            s.register_source(BCAST_SRC, "bcast", Args3D, threads=96)   # 32-byte struct vs the kernel's 24
        assert e.value.status == S.EINVAL
    code = ("import sys; sys.path.insert(0, %r); sys.path.insert(0, %r)\n"
            "from test_user_kernels import BCAST_SRC, ArgsBcast\n"
            "from paper_conf_ipps_allenf019_b200 import slate as S\n"
            "with S.Session(None, 0) as s:\n"
            "    s.register_source(BCAST_SRC.replace('64', '65'), 'bcast', ArgsBcast, threads=160)\n"
            "print(*S.rtc_stats())\n") % (ROOT, os.path.join(ROOT, "tests"))
    with tempfile.TemporaryDirectory() as d:
        env = dict(os.environ, SLATE_RTC_CACHE=os.path.join(d, "rtc"))
        runs = [subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
                for _ in range(2)]
        for r in runs:
            assert r.returncode == 0, r.stderr
        first = list(map(int, runs[0].stdout.split()))
        second = list(map(int, runs[1].stdout.split()))
        assert first == [1, 0, 0] and second == [0, 0, 1], (first, second)
        assert len(os.listdir(os.path.join(d, "rtc"))) == 1
