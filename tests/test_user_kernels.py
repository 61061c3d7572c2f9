"""NEXT-3, the runtime kernel transformation: a user's CUDA kernel
source is scanned, turned into a device body, wrapped into the slate worker
and the original kernel, and compiled with NVRTC.  CPU tests check the
transformation and that NVRTC compiles its output for sm_100a (no GPU needed);
the -m gpu test runs a 2-D user kernel through the worker against its original
kernel (bit-exact), numpy (exact: integer inputs), the exact counters and the
coverage log (every original block exactly once)."""
import ctypes
import os

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


@pytest.fixture(scope="module")
def S():
    from paper_conf_ipps_allenf019_b200 import build
    build.build()
    from paper_conf_ipps_allenf019_b200 import slate
    return slate


def test_transform_renames_and_wraps(S):
    g = S.transform_source(USER_SRC, "axpb2d", threads=128)
    body = g[g.index("slate_user_body("):g.index("// ---- generated")]
    assert "blockIdx" not in body and "gridDim" not in body          # renamed inside the body
    assert "slate_bidx.x" in body and "slate_gdim.x" in body and "blockDim.x" in body
    assert "__global__ void axpb2d" not in g                          # the kernel became a device body
    assert "__device__ float shift(int row)" in g                     # the rest of the source is kept
    assert "struct SlateUserArgs {" in g and "float a;" in g and "int h;" in g
    assert "slate_user_body(make_uint3(x, y, z), slate_user_gdim, a.x, a.y, a.a, a.b, a.w, a.h)" in g
    assert "slate::worker_body<SlateUserTenant>(p)" in g and "slate_user_original(" in g
    assert "kThreads = 128" in g
    with pytest.raises(S.SlateError):
        S.transform_source(USER_SRC, "no_such_kernel")


def test_generated_source_compiles_with_nvrtc(S):
    """NVRTC (the server's compiler) builds the generated worker for sm_100a."""
    try:
        nv = ctypes.CDLL("libnvrtc.so")
    except OSError:
        nv = ctypes.CDLL("/usr/local/cuda/lib64/libnvrtc.so")
    g = S.transform_source(USER_SRC, "axpb2d", threads=128).encode()
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


@pytest.mark.gpu
def test_user_kernel_through_the_worker(S):
    import torch
    from oracle import tenants as OT

    class Args(ctypes.Structure):
        _fields_ = [("x", ctypes.c_uint64), ("y", ctypes.c_uint64), ("a", ctypes.c_float), ("b", ctypes.c_float),
                    ("w", ctypes.c_int32), ("h", ctypes.c_int32)]

    w, h, T = 1000, 37, 128
    rng = np.random.default_rng(160)
    x = rng.integers(-100, 100, size=(h, w)).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(h, w, device="cuda:0")
    grid = (-(-w // T), h, 1)
    args = Args(xd.data_ptr(), yd.data_ptr(), 2.0, 1.0, w, h)
    expect = 2.0 * x.astype(np.float64) + 1.0 + (np.arange(h) % 3)[:, None]   # exact on these integers
    with S.Session(None, 0) as s:
        k_std = s.register_source(USER_SRC, "axpb2d", Args, threads=T)
        torch.cuda.synchronize()
        s.sync(s.launch(k_std, args, grid, mode=S.MODE_STANDALONE))
        torch.cuda.synchronize()
        ref = yd.clone()
        assert np.array_equal(ref.cpu().numpy().astype(np.float64), expect)
        n = s.info()["num_sms"]
        B = grid[0] * grid[1]
        for iters in (1, 3):
            k = s.register_source(USER_SRC, "axpb2d", Args, threads=T, iters=iters, flags=S.KFLAG_COVERAGE)
            for sm in [(0, n - 1), (5, 5 + n // 4)]:
                yd.zero_()
                cov = torch.zeros(B, dtype=torch.int32, device="cuda:0")
                torch.cuda.synchronize()
                lid = s.launch(k, args, grid, placement=S.PLACE_CORUN, sm=sm, coverage=cov)
                s.sync(lid)
                torch.cuda.synchronize()
                assert torch.equal(yd, ref), (iters, sm)
                q = s.query(lid)
                ex = OT.expected_counters(B, iters)
                assert (q["blocks_done"], q["tasks_done"], q["next_clamped"]) == \
                    (ex["blocks_done"], ex["tasks_done"], ex["next_clamped"])
                assert q["coverage_ok"] == 1 and np.array_equal(cov.cpu().numpy(), ex["coverage"].astype(np.int32))
