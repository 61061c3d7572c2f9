"""The client/server path (-m gpu): a `slated` daemon process, client processes
attached through the shared-memory endpoint with their buffers shared by CUDA
IPC, four tenants from four processes at once (config C4's
shape), and a client that dies with launches in flight."""
import os
import signal
import subprocess
import sys
import time

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLIENT = os.path.join(ROOT, "tests", "ipc_client.py")


@pytest.fixture(scope="module")
def daemon():
    from paper_conf_ipps_allenf019_b200 import slate as S
    ep = "/slate-test-%d" % os.getpid()
    p = subprocess.Popen([S.DAEMON, "--device", "0", "--endpoint", ep], stderr=subprocess.PIPE)
    deadline = time.time() + 60
    while time.time() < deadline:
        try:
            s = S.Session(ep)
            s.close()
            break
        except S.SlateError:
            if p.poll() is not None:
                raise RuntimeError("slated exited: %s" % p.stderr.read().decode())
            time.sleep(0.2)
    yield ep
    p.send_signal(signal.SIGTERM)
    try:
        p.wait(timeout=30)
    except subprocess.TimeoutExpired:
        p.kill()


def _client(ep, kind, seed, *extra):
    return subprocess.Popen([sys.executable, CLIENT, ep, kind, str(seed)] + list(extra), stdout=subprocess.PIPE,
                            stderr=subprocess.STDOUT, text=True)


def test_one_client(daemon):
    p = _client(daemon, "triad", 301)
    out, _ = p.communicate(timeout=120)
    assert p.returncode == 0 and "OK triad" in out, out


def test_four_clients_at_once(daemon):
    ps = [_client(daemon, k, 310 + i) for i, k in enumerate(["triad", "spmv", "stencil", "gemm"])]
    for p in ps:
        out, _ = p.communicate(timeout=180)
        assert p.returncode == 0 and "OK" in out, out


def test_dead_client_is_cleaned_up(daemon):
    p = _client(daemon, "bs", 320, "--hang")
    line = p.stdout.readline()
    assert "READY" in line, line + p.stdout.read()
    p.kill()
    p.wait()
    # the server frees the slot and the queue; new clients still work
    time.sleep(1.0)
    q = _client(daemon, "triad", 321)
    out, _ = q.communicate(timeout=120)
    assert q.returncode == 0 and "OK triad" in out, out


def test_unshared_pointer_is_rejected(daemon):
    import torch
    from paper_conf_ipps_allenf019_b200 import slate as S
    s = S.Session(daemon)
    a, b, c = (torch.zeros(4096, device="cuda:0") for _ in range(3))
    torch.cuda.synchronize()
    k = s.register_kernel(S.KIND_TRIAD)
    args, grid = S.triad_args(a, b, c, 1.0)
    with pytest.raises(S.SlateError) as e:
        s.launch(k, args, grid)
    assert e.value.status == S.EINVAL
    s.close()


def test_user_kernel_through_the_daemon(daemon):
    """NEXT-3 through an endpoint: the source goes over the command channel, the
    daemon compiles it and rewrites the kernel's pointer parameters (found by
    the transformation) to its mappings of this client's shared buffers."""
    import numpy as np
    import torch
    from oracle import tenants as OT
    from paper_conf_ipps_allenf019_b200 import slate as S
    from test_user_kernels import PROBE3D_SRC, Args3D
    shape, block = (5, 9, 70), (16, 2, 2)
    grid = OT.probe3d_grid(shape, block)
    rng = np.random.default_rng(11)
    x = rng.integers(-300, 300, size=shape).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(shape, device="cuda:0")
    torch.cuda.synchronize()
    s = S.Session(daemon)
    s.share_buffer(xd)
    s.share_buffer(yd)
    k = s.register_source(PROBE3D_SRC, "probe3d", Args3D, block=block, iters=3)
    args = Args3D(xd.data_ptr(), yd.data_ptr(), shape[2], shape[1], shape[0])
    s.sync(s.launch(k, args, grid))
    assert np.array_equal(yd.cpu().numpy().astype(np.float64), OT.probe3d(x, block))
    s.close()
