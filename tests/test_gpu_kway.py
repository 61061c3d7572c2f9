"""NEXT-4, k-way co-runs (-m gpu): with two jobs co-running (a compute job and a
memory job, Tab I), a third job -- a compute job on a grid too small to fill
the chip -- is admitted into the group when the fluid model predicts a gain
(slate_kway_admit, reading Q49), and runs on its own share of SMs
beside the other two.  Checked: every output (oracle, exact on integer
inputs, or bit-exact against the original kernel), exactly-once coverage, and
the rank log -- the third job's tasks ran on a strict sub-range while the
other two were still running, on ranks inside the range in force."""
import numpy as np
import pytest
import torch

from paper_conf_ipps_allenf019_b200 import slate as S

from gpu_helpers import make_bs, make_sgemm_tiled, make_triad

pytestmark = pytest.mark.gpu
FLAGS = S.KFLAG_COVERAGE | S.KFLAG_RANKLOG


def test_third_corunner_is_admitted():
    ta = make_bs(1 << 22, 601, n_scen=32)              # compute, H_C, scales with SMs
    tb = make_triad(1 << 26, 602, "int")               # memory, H_M, saturates at ~half the chip
    tc = make_sgemm_tiled(256, 512, 4096, 603, "int")  # compute on 128 blocks: cannot fill 148 SMs
    sess = [S.Session(None, 0) for _ in range(3)]
    try:
        n = sess[0].info()["num_sms"]
        ks, refs = [], []
        for s, t in zip(sess, (ta, tb, tc)):
            k0 = s.register_kernel(t.kind)
            t.zero_outputs()
            s.sync(s.launch(k0, t.args, t.grid, mode=S.MODE_STANDALONE))
            torch.cuda.synchronize()
            refs.append(t.snapshot())
            s.profile(k0, t.args, t.grid, S.PROF_CURVE)
            ks.append(s.register_kernel(t.kind, flags=FLAGS))
        reps = (6, 24, 3)
        covs, ids = [], []
        for s, t, k, r in zip(sess, (ta, tb, tc), ks, reps):
            B = int(np.prod(t.grid))
            c = [torch.zeros(2 * B, dtype=torch.int32, device="cuda:0") for _ in range(r)]
            covs.append(c)
        for t in (ta, tb, tc):
            t.zero_outputs()
        torch.cuda.synchronize()
        for s, t, k, c in zip(sess, (ta, tb, tc), ks, covs):
            ids.append([s.launch(k, t.args, t.grid, placement=S.PLACE_AUTO, coverage=x) for x in c])
        for s in sess:
            s.sync(0)
        torch.cuda.synchronize()
        for t, ref in zip((ta, tb, tc), refs):
            for x, y in zip(t.snapshot(), ref):
                assert torch.equal(x, y)
        ranges = []
        for t, c in zip((ta, tb, tc), covs):
            B = int(np.prod(t.grid))
            rs = set()
            for x in c:
                v = x.cpu().numpy().view(np.uint32)
                assert np.all(v[:B] == 1)
                log = v[B:]
                rank, lo, hi, out = log & 0xff, (log >> 8) & 0xff, (log >> 16) & 0xff, (log >> 24) & 1
                assert np.all(((rank >= lo) & (rank <= hi)) | (out == 1))
                rs |= set(zip(lo.tolist(), hi.tolist()))
            ranges.append(rs)
        # the third job ran on a strict sub-range: admitted into the running group
        assert any(hi - lo + 1 < n for lo, hi in ranges[2]), ranges[2]
        # and the memory job and the first compute job were split too
        assert any(hi - lo + 1 < n for lo, hi in ranges[0]) and any(hi - lo + 1 < n for lo, hi in ranges[1])
    finally:
        for s in sess:
            s.close()
