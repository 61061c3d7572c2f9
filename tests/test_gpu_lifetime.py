"""Launch-record lifetime (-m gpu): the server keeps completed launches for
slate_query for the newest SLATE_KEEP_FINISHED of them and then drops the
records and their CUDA events in bulk, so a long-running slated stays bounded
(ADVICE r1).  A subprocess with a window of 16 runs 300 launches."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CODE = r'''
import sys
sys.path.insert(0, %r); sys.path.insert(0, %r)
import torch
from gpu_helpers import make_triad
from paper_conf_ipps_allenf019_b200 import slate as S
t = make_triad(1024 * 8, 1, "int")
s = S.Session(None, 0)
k = s.register_kernel(t.kind, iters=2)
ids = []
for _ in range(10):
    ids += s.launch_n(k, t.args, t.grid, 30)
    s.sync(0)
old, new = ids[0], ids[-1]
assert s.query(new)["state"] == 2
try:
    s.query(old)
    print("OLD-STILL-THERE")
except S.SlateError as e:
    print("OLD-GONE", e.status)
print("SYNC-OLD", s.sync(old))
assert t.check(t.snapshot())[0]
s.close()
print("DONE")
''' % (ROOT, os.path.join(ROOT, "tests"))


def test_finished_launch_records_are_bounded():
    env = dict(os.environ, SLATE_KEEP_FINISHED="16")
    r = subprocess.run([sys.executable, "-c", CODE], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-3000:]
    out = r.stdout.split()
    assert "OLD-GONE" in out and out[out.index("OLD-GONE") + 1] == "-6"     # ENOTFOUND: dropped
    assert "SYNC-OLD" in out and out[out.index("SYNC-OLD") + 1] == "0"      # an old id has completed
    assert "DONE" in out
