"""The server watchdog (slate.h slate_sync): a launch still running
SLATE_WATCHDOG_S after its issue makes slate_sync return ECUDA ("watchdog")
instead of blocking forever -- a kernel cannot be preempted, the report is what
a client gets.  Run in a subprocess with a 0.3-s limit and a user kernel that
spins for 2 s (NEXT-3 registration)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CODE = r'''
import ctypes, sys, time
sys.path.insert(0, %r)
from paper_conf_ipps_allenf019_b200 import slate as S
SRC = """
__global__ void spin(unsigned long long ns) {
  unsigned long long t0; asm volatile("mov.u64 %%0, %%%%globaltimer;" : "=l"(t0));
  for (;;) { unsigned long long t; asm volatile("mov.u64 %%0, %%%%globaltimer;" : "=l"(t)); if (t - t0 > ns) break; }
}
"""
class A(ctypes.Structure):
    _fields_ = [("ns", ctypes.c_uint64)]
s = S.Session(None, 0)
k = s.register_source(SRC, "spin", A, threads=32, iters=1)
t0 = time.time()
lid = s.launch(k, A(2000000000), (1, 1, 1), placement=S.PLACE_SOLO)
try:
    s.sync(lid)
    print("NO-ERROR")
except S.SlateError as e:
    print("ERR", e.status, "%%.2f" %% (time.time() - t0), "watchdog" in str(e))
s.close()
print("CLOSED", "%%.2f" %% (time.time() - t0))
''' % ROOT


def test_watchdog_reports_a_hung_launch():
    env = dict(os.environ, SLATE_WATCHDOG_S="0.3")
    r = subprocess.run([sys.executable, "-c", CODE], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-3000:]
    err = [l for l in r.stdout.splitlines() if l.startswith("ERR")]
    assert err, r.stdout + r.stderr[-2000:]
    _, status, t, has_msg = err[0].split()
    assert int(status) == -3 and float(t) < 1.5 and has_msg == "True"
    assert "watchdog" in r.stderr
    assert any(l.startswith("CLOSED") for l in r.stdout.splitlines())
