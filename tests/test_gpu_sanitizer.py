"""compute-sanitizer over every worker (SURVEY §4 T1, §5 race detection): the
runtime's hand-rolled ordering -- relaxed resize-word loads completed by a
fence, fence-free mapped-memory stores, the mbarrier rings of the copy, SpMV
and GEMM workers and the GEMM pair's cross-CTA arrives -- run on tiny configs
(tests/sanitize_target.py) under memcheck (out-of-bounds / misaligned global
and shared accesses), racecheck (shared-memory hazards) and synccheck (barrier
misuse).  A tool that reports any error fails the test; the target itself
checks every output against the oracle."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
GROUPS = ["generic", "apps", "spmv", "gemm", "user", "fused"]


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
@pytest.mark.parametrize("group", GROUPS)
def test_sanitizer(tool, group):
    cmd = [SAN, "--tool", tool, "--error-exitcode", "97", "--print-limit", "20"]
    if tool == "memcheck":
        cmd += ["--leak-check", "no"]
    cmd += [sys.executable, os.path.join(HERE, "sanitize_target.py"), group]
    env = dict(os.environ, SLATE_STANDBY_TIMEOUT_US="20000")   # a slower world: no early liveness joins
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, env=env)
    tail = (r.stdout + r.stderr)[-4000:]
    assert r.returncode == 0, tail
    assert "SANITIZE-OK %s" % group in r.stdout, tail
    assert "ERROR SUMMARY: 0 errors" in r.stdout + r.stderr, tail
