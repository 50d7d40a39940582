"""compute-sanitizer over the particle loop: memcheck,
racecheck (shared-memory hazards of the TMA stages, mbarrier releases,
per-warp append rings and hop queues) and synccheck on a small C1-style run
(tests/sanitize_case.py) through the C ABI (-m gpu)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool,dep,dh", [("memcheck", 1, 1), ("racecheck", 1, 1), ("racecheck", 2, 0),
                                         ("synccheck", 1, 1), ("memcheck", 0, 2)])
def test_sanitizer_clean(tool, dep, dh):
    cmd = [SAN, "--tool", tool, "--error-exitcode", "99", "--print-limit", "20",
           sys.executable, os.path.join(ROOT, "tests", "sanitize_case.py"), str(dep), str(dh)]
    if tool == "memcheck":
        cmd[3:3] = ["--leak-check", "no"]
    out = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    log = out.stdout[-4000:] + out.stderr[-4000:]
    assert out.returncode == 0, log
    assert "sanitize case ok" in out.stdout
    assert "ERROR SUMMARY: 0 errors" in log or "RACECHECK SUMMARY: 0 hazards" in log, log
