"""compute-sanitizer over a small-shape workload of every entry point
(tools/sanitize.py: every variant x dtype x band height, segments and the
unit queue, generic path, seeded, sharded, widening, fused box filter; each
call also checked against the oracle).  The look-back protocol's flags and
mbarrier phases are exactly what racecheck/synccheck look at."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer_clean(tool):
    exe = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    assert os.path.exists(exe), "compute-sanitizer not found"
    r = subprocess.run([exe, "--tool", tool, "--error-exitcode", "9", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize.py")],
                       capture_output=True, text=True, timeout=1200)
    out = r.stdout + r.stderr
    assert r.returncode == 0, out[-4000:]
    assert "sanitize workload ok" in out
    assert ("0 errors" in out) or ("0 hazards" in out), out[-2000:]
