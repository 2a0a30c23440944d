"""compute-sanitizer (memcheck, racecheck, synccheck) over small invocations
of every kernel."""

import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _sanitizer():
    for c in ("/usr/local/cuda/bin/compute-sanitizer", shutil.which("compute-sanitizer")):
        if c and os.path.exists(c):
            return c
    pytest.skip("compute-sanitizer not found")


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_sanitizer_clean(tool):
    cmd = [_sanitizer(), "--tool", tool, "--error-exitcode", "17", sys.executable,
           os.path.join(ROOT, "scripts", "sanitize_target.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT)
    out = r.stdout + r.stderr
    if r.returncode == 86 and "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses to run (it has left
        # GPUs needing a reset); the tool is unavailable, not failing
        pytest.skip("compute-sanitizer closed on this GPU pool")
    assert r.returncode == 0, out[-4000:]
    assert "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards" in out, out[-4000:]
