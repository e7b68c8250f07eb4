"""compute-sanitizer memcheck / racecheck / synccheck over a small end-to-end run of the library."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _sanitizer():
    for c in ("/usr/local/cuda/bin/compute-sanitizer", shutil.which("compute-sanitizer")):
        if c and os.path.exists(c):
            return c
    pytest.skip("compute-sanitizer not found")


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(cuda_device, tool):
    cmd = [_sanitizer(), "--tool", tool, "--error-exitcode", "7", "--print-limit", "20",
           sys.executable, os.path.join(HERE, "tools", "sanitize_run.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
    tail = (r.stdout + r.stderr)[-4000:]
    assert r.returncode == 0, tail
    assert "sanitize run ok" in r.stdout, tail
    assert "ERROR SUMMARY: 0 errors" in (r.stdout + r.stderr) or "0 hazards" in (r.stdout + r.stderr), tail
