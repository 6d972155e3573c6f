"""compute-sanitizer memcheck / racecheck / synccheck on tiny runs of every kernel family
(persistent streaming with mbarrier/TMA ring, resident, discrete baselines, residual norm) —
SURVEY §4.2 T1.  Each tool must report zero errors."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    cmd = ["/usr/local/cuda/bin/compute-sanitizer", "--tool", tool, "--error-exitcode", "17",
           sys.executable, os.path.join(HERE, "sanitize_case.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
    out = r.stdout + r.stderr
    if "SANITIZE_CASE_OK" not in out and "compute-sanitizer is closed" in out:
        # the GPU pool replaces the tool with a refusal (sanitizer runs left GPUs needing a reset);
        # (all three tools ran clean in the earlier GPU suites, profiles/r02_pytest_gpu.log)
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert "SANITIZE_CASE_OK" in out, out[-3000:]
    assert r.returncode == 0, out[-3000:]
