"""compute-sanitizer over small multiplies that reach every kernel (SURVEY §4/§5:
memcheck, racecheck, synccheck, initcheck): tools/sanitize_driver.py checks each case
against the CPU oracle, the sanitizer must report no error and no hazard."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck", "initcheck"])
def test_compute_sanitizer(tool, cuda_available):
    if not os.path.exists(SAN):
        pytest.fail("compute-sanitizer not found")
    r = subprocess.run([SAN, "--tool", tool, "--print-limit", "20", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_driver.py")],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    out = r.stdout + r.stderr
    if r.returncode != 0 and "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses every run (profiles/r1l_sanitizer.md
        # holds the round-1 results); nothing ran, so nothing is claimed
        pytest.skip("compute-sanitizer is disabled on this GPU pool")
    assert r.returncode == 0, out[-4000:]
    assert "sanitize-driver ok" in out, out[-4000:]
    if tool == "racecheck":
        assert "0 hazards displayed (0 errors, 0 warnings)" in out, out[-4000:]
    else:
        assert "ERROR SUMMARY: 0 errors" in out, out[-4000:]
