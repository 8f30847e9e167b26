"""compute-sanitizer over every kernel variant: memcheck (out-of-bounds / misaligned
accesses) and racecheck (shared-memory hazards, the concern of the in-place sweeps) on tiny
shapes driven by tools/sanitize_drive.py; the drive itself asserts no NaN appears in Psi."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck"])
def test_compute_sanitizer_clean(tool):
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not found")
    r = subprocess.run([SAN, "--tool", tool, "--error-exitcode", "17", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_drive.py")],
                       capture_output=True, text=True, timeout=900)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "sanitize drive ok" in out, out[-4000:]
    assert ("ERROR SUMMARY: 0 errors" in out or "(0 errors, 0 warnings)" in out), out[-4000:]
