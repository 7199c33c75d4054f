"""compute-sanitizer memcheck / racecheck / synccheck over every kernel path
(tools/sanitize_case.py): no out-of-bounds or misaligned access, no shared
memory race, no barrier misuse (SURVEY §4 test pyramid, level 2)."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer_clean(tool):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, PYTHONPATH=ROOT, SOMIER_NO_GRAPH="1")
    r = subprocess.run([SAN, "--tool", tool, "--error-exitcode", "7", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_case.py")],
                       capture_output=True, text=True, timeout=1200, env=env)
    out = r.stdout + r.stderr
    if r.returncode != 0 and "compute-sanitizer is closed" in out:
        # the GPU pool can replace the tool by a wrapper that refuses to run (exit 86);
        # the bounds / parity suites still cover the kernels there
        pytest.skip("compute-sanitizer unavailable on this GPU pool: " + out.strip().splitlines()[-1][:200])
    assert r.returncode == 0, out[-4000:]
    assert "sanitize case ok" in out
    assert ("ERROR SUMMARY: 0 errors" in out or "SUMMARY: 0 hazards displayed (0 errors, 0 warnings)" in out), \
        out[-4000:]
