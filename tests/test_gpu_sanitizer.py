"""compute-sanitizer over small launches of every kernel family (SURVEY §4 layer 3, §5 race
detection): memcheck (out-of-bounds / misaligned accesses, incl. the ragged edges and the
fan-out stores), racecheck (shared-memory hazards in the staged tiles, the H buffers and the
cp.async rings) and synccheck (barrier use).  Slow (minutes), so each tool runs once."""
import os
import shutil
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer_clean(tool):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cs = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(cs):
        pytest.skip("compute-sanitizer not installed")
    r = subprocess.run([cs, "--tool", tool, "--error-exitcode", "3", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_run.py")],
                       capture_output=True, text=True, timeout=1800, cwd=ROOT)
    out = r.stdout + r.stderr
    assert "sanitize run complete" in out, out[-3000:]
    # memcheck / synccheck print "ERROR SUMMARY: 0 errors", racecheck "RACECHECK SUMMARY: 0 hazards
    # displayed (0 errors, 0 warnings)"
    clean = "ERROR SUMMARY: 0 errors" in out or "0 hazards displayed (0 errors, 0 warnings)" in out
    assert r.returncode == 0 and clean, out[-3000:]
