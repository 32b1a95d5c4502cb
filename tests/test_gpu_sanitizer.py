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
    if "sanitize run complete" not in out and "compute-sanitizer is closed" in out:
        # the GPU pool's operators disabled the tool (its runs left GPUs needing a reset); the
        # earlier clean runs stay recorded in profiles/, bounds are covered by the parity tests
        pytest.skip("compute-sanitizer closed on this GPU pool: " + out.strip().splitlines()[0][:200])
    assert "sanitize run complete" in out, out[-3000:]
    # memcheck / synccheck print "ERROR SUMMARY: 0 errors", racecheck "RACECHECK SUMMARY: 0 hazards
    # displayed (0 errors, 0 warnings)"
    clean = "ERROR SUMMARY: 0 errors" in out or "0 hazards displayed (0 errors, 0 warnings)" in out
    assert r.returncode == 0 and clean, out[-3000:]
