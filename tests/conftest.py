import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs the CUDA path through the C-ABI)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def occ_ref(tmp_path_factory):
    """NVIDIA's header-only occupancy calculator, compiled as a CLI (test helper)."""
    exe = str(tmp_path_factory.mktemp("occ") / "occ_ref")
    subprocess.check_call(["g++", "-O1", "-I/usr/local/cuda/include",
                           os.path.join(ROOT, "tests", "helpers", "occ_ref.cpp"), "-o", exe])

    def run(cases, mask=False):
        """CTAs/SM per case; with mask=True, (CTAs/SM, limitingFactors) pairs."""
        inp = "".join(" ".join(str(x) for x in (tuple(c) + (100,))[:5]) + "\n" for c in cases)
        out = subprocess.run([exe] + (["--mask"] if mask else []), input=inp, capture_output=True,
                             text=True, check=True).stdout
        vals = [int(x) for x in out.split()]
        return list(zip(vals[0::2], vals[1::2])) if mask else vals
    return run
