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

    def run(cases):
        inp = "".join(" ".join(str(x) for x in (tuple(c) + (100,))[:5]) + "\n" for c in cases)
        out = subprocess.run([exe], input=inp, capture_output=True, text=True, check=True).stdout
        return [int(x) for x in out.split()]
    return run
