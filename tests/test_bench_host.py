"""Host logic of bench.py that needs no GPU: the energy report of the clock sampler."""
import importlib.util
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod


def _sampler(bench, e0, e1, t0, t1):
    s = bench.ClockSampler.__new__(bench.ClockSampler)
    s.ok, s.e0, s.e1, s.t0, s.t1 = True, e0, e1, t0, t1
    return s


def test_energy_short_window_is_null(bench):
    # a 1 ms timed region: the coarse NVML counter has not ticked, 0 J is not a measurement
    e = _sampler(bench, 5000, 5000, 10.0, 10.001).energy(300)
    assert e["joules_per_step"] is None and e["mean_watts"] is None and "note" in e


def test_energy_long_window(bench):
    # 600 J over 1 s and 100 steps: 6 J per step, 600 W
    e = _sampler(bench, 1_000_000, 1_600_000, 10.0, 11.0).energy(100)
    assert e["joules_per_step"] == pytest.approx(6.0)
    assert e["mean_watts"] == pytest.approx(600.0)


def test_energy_unavailable(bench):
    assert _sampler(bench, None, 5, 0.0, 1.0).energy(1) is None
