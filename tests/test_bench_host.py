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
    # 720 J over 1.2 s and 100 steps: 7.2 J per step, 600 W
    e = _sampler(bench, 1_000_000, 1_720_000, 10.0, 11.2).energy(100)
    assert e["joules_per_step"] == pytest.approx(7.2)
    assert e["mean_watts"] == pytest.approx(600.0)
    # a 0.3 s window is below the 1 s energy window: null, not a number
    assert _sampler(bench, 1_000_000, 1_300_000, 10.0, 10.3).energy(100)["joules_per_step"] is None


def test_energy_unavailable(bench):
    assert _sampler(bench, None, 5, 0.0, 1.0).energy(1) is None


def test_spawn_command_is_one_process_per_gpu(bench):
    cmd = bench.spawn_command(4, ["--steps", "3"], 29555)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd and "--master-port=29555" in cmd
    assert cmd[-3:] == [os.path.join(ROOT, "bench.py"), "--steps", "3"]


@pytest.mark.parametrize("n,height,chunks", [(2, 37, 1), (3, 20, 1), (1, 9, 1), (3, 37, 4), (2, 37, 3)])
def test_gpus_flag_spawns_ranks_gloo_plumbing(n, height, chunks):
    # `bench.py --gpus N` without torchrun re-launches itself on N ranks; the plumbing check
    # (CPU, gloo: bands + halos, gather, max over ranks; the kernel replaced by a copy) must
    # print exactly ONE JSON line, from rank 0, with n_gpus = N and the gathered image intact.
    import json
    import subprocess
    import sys
    env = dict(os.environ, ORION_BENCH_BACKEND="gloo", OMP_NUM_THREADS="1")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--plumbing-check",
                        "--size", str(height), "--c5-chunks", str(chunks)], capture_output=True, text=True, env=env,
                       timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["plumbing_check"] and d["ok"] and d["n_gpus"] == n
    if n > 1:
        assert d["spawned"] == "1"
        rows = [b[:2] for b in d["bands"]]
        assert rows[0][0] == 0 and rows[-1][1] == height
        assert all(rows[k][1] == rows[k + 1][0] for k in range(n - 1))


@pytest.mark.parametrize("gpus", [1, 2])
def test_reference_arm_runs_the_oracle_on_rank0_only(gpus):
    # --impl reference: the CPU oracle on a bounded sample of the headline workload, one JSON line
    # from rank 0 (under --gpus 2 the other rank exits without work), e2e with no copies
    import json
    import subprocess
    import sys
    env = dict(os.environ, ORION_BENCH_BACKEND="gloo", OMP_NUM_THREADS="1")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", str(gpus),
                        "--steps", "1", "--warmup", "3"], capture_output=True, text=True, env=env, timeout=600,
                       cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == gpus and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
