#!/usr/bin/env python3
"""bench.py -- Orion occupancy-tuned hot path on B200 (BASELINE.json metric).

One "step" = one application iteration of the whole hot path on one synthetic frame:
orion_tune_step (Fig. 9 dynamic selection over the Fig. 8 ladder of the occupancy variants
orion_build_variants produced from orion_levels) launching the configuration's kernel.
Variants are built and every level is swept (orion_sweep, the exhaustive brute-force
reference) before the timed region.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--workload c1|c2|c3|c4|c5|srad] [--only] [--no-cpu-baseline]

N = 1 (default): the headline is C2 (NLM 2048^2, BASELINE.json configs[1]); the same JSON
line carries a sub-record per other configuration (C1, C3, C4, C5 at P = 1, SRAD) with its
sweep, tuner walk, regret, vs max-occupancy, roofline and end-to-end figure, plus the NEXT-3
resource-saving / energy record (Fig. 12 / 13 analogue).  --only: the headline workload alone.

N > 1: the headline is C5 -- one 16384^2 NLM frame row-sharded over the N ranks (slab + 6-row
halo generated in place, a tuner per rank, the output bands gathered into every rank's full
image over NVLink) -- with C5 at P = 1 on rank 0 as the anchor of the curve.  Without
torchrun, `--gpus N` re-launches itself under torch.distributed.run (one process per GPU).

Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "tuned Mpix/s vs max-occupancy build; tuner regret vs exhaustive level sweep"

# Workloads (BASELINE.json configs).  `insts`: algorithmic FP32-pipe instructions per output
# unit of the formulation each kernel implements; `bytes`: HBM bytes per unit.
WORKLOADS = {
    # KNN: 49 taps x (3 FSUB + FMUL + 2 FFMA distance, 1 FFMA exponent, 3 FFMA + 1 FADD
    # accumulate, 1 compare) + ~10 for the blend
    # C1's 64x64 frames run as batches (orion_args.batch: B frames per launch, one batch per
    # tuner iteration and per step) through the tile kernel with 256-thread CTAs; --batch 1
    # restores one frame per step (use --kernel knn_f4_t16, the small-frame kernel, then)
    "c1": dict(kernel="knn_f4", threads=256, batch=256, W=64, H=64, sigma=0.2, unit="Mpix/s",
               name="imageDenoising KNN 64x64 RGBA r=3", insts=49 * 12 + 10, bytes=32, steps=300, cfg_index=0),
    # NLM box-sum + symmetric pairs, per pixel and offset pair: 1 difference (6), 1 horizontal
    # and 2 vertical blocked 7-sums (4 each), 2 x (1 FFMA exponent + 3 FFMA + 1 FADD + 1 compare)
    "c2": dict(kernel="nlm_f4_w", W=2048, H=2048, sigma=0.13, unit="Mpix/s", name="imageDenoising NLM 2048x2048 RGBA",
               insts=24 * 30 + 10, bytes=32, steps=300, cfg_index=1),
    # thermal stencil: four explicit steps per launch (hotspot4h_f32), 12 B per cell per launch
    "c3": dict(kernel="hotspot4h_f32", W=8192, H=8192, unit="Mcell-steps/s", name="thermal stencil 8192x8192 fp32",
               insts=12, bytes=12, steps=25, cfg_index=2),
    # register-heavy direct NLM: 2401 patch terms x 6 + 49 x 6 per-offset terms + blend
    "c4": dict(kernel="nlm_f4_regheavy", W=4096, H=4096, sigma=0.13, unit="Mpix/s",
               name="register-heavy NLM 4096x4096 RGBA, maxrregcount caps", insts=2401 * 6 + 49 * 6 + 10, bytes=32,
               steps=30, cfg_index=3),
    "c5": dict(kernel="nlm_f4_w", W=16384, H=16384, sigma=0.13, unit="Mpix/s",
               name="imageDenoising NLM 16384x16384 RGBA row-sharded with halos + all-gather",
               insts=24 * 30 + 10, bytes=32, steps=10, cfg_index=4),
    # NEXT-4: a second Rodinia stencil (srad), 8 B/cell-iteration (read J, write J')
    "srad": dict(kernel="srad_f32hs", W=8192, H=8192, unit="Mcell-steps/s", name="SRAD 8192x8192 fp32 (NEXT-4)",
                 insts=60, bytes=8, steps=100, cfg_index=None),
}
SUB_RECORDS = ("c1", "c3", "c4", "srad", "c5")
ROI = (0, 127, 0, 127)     # SRAD's ROI statistics window (reading R-SRAD: Rodinia's default)


def is_stencil_id(kernel: str) -> bool:
    return kernel.startswith("hotspot") or kernel.startswith("srad")


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


# throttle reasons that void a timed region (re-measured once); sw_power_cap is kept and noted
THROTTLE_REJECT = {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "hw_power_brake_slowdown"}


class ClockSampler:
    """nvidia-smi-equivalent sampling (NVML) of SM clock + throttle reasons during the timed
    region, and the board energy counter over it.  Call ``mark_end()`` right after the closing
    synchronize: the window then ends with the GPU work, not after the sampler thread joins."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}

    MIN_WINDOW_S = 1.0

    def __init__(self, index: int, period: float = 0.02):
        self.samples, self.reasons, self.ok = [], set(), False
        self.period = period
        self.stop = threading.Event()
        self.e1 = self.t1 = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)
            self.max_mhz = None

    def _sample(self):
        try:
            self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            for bit, name in self.REASONS.items():
                if r & bit:
                    self.reasons.add(name)
        except Exception:
            pass

    def _run(self):
        self._sample()
        while not self.stop.wait(self.period):     # returns at once when stopped
            self._sample()

    def _energy_mj(self):
        try:
            return self.nv.nvmlDeviceGetTotalEnergyConsumption(self.h)
        except Exception:
            return None

    def __enter__(self):
        if self.ok:
            self.e0, self.t0 = self._energy_mj(), time.perf_counter()
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def mark_end(self):
        if self.ok and self.t1 is None:
            self.e1, self.t1 = self._energy_mj(), time.perf_counter()

    def __exit__(self, *a):
        if self.ok:
            self.mark_end()
            self.stop.set()
            self.t.join()

    def energy(self, steps: int):
        """Board energy over the timed region (NVML counter, mJ): J per step and mean W."""
        if not self.ok or self.e0 is None or self.e1 is None:
            return None
        j = (self.e1 - self.e0) / 1e3
        window = self.t1 - self.t0
        if j <= 0 or window < self.MIN_WINDOW_S:
            # The board counter advances in coarse ticks: a short timed region reads 0 J or a
            # few ticks, which is not a measurement (next3_energy uses >= 1.2 s windows).
            return {"joules_per_step": None, "mean_watts": None, "source": "nvml total energy",
                    "note": f"timed region {window * 1e3:.1f} ms is below the {self.MIN_WINDOW_S:.1f} s "
                            f"energy window"}
        return {"joules_per_step": j / steps, "mean_watts": j / window, "window_s": window,
                "source": "nvml total energy"}

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons - {"gpu_idle"}), "samples": len(self.samples)}


# ---- processes: one per GPU -------------------------------------------------------------------
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def spawn_command(n: int, argv: list[str], port: int) -> list[str]:
    """The torchrun re-launch of this script on n ranks (one process per GPU)."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
            "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *argv]


def spawn(n: int, argv: list[str]) -> int:
    """`--gpus N` without torchrun: re-launch under torch.distributed.run and pass its exit
    code on (rank 0's JSON line is the only stdout line)."""
    env = dict(os.environ, ORION_BENCH_SPAWNED="1")
    return subprocess.run(spawn_command(n, argv, free_port()), env=env).returncode


def dist_initialized() -> bool:
    import torch.distributed as dist
    return dist.is_available() and dist.is_initialized()


def backend_name() -> str:
    """ORION_BENCH_BACKEND=gloo only exists to exercise the multi-rank control flow on one GPU
    (ranks then share device local % device_count) or on CPU (--plumbing-check)."""
    return os.environ.get("ORION_BENCH_BACKEND", "nccl")


def init_dist(world: int, local: int) -> int:
    """One process per GPU: bind the device and (N > 1) the process group."""
    import torch
    import torch.distributed as dist
    backend = backend_name()
    dev = local % max(1, torch.cuda.device_count()) if backend != "nccl" else local
    torch.cuda.set_device(dev)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
    return dev


# ---- the CPU oracle timed on the host (a baseline, not the target) ------------------------------
_SLAB_CACHE: dict = {}


def _oracle_slab(W, H, sigma):
    import synth
    y0 = H // 2
    key = (W, H, sigma)
    if key not in _SLAB_CACHE:   # the input slab is drawn once, outside any timing
        _SLAB_CACHE[key] = synth.noisy_rgba(W, H, seed=1, sigma=sigma, row_begin=y0 - 6, row_end=y0 + 6 + 1024)
    return y0, _SLAB_CACHE[key]


def cpu_baseline_nlm(kind: str, W: int, H: int, sigma: float, budget_s: float):
    """The oracle (C, double, single thread) timed on a bounded row band of the same frame."""
    import oracle
    rows_per = 2 if kind == "nlm" else 16
    y0, img = _oracle_slab(W, H, sigma)
    t0 = time.perf_counter()
    n = 0
    y = y0
    while True:
        oracle.denoise(kind, img, height=H, row0=y0 - 6, y_begin=y, y_end=min(H, y + rows_per))
        n += min(H, y + rows_per) - y
        y += rows_per
        dt = time.perf_counter() - t0
        if dt >= budget_s or y >= min(H, y0 + 1024):
            break
    return n * W, dt, f"{n} rows x {W} px of the {W}x{H} frame (rows {y0}..{y0 + n}), oracle/denoise.c, double"


def cpu_baseline_nlm_threads(kind: str, W: int, H: int, sigma: float, budget_s: float, threads: int):
    """The same oracle call, unchanged, on `threads` host threads at once (ctypes releases the
    GIL inside the C function): each thread takes the next row chunk of the same slab."""
    import oracle
    rows_per = 2 if kind == "nlm" else 16
    y0, img = _oracle_slab(W, H, sigma)
    span = min(H - y0, 1024)
    lock = threading.Lock()
    state = {"next": 0, "rows": 0}
    t0 = time.perf_counter()

    def worker():
        while time.perf_counter() - t0 < budget_s:
            with lock:
                k = state["next"]
                state["next"] += 1
            y = y0 + (k * rows_per) % span
            y1 = min(y0 + span, y + rows_per)
            oracle.denoise(kind, img, height=H, row0=y0 - 6, y_begin=y, y_end=y1)
            with lock:
                state["rows"] += y1 - y

    ts = [threading.Thread(target=worker) for _ in range(threads)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    dt = time.perf_counter() - t0
    return state["rows"] * W, dt, f"{state['rows']} rows x {W} px of the {W}x{H} frame on {threads} threads"


def host_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def cpu_baseline_srad(W: int, steps: int, budget_s: float):
    import oracle
    import synth
    rows = 128
    t0a, _ = synth.thermal_inputs(W, rows, seed=1)
    t0 = time.perf_counter()
    n = 0
    while True:
        oracle.srad(t0a.astype("float64"), steps, 0.5, (0, 127, 0, 127))
        n += 1
        dt = time.perf_counter() - t0
        if dt >= budget_s:
            break
    return n * rows * W * steps, dt, f"{n} x ({rows} x {W} cells x {steps} iterations), oracle/srad.c f64"


def cpu_baseline_hotspot(W: int, steps: int, budget_s: float):
    import oracle
    import synth
    rows = 64
    t0a, pw = synth.thermal_inputs(W, rows, seed=1)
    t0 = time.perf_counter()
    n = 0
    while True:
        oracle.hotspot(t0a, pw, steps, precision="f64")
        n += 1
        dt = time.perf_counter() - t0
        if dt >= budget_s:
            break
    return n * rows * W * steps, dt, f"{n} x ({rows} x {W} cells x {steps} steps), oracle/stencil.c f64"


def cpu_baseline(kernel: str, wl: dict, seconds: float, all_cores: bool):
    """The oracle as it stands on a bounded sample of the workload (rank 0, N = 1)."""
    W, H = wl["W"], wl["H"]
    if kernel.startswith("hotspot"):
        u, dt, sample = cpu_baseline_hotspot(W, 1, seconds)
    elif kernel.startswith("srad"):
        u, dt, sample = cpu_baseline_srad(W, 1, seconds)
    else:
        u, dt, sample = cpu_baseline_nlm("knn" if kernel.startswith("knn") else "nlm", W, H, wl["sigma"], seconds)
    cpu = {"value": u / dt / 1e6, "unit": wl["unit"], "cores": 1, "kind": "oracle", "sample": sample}
    if all_cores and not (kernel.startswith("hotspot") or kernel.startswith("srad")) and host_threads() > 1:
        nt = host_threads()   # also row-parallel on every host core
        u2, dt2, sample2 = cpu_baseline_nlm_threads("knn" if kernel.startswith("knn") else "nlm", W, H, wl["sigma"],
                                                    seconds, nt)
        cpu["all_cores"] = {"value": u2 / dt2 / 1e6, "unit": wl["unit"], "cores": nt, "kind": "oracle",
                            "sample": sample2}
    return cpu


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, timed on bounded samples (rank 0 only)."""
    world, rank, _ = dist_env()
    if rank != 0:
        return
    wl = WORKLOADS[args.workload if world == 1 else "c5"]
    K, Wm = args.steps or 5, args.warmup
    per_step = max(0.2, min(2.0, 150.0 / max(1, K + Wm)))
    times, units = [], []
    sample = ""
    for s in range(Wm + K):
        if wl["kernel"].startswith("hotspot"):
            u, dt, sample = cpu_baseline_hotspot(wl["W"], 1, per_step)
        elif wl["kernel"].startswith("srad_f32"):
            u, dt, sample = cpu_baseline_srad(wl["W"], 1, per_step)
        else:
            u, dt, sample = cpu_baseline_nlm("knn" if wl["kernel"].startswith("knn") else "nlm", wl["W"], wl["H"],
                                             wl.get("sigma", 0.13), per_step)
        if s >= Wm:
            times.append(dt)
            units.append(u)
    value = sum(units) / sum(times) / 1e6
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": wl["unit"], "n_gpus": world,
            "steps": K, "warmup": Wm, "ms_per_step": 1e3 * sum(times) / len(times), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl["name"], "impl": "CPU oracle (plain C, double), single thread"},
            "cpu_baseline": {"value": value, "unit": wl["unit"], "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": wl["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---- one configuration on one GPU ---------------------------------------------------------------
def _roofline(kernel, wl, units_per_launch, kernel_ms):
    peaks, peak_kind = load_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    stencil = kernel.startswith("hotspot") or kernel.startswith("srad")
    if stencil:
        achieved = wl["bytes"] * units_per_launch / (kernel_ms * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / peaks["hbm_gbs"], "peak_kind": peak_kind + " (copy bandwidth)"}
    else:
        peak = 148 * 128 * sm_max * 1e6 / 1e12
        achieved = wl["insts"] * units_per_launch / (kernel_ms * 1e-3) / 1e12
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tinst/s (FP32 pipe lane-ops)",
                "frac": achieved / peak,
                "peak_kind": f"derived: 148 SM x 128 FP32 lanes x {sm_max:.0f} MHz (sm_max_mhz, {peak_kind})",
                "hbm_frac": wl["bytes"] * units_per_launch / (kernel_ms * 1e-3) / 1e9 / peaks["hbm_gbs"]}
    roof["traffic"] = None
    prof = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                ent = json.load(f).get(kernel) or {}
            roof["traffic"] = ent.get("dram_bytes_per_launch")
            m = ent.get("metrics", {})

            def num(k):
                return float(m[k].split()[0].replace(",", ""))
            wf = num("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum")
            dur = num("gpu__time_duration.sum") * {"ns": 1e-9, "us": 1e-6, "ms": 1e-3}.get(
                m["gpu__time_duration.sum"].split()[-1][:2], 1e-6)
            sm_hz = num("sm__cycles_elapsed.avg.per_second") * 1e9
            roof["ncu"] = {"report": ent.get("report"), "smem_wavefront_frac": wf / (148 * dur * sm_hz),
                           "issue_active_pct": num("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                           "lsu_pipe_pct": num("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"),
                           "fma_pipe_pct": num("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active")}
        except Exception:
            pass
    roof["kernel"] = kernel
    roof["algorithmic_per_unit"] = wl["insts"] if not stencil else wl["bytes"]
    return roof


def measure_single(key: str, args, *, steps: int, warmup: int, rounds: int, cpu_seconds: float,
                   carveout_axis: bool, kernel: str | None = None, select: str = "fastest", world: int = 1,
                   rank: int = 0, local: int = 0):
    """Build, sweep, tune and time one configuration on this rank's GPU.  Returns the record
    (rank 0) -- the same keys as the headline line."""
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_hayeslcsz16_b200 import orion as O

    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    sp = stream.cuda_stream
    wl = WORKLOADS[key]
    kernel, W, H = kernel or wl["kernel"], wl["W"], wl["H"]
    # frames per launch / step (orion_args.batch): --batch for the headline workload, else the
    # workload's default (C1: 256)
    batch = max(1, args.batch if args.batch > 0 and key == args.workload else wl.get("batch", 1))
    if is_stencil_id(kernel):
        batch = 1
    threads = wl.get("threads", 0) if kernel == wl["kernel"] else 0
    is_srad = kernel.startswith("srad_f32")
    is_stencil = kernel.startswith("hotspot") or is_srad
    fused = kernel == "srad_f32hs"
    # launch-bound frames (C1 by default) replay their settled iterations as one CUDA graph,
    # whose kernel nodes are plain launches: the whole configuration (sweep included) then runs
    # without programmatic dependent launch, so every level is timed the way the loop runs it
    graph_loop = (args.graph == "on" or (args.graph == "auto" and key == "c1")) and not is_stencil
    pdl_prev = O.set_pdl(False) if graph_loop else None

    # ---- multi-version binary: probe -> levels -> build (offline, untimed) ----------------
    t_build = time.perf_counter()
    realise = O.REALISE_MIN_CARVEOUT if args.realise == "min" else O.REALISE_MAX_SMEM
    variants, res = O.build_all_levels(local, kernel, block_threads=threads, mode=realise)
    t_build = time.perf_counter() - t_build
    nlev = len(variants)
    lv = [variants.level(i) for i in range(nlev)]
    infos = [variants.info(i) for i in range(nlev)]
    orig = max((i for i, l in enumerate(variants.planned) if l.reg_cap == 0),
               key=lambda i: variants.planned[i].ctas_per_sm)   # the original / nvcc-default build
    kmax = nlev - 1

    # ---- inputs resident in HBM: a pool of frames larger than L2 -------------------------
    chain = None
    frame_bytes = W * H * (4 if is_stencil else 16)
    # frames (or, batched, batches of frames) in the pool: inputs + outputs larger than L2
    nframes = max(2, math.ceil(2 * 126e6 / (2 * frame_bytes * batch)) + 1)
    if is_stencil:
        nframes = 1
        # srad_f32hs: the ROI statistics slots travel behind each grid
        extra = O.SRAD_STATS_FLOATS if fused else 0
        t_a = torch.empty(H * W + extra, device=dev)[:H * W].view(H, W)
        t_b = torch.empty(H * W + extra, device=dev)[:H * W].view(H, W)
        pw = torch.empty((H, W), device=dev)
        O.generate_thermal(local, t_a.data_ptr(), pw.data_ptr(), W, H, seed=1 + rank, stream=sp)
        if fused:
            O.srad_stats_init(local, t_a.data_ptr(), W, H, ROI, sp)
        state = {"a": t_a, "b": t_b}
        q0 = torch.empty(1, device=dev)   # srad: the ROI statistic of the current iteration

        # consecutive iterations overlapped tile by tile (orion_chain) where the family allows it;
        # the sweep below repeats one launch and runs unchained
        chain = O.Chain(variants, W, H) if kernel in O.CHAINABLE and not args.no_chain else None

        def grid_args(src, dst, ch=None):
            if is_srad:
                return O.srad_args(src.data_ptr(), dst.data_ptr(), 0 if fused else q0.data_ptr(), W, H,
                                   roi=ROI if fused else None, chain=ch)
            return O.hotspot_args(src.data_ptr(), dst.data_ptr(), pw.data_ptr(), W, H, chain=ch)

        def step_args(s):
            if is_srad and not fused:   # the iteration's ROI statistics precede the tuned update kernel
                O.srad_roi_stats(local, state["a"].data_ptr(), W, H, ROI, q0.data_ptr(), sp)
            a = grid_args(state["a"], state["b"], chain)
            state["a"], state["b"] = state["b"], state["a"]
            return a
    else:
        shape = (batch, H, W, 4) if batch > 1 else (H, W, 4)
        srcs = [torch.empty(shape, device=dev) for _ in range(nframes)]
        dsts = [torch.empty(shape, device=dev) for _ in range(nframes)]
        for f, t in enumerate(srcs):
            for b_ in range(batch):
                fr = t[b_] if batch > 1 else t
                O.generate_rgba(local, fr.data_ptr(), W, H, seed=1 + f * batch + b_ + 97 * rank, sigma=wl["sigma"],
                                stream=sp)

        def step_args(s, independent=True):
            # consecutive frames (batches) live in their own buffers (nframes >= 2): each launch is
            # independent of the stream's previous one (ORION_ARGS_INDEPENDENT), so with PDL a
            # frame's CTAs start in the previous frame's last wave
            f = s % nframes
            return O.denoise_args(kernel, srcs[f].data_ptr(), dsts[f].data_ptr(), W, H,
                                  independent=independent and nframes > 1, batch=batch)
    torch.cuda.synchronize()

    # ---- exhaustive sweep (brute-force reference, Fig. 11 Orion-Max/Min) ------------------
    # (repeats one frame: not independent launches)
    sweep_args = step_args(0) if is_stencil else step_args(0, independent=False)
    if is_stencil:
        state["a"], state["b"] = t_a, t_b
        if is_srad and not fused:
            O.srad_roi_stats(local, t_a.data_ptr(), W, H, ROI, q0.data_ptr(), sp)
        sweep_args = grid_args(t_a, t_b)
    ms = variants.sweep(sweep_args, sp, rounds=rounds)
    best = min(range(nlev), key=lambda i: ms[i])
    worst = max(range(nlev), key=lambda i: ms[i])
    caxis = None
    if carveout_axis:   # the carveout axis (Table 3 analogue): the same levels realised the other way
        other = O.REALISE_MAX_SMEM if realise == O.REALISE_MIN_CARVEOUT else O.REALISE_MIN_CARVEOUT
        v2, _ = O.build_all_levels(local, kernel, mode=other)
        ms2 = v2.sweep(sweep_args, sp, rounds=rounds)
        caxis = {"realise": "min_carveout" if other == O.REALISE_MIN_CARVEOUT else "max_smem",
                 "levels": [{"k": v2.level(i).ctas_per_sm, "carveout_kb": v2.level(i).carveout_kb,
                             "pad": v2.level(i).smem_pad_bytes, "ms": round(ms2[i], 5)} for i in range(len(v2))],
                 "ms_best": min(ms2)}
        v2.close()

    # ---- the tuned loop: warmup (includes Fig. 9 exploration) then K timed steps ----------
    cfg = O.default_cfg(select_mode=O.SELECT_LOWEST_WITHIN_TOL if select == "lowest" else O.SELECT_FASTEST,
                        samples_per_level=args.samples, async_timing=int(args.async_timing))
    tuner = O.Tuner(variants, cfg)
    direction, ladder = tuner.ladder()
    if is_stencil:
        state["a"], state["b"] = t_a, t_b
    step = 0
    explore_ms = []
    ran_levels = []
    settle_extra = 0
    while True:
        # W warm-up iterations, extended (if need be) until Fig. 9 has set the final kernel: the
        # timed region measures the settled loop; exploration is charged in fig11's Orion-Select
        if step >= warmup and (tuner.final()[0] >= 0 or settle_extra >= 500):
            break
        r = tuner.step(step_args(step), sp)
        ran_levels.append(r.level_idx)
        if r.phase == 0 and r.ms >= 0:
            explore_ms.append(r.ms)
        if step >= warmup:
            settle_extra += 1
        step += 1
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n_launch0 = O.launch_count()
    # launch-bound frames (C1 by default): the K settled iterations replay as one CUDA graph.
    use_graph = graph_loop and tuner.final()[0] >= 0
    native = not use_graph and args.graph == "native"
    graph = None
    native_args = None
    if use_graph:
        # the settled frames are independent (ORION_ARGS_INDEPENDENT): captured with PDL on, the
        # graph keeps programmatic edges and consecutive 64^2 frames run concurrently (the sweep
        # and the tuner's exploration above ran without PDL)
        O.set_pdl(True)
        graph = tuner.capture([step_args(step + k) for k in range(steps)])
        step += steps
        torch.cuda.synchronize()
    elif native:
        native_args = [step_args(step + k) for k in range(steps)]
        step += steps
    remeasured = None
    for attempt in range(2):
        n_launch0 = O.launch_count()
        torch.cuda.nvtx.range_push("timed")   # the launch list (ncu --nvtx-include "timed/") covers only this
        with ClockSampler(local) as clk:
            e0.record(stream)
            if graph is not None:
                graph.launch(sp)
            elif native_args is not None:
                tuner.steps(native_args, sp)
            else:
                for _ in range(steps):
                    tuner.step(step_args(step), sp)
                    step += 1
            e1.record(stream)
            torch.cuda.synchronize()
            clk.mark_end()
        torch.cuda.nvtx.range_pop()
        # a timed region that saw a hardware / thermal slowdown is not a measurement: measure it
        # once more (the same K steps), and keep what the second run saw
        bad = sorted(THROTTLE_REJECT & set(clk.summary()["reasons"]))
        flag = torch.tensor([1 if bad else 0], device=dev)
        if world > 1:
            dist.all_reduce(flag, op=dist.ReduceOp.MAX)
        if not int(flag.item()) or attempt == 1:
            break
        remeasured = {"first_run_reasons": bad}
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    if graph is not None:
        graph.close()
    launches = O.launch_count() - n_launch0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    total_ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([total_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    final, iters_to_final = tuner.final()
    spl = O.STEPS_PER_LAUNCH.get(kernel, 1)                # stencil steps per launch (temporal blocking)
    units_per_step = W * H * spl * batch
    value = world * units_per_step * steps / (total_ms * 1e-3) / 1e6
    ms_step = total_ms / steps
    t_final = ms[final] if final >= 0 else float("nan")

    # ---- end to end through the C ABI with pinned host buffers ---------------------------
    if not is_stencil:
        # orion_host_pipe: every step copies its frame host->device, runs the tuned kernel and
        # copies the result device->host; H2D(n+1) / kernel(n) / D2H(n-1) overlap on the pipe's
        # three streams.  The synchronous orion_tune_step_host is reported beside it.
        host_in = [srcs[f].cpu().pin_memory() for f in range(2)]
        host_out = [torch.empty(srcs[0].shape).pin_memory() for _ in range(2)]
        has = [O.denoise_args(kernel, host_in[f].data_ptr(), host_out[f].data_ptr(), W, H, batch=batch)
               for f in range(2)]
        n_e2e = max(4, min(steps, 60 if frame_bytes * batch > 1 << 20 else 2000))
        pipe = O.HostPipe(tuner, W, H * batch, depth=3)
        for f in range(2):
            pipe.submit(has[f])                                                    # warm
        pipe.drain()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        hi = ho = 0
        for s_ in range(n_e2e):
            _, hi, ho = pipe.submit(has[s_ % 2])
        pipe.drain()
        dt = time.perf_counter() - t0
        pipe.close()
        t0 = time.perf_counter()
        n_sync = max(3, n_e2e // 4)
        for s_ in range(n_sync):
            tuner.step_host(has[s_ % 2], srcs[0].data_ptr(), dsts[0].data_ptr(), stream=sp)
        dt_sync = time.perf_counter() - t0
        if world > 1:
            t = torch.tensor([dt, dt_sync], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt, dt_sync = (float(x) for x in t.tolist())
        e2e = {"value": world * W * H * batch * n_e2e / dt / 1e6, "unit": wl["unit"], "h2d_bytes_per_step": hi,
               "d2h_bytes_per_step": ho, "steps": n_e2e, "api": "orion_host_pipe (depth 3, pinned host frames)",
               "sync_api_value": world * W * H * batch * n_sync / dt_sync / 1e6}
        del host_in, host_out
    else:
        # a whole run per job (orion_tune_run_host): host grids -> device, the config's 100
        # time steps under a FRESH tuner (its exploration included), final grid -> host
        launches_per_job = 100 // spl
        h_t = t_a.cpu().pin_memory()
        h_p = pw.cpu().pin_memory()
        h_o = torch.empty((H, W)).pin_memory()
        if is_srad:
            ja = O.srad_args(h_t.data_ptr(), h_o.data_ptr(), 0, W, H)
            aux_dev, roi = q0, ROI
        else:
            ja = O.hotspot_args(h_t.data_ptr(), h_o.data_ptr(), h_p.data_ptr(), W, H)
            aux_dev, roi = pw, None
        jobs = 2
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        hi = ho = 0
        for _ in range(jobs):
            jt = O.Tuner(variants, cfg)
            hi, ho = jt.run_host(ja, launches_per_job, t_b.data_ptr(), t_a.data_ptr(), aux_dev.data_ptr(), roi, sp)
            jt.close()
        dt = time.perf_counter() - t0
        if world > 1:
            t = torch.tensor([dt], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t.item())
        e2e = {"value": world * W * H * spl * launches_per_job * jobs / dt / 1e6, "unit": wl["unit"],
               "h2d_bytes_per_step": hi / launches_per_job, "d2h_bytes_per_step": ho / launches_per_job,
               "steps": launches_per_job * jobs,
               "api": f"orion_tune_run_host ({jobs} runs of {launches_per_job} launches from pinned host grids, "
                      f"a fresh tuner per run)"}

    rec = None
    if rank == 0:
        cpu = None
        if world == 1 and cpu_seconds > 0:
            cpu = cpu_baseline(kernel, wl, cpu_seconds, all_cores=True)
        # Orion-Select (Fig. 11, P:L747-P:L755) = the tuned run INCLUDING its exploration: every
        # iteration charged the sweep time of the level it ran (one timing method for all bars)
        horizon = ran_levels + [final] * steps      # warm-up (incl. any extension) + timed iterations
        select_ms = sum(ms[i] for i in horizon) / len(horizon)
        lvl_rows = [{"k": lv[i].ctas_per_sm, "occ": lv[i].occupancy_permille / 1000, "reg_cap": lv[i].reg_cap,
                     "regs": infos[i].regs, "pad": lv[i].smem_pad_bytes, "carveout_kb": lv[i].carveout_kb,
                     "spill_st": infos[i].spill_store, "ms": round(ms[i], 5)} for i in range(nlev)]
        rec = {
            "metric": METRIC, "value": value, "unit": wl["unit"], "n_gpus": world, "steps": steps,
            "warmup": warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": wl["name"], "baseline_config_index": wl["cfg_index"], "kernel": kernel,
                       "block_threads": res.block_threads, "width": W, "height": H, "frames_per_step": batch, "frames_in_pool": nframes * batch,
                       "l2": "inputs larger than L2: rotating pool of frames" if not is_stencil else
                             "grids (3 x 256 MiB) > L2 (126 MB)",
                       "parallelism": f"dp{world} (independent frames per GPU)",
                       "cuda_graph": graph is not None,
                       "overlap": ("orion_chain (tile-level waits between iterations)" if chain is not None else
                                   "none (each iteration waits for the whole previous grid)") if is_stencil else
                                  ("independent frames (ORION_ARGS_INDEPENDENT: no grid-wide wait)"
                                   if nframes > 1 and graph is None else "none"),
                       "issue": "graph" if graph is not None else ("orion_tune_steps" if native_args is not None
                                                                   else "orion_tune_step per step")},
            "roofline": _roofline(kernel, wl, W * H * batch, ms_step),      # bytes / instructions per cell or pixel per launch
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": dict(clk.summary(), remeasured=remeasured),
            "energy": clk.energy(steps), "select_mode": select,
            "resources": {"final_regs": infos[final].regs if final >= 0 else None,
                          "natural_regs": res.regs_per_thread,
                          "final_warps_per_sm": lv[final].warps_per_sm if final >= 0 else None,
                          "best_warps_per_sm": lv[best].warps_per_sm,
                          "register_file_used_frac": (infos[final].regs * lv[final].warps_per_sm * 32 / 65536)
                          if final >= 0 else None},
            "tuner": {"direction": "increasing" if direction == 1 else "decreasing",
                      "ladder_k": [lv[i].ctas_per_sm for i in ladder],
                      "final_k": lv[final].ctas_per_sm if final >= 0 else None,
                      "final_occupancy": lv[final].occupancy_permille / 1000 if final >= 0 else None,
                      "iterations_to_final": iters_to_final, "explore_ms": explore_ms,
                      "explored_k": [lv[i].ctas_per_sm for i in ran_levels[:max(0, iters_to_final)]],
                      "samples_per_level": args.samples, "async_timing": bool(args.async_timing),
                      "warmup_extended_by": settle_extra},
            "sweep": {"rounds": rounds, "n_levels": nlev, "levels": lvl_rows, "best_k": lv[best].ctas_per_sm,
                      "ms_best": ms[best], "worst_k": lv[worst].ctas_per_sm, "ms_worst": ms[worst],
                      "maxocc_k": lv[kmax].ctas_per_sm, "ms_maxocc": ms[kmax],
                      "nvcc_default_k": lv[orig].ctas_per_sm, "ms_nvcc_default": ms[orig]},
            "regret": t_final / ms[best] - 1.0,
            "fig11": {"orion_min_ms": ms[worst], "orion_max_ms": ms[best], "nvcc_ms": ms[orig],
                      "orion_select_ms": select_ms, "speedup_select_vs_nvcc": ms[orig] / select_ms,
                      "speedup_max_vs_nvcc": ms[orig] / ms[best], "speedup_min_vs_nvcc": ms[orig] / ms[worst],
                      "note": "every bar timed by orion_sweep (interleaved rounds); Orion-Select charges each "
                              "warm-up + timed iteration the sweep time of the level it ran"},
            "vs_maxocc": ms[kmax] / t_final,
            "vs_nvcc_default": ms[orig] / t_final,
            "build_seconds": round(t_build, 2),
            "realise": "min_carveout" if realise == O.REALISE_MIN_CARVEOUT else "max_smem",
            "carveout_axis": caxis,
        }
    torch.cuda.synchronize()
    if chain is not None:
        chain.close()
    tuner.close()
    variants.close()
    if graph_loop:
        O.set_pdl(pdl_prev)
    torch.cuda.empty_cache()
    return rec


# ---- NEXT-3: resource-saving selection and energy (Fig. 12 / 13 analogues) ---------------------
def measure_energy(key: str, args, kernel: str, local: int = 0, window_s: float = 1.2):
    """Fig. 12 (registers saved, P:L873-P:L939) and Fig. 13 (energy, P:L943-P:L979) analogues for
    one configuration: the level LOWEST_WITHIN_TOL selects (the paper's resource-saving reading,
    R-A4), the level FASTEST selects, the exhaustive-best and the max-occupancy level; each is
    replayed as a CUDA graph of its settled iterations over NVML windows >= `window_s` s."""
    import torch
    from paper_conf_middleware_hayeslcsz16_b200 import orion as O

    sp = torch.cuda.current_stream().cuda_stream
    wl = WORKLOADS[key]
    W, H = wl["W"], wl["H"]
    is_srad = kernel.startswith("srad")
    is_stencil = kernel.startswith("hotspot") or is_srad
    fused = kernel == "srad_f32hs"
    realise = O.REALISE_MIN_CARVEOUT if args.realise == "min" else O.REALISE_MAX_SMEM
    pdl_prev = O.set_pdl(False)          # every level below is replayed as a CUDA graph (plain launches)
    batch = wl.get("batch", 1) if kernel == wl["kernel"] else 1
    v, res = O.build_all_levels(local, kernel, block_threads=wl.get("threads", 0) if kernel == wl["kernel"] else 0,
                                mode=realise)
    n = len(v)
    if is_stencil:
        extra = O.SRAD_STATS_FLOATS if fused else 0
        a_ = torch.empty(H * W + extra, device="cuda")[:H * W].view(H, W)
        b_ = torch.empty(H * W + extra, device="cuda")[:H * W].view(H, W)
        p_ = torch.empty((H, W), device="cuda")
        O.generate_thermal(local, a_.data_ptr(), p_.data_ptr(), W, H, seed=1, stream=sp)
        q0 = torch.empty(1, device="cuda")
        if fused:
            O.srad_stats_init(local, a_.data_ptr(), W, H, ROI, sp)
            O.srad_stats_init(local, b_.data_ptr(), W, H, ROI, sp)
            args_pp = [O.srad_args(a_.data_ptr(), b_.data_ptr(), 0, W, H, roi=ROI),
                       O.srad_args(b_.data_ptr(), a_.data_ptr(), 0, W, H, roi=ROI)]
        elif is_srad:
            O.srad_roi_stats(local, a_.data_ptr(), W, H, ROI, q0.data_ptr(), sp)
            args_pp = [O.srad_args(a_.data_ptr(), b_.data_ptr(), q0.data_ptr(), W, H),
                       O.srad_args(b_.data_ptr(), a_.data_ptr(), q0.data_ptr(), W, H)]
        else:
            args_pp = [O.hotspot_args(a_.data_ptr(), b_.data_ptr(), p_.data_ptr(), W, H),
                       O.hotspot_args(b_.data_ptr(), a_.data_ptr(), p_.data_ptr(), W, H)]
    else:
        nfr = max(2, math.ceil(2 * 126e6 / (2 * W * H * 16 * batch)) + 1)
        shape = (batch, H, W, 4) if batch > 1 else (H, W, 4)
        srcs = [torch.empty(shape, device="cuda") for _ in range(nfr)]
        dsts = [torch.empty(shape, device="cuda") for _ in range(nfr)]
        for f, t in enumerate(srcs):
            for b_ in range(batch):
                O.generate_rgba(local, (t[b_] if batch > 1 else t).data_ptr(), W, H, seed=1 + f * batch + b_,
                                sigma=wl["sigma"], stream=sp)
        args_pp = [O.denoise_args(kernel, srcs[f].data_ptr(), dsts[f].data_ptr(), W, H, batch=batch)
                   for f in range(nfr)]
    torch.cuda.synchronize()
    ms = v.sweep(args_pp[0], sp, rounds=args.rounds)

    def tuned(mode):
        t = O.Tuner(v, O.default_cfg(select_mode=mode, samples_per_level=args.samples))
        for i in range(200):
            t.step(args_pp[i % len(args_pp)], sp)
            if t.final()[0] >= 0:
                break
        torch.cuda.synchronize()
        f = t.final()[0]
        t.close()
        return f

    lowest = tuned(O.SELECT_LOWEST_WITHIN_TOL)
    fastest = tuned(O.SELECT_FASTEST)
    best = min(range(n), key=lambda i: ms[i])
    picks = {"lowest_within_tol": lowest, "fastest": fastest, "exhaustive_best": best, "max_occupancy": n - 1}
    per_graph = max(1, min(2000, int(math.ceil(20.0 / max(ms[best], 1e-3)))))   # ~20 ms of work per replay
    out = {}
    for name, lvl in picks.items():
        if lvl < 0:
            out[name] = None
            continue
        t = O.Tuner(v, O.default_cfg())
        t.resume(lvl)
        g = t.capture([args_pp[i % len(args_pp)] for i in range(per_graph)])
        g.launch(sp)                                   # warm
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 0
        with ClockSampler(local) as clk:
            e0.record()
            t0 = time.perf_counter()
            while True:
                g.launch(sp)
                reps += 1
                if reps % 8 == 0:
                    torch.cuda.synchronize()
                    if time.perf_counter() - t0 >= window_s:
                        break
            e1.record()
            torch.cuda.synchronize()
            clk.mark_end()
        g.close()
        t.close()
        iters = reps * per_graph
        en = clk.energy(iters)
        L, inf = v.level(lvl), v.info(lvl)
        out[name] = {"k": L.ctas_per_sm, "occupancy": L.occupancy_permille / 1000, "regs": inf.regs,
                     "register_file_frac": inf.regs * L.warps_per_sm * 32 / 65536,
                     "ms_per_iteration": e0.elapsed_time(e1) / iters, "sweep_ms": ms[lvl],
                     "joules_per_iteration": en["joules_per_step"] if en else None,
                     "mean_watts": en["mean_watts"] if en else None, "window_s": en.get("window_s") if en else None,
                     "clocks": clk.summary()}
    rec = {"kernel": kernel, "workload": wl["name"], "natural_regs": res.regs_per_thread, "levels": out,
           "iterations_per_graph": per_graph}
    lo = out.get("lowest_within_tol")
    for ref in ("exhaustive_best", "max_occupancy"):
        fa = out.get(ref)
        if lo and fa:
            c = {"registers_saved_frac": 1.0 - lo["register_file_frac"] / fa["register_file_frac"],
                 "warps_saved_frac": 1.0 - lo["occupancy"] / fa["occupancy"],
                 "runtime_change": lo["ms_per_iteration"] / fa["ms_per_iteration"] - 1.0}
            if lo["joules_per_iteration"] and fa["joules_per_iteration"]:
                c["energy_change"] = lo["joules_per_iteration"] / fa["joules_per_iteration"] - 1.0
            rec[f"lowest_vs_{ref}"] = c
    v.close()
    O.set_pdl(pdl_prev)
    torch.cuda.empty_cache()
    return rec


# ---- C5: the row-sharded frame -------------------------------------------------------------
def measure_c5(args, *, world: int, rank: int, local: int, steps: int, warmup: int, group=None, size: int = 0,
               mode_req: str = "auto", chunks_req: int = 4, e2e: bool = True):
    """One 16384^2 NLM frame row-sharded over the `world` ranks of `group` (strong scaling).  A
    step = every rank's tuned NLM launch on its band (input slab + 6-row halo generated in
    place before the timed region) and the exchange of the output bands into every rank's full
    image.  Returns the record on rank 0 of the group, else None."""
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_hayeslcsz16_b200 import orion as O
    from paper_conf_middleware_hayeslcsz16_b200 import shard

    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    sp = stream.cuda_stream
    wl = WORKLOADS["c5"]
    kernel = args.kernel if args.kernel and args.workload == "c5" else wl["kernel"]
    W = H = size or wl["W"]
    b = shard.band(rank, world, H, 6)
    src = torch.empty((b.src_rows, W, 4), device=dev)
    O.generate_rgba(local, src.data_ptr(), W, H, b.src_begin, b.src_end, seed=1, sigma=wl["sigma"], stream=sp)
    out = torch.empty((b.rows_per_rank, W, 4), device=dev)
    variants, res = O.build_all_levels(local, kernel, mode=O.REALISE_MIN_CARVEOUT if args.realise == "min"
                                       else O.REALISE_MAX_SMEM)
    nlev = len(variants)
    a = O.denoise_args(kernel, src.data_ptr(), out.data_ptr(), W, H, b.row_begin, b.row_end, b.src_begin,
                       b.src_end, b.row_begin)
    ms = variants.sweep(a, sp, rounds=max(3, args.rounds // 3))
    tuner = O.Tuner(variants, O.default_cfg(samples_per_level=args.samples))
    # the exchange: the kernels' fan-out stores into every rank's symmetric-memory image (compute
    # + gather in one kernel over NVLink), else chunked all-gathers overlapped with compute
    # P = 1: no exchange, unless the fan-out or the gather is requested explicitly (either path
    # exercised on one GPU over a one-rank NCCL group, see run_single)
    mode, fan, fan_note = ("none" if world == 1 and mode_req not in ("fanout", "gather") else mode_req), None, None
    full = None
    if mode in ("auto", "fanout"):
        try:
            if backend_name() != "nccl":
                raise RuntimeError("symmetric memory needs the nccl backend")
            fan = shard.FanoutImage((H, W, 4), dev, group)
            a = O.with_fanout(type(a).from_buffer_copy(a), fan.ptrs)
            mode = "fanout"
        except Exception as ex:   # no symmetric memory on this group / backend
            if mode == "fanout":
                raise
            mode, fan_note = "gather", f"fan-out unavailable ({type(ex).__name__}: {ex}); chunked all-gather used"
    if mode == "gather":
        full = torch.empty((world * b.rows_per_rank, W, 4), device=dev)
    chunks = max(1, chunks_req) if mode == "gather" else 1
    plan = shard.chunk_plan(b, chunks)     # the same gathered rows on every rank
    comm = torch.cuda.Stream() if mode == "gather" else None

    def one_step(ev=None, recorded=None):
        """Compute the band (as `chunks` row chunks when gathering) and exchange it."""
        if mode == "fanout":
            tuner.step(a, sp)                 # stores its band into every rank's image
            if ev is not None:
                ev[1].record(stream)
            fan.barrier()                     # every rank's stores have landed
            return
        if mode == "none":
            tuner.step(a, sp)
            if ev is not None:
                ev[1].record(stream)
            return
        for r0, r1, k0, k1 in plan:
            ca = O.denoise_args(kernel, src.data_ptr(), out.data_ptr(), W, H, b.row_begin + k0, b.row_begin + k1,
                                b.src_begin, b.src_end, b.row_begin)
            ce = None
            if recorded is not None and k0 < k1:
                ce = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                ce[0].record(stream)
            tuner.step(ca, sp)
            if ce is not None:
                ce[1].record(stream)
                recorded.append(ce)
            comm.wait_stream(stream)
            with torch.cuda.stream(comm):
                shard.gather_rows(out, full, b.rows_per_rank, r0, r1, group=group)
        if ev is not None:
            ev[1].record(stream)
        stream.wait_stream(comm)

    def all_settled():
        ok = torch.tensor([1 if tuner.final()[0] >= 0 else 0], device=dev)
        if world > 1:          # every rank runs the same number of steps (the exchange is collective)
            dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
        return bool(ok.item())

    done = 0
    while done < warmup or (done < warmup + 500 and not all_settled()):
        one_step()                    # warm-up, extended until every rank's Fig. 9 has set its final kernel
        done += 1
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier(group=group)
    remeasured = None
    for attempt in range(2):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
               torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        recorded = [] if mode == "gather" else None
        n0 = O.launch_count()
        with ClockSampler(local) as clk:
            for e in ev:
                e[0].record(stream)
                one_step(e, recorded)
                e[2].record(stream)
            torch.cuda.synchronize()
            clk.mark_end()
        bad = sorted(THROTTLE_REJECT & set(clk.summary()["reasons"]))   # a slowed-down region: once more
        flag = torch.tensor([1 if bad else 0], device=dev)
        if world > 1:
            dist.all_reduce(flag, op=dist.ReduceOp.MAX, group=group)
        if not int(flag.item()) or attempt == 1:
            break
        remeasured = {"first_run_reasons": bad}
        if world > 1:
            dist.barrier(group=group)
    launches = O.launch_count() - n0
    tot = ev[0][0].elapsed_time(ev[-1][2])
    if recorded is not None:
        comp = sum(x.elapsed_time(y) for (x, y) in recorded)
    else:
        comp = sum(e0.elapsed_time(e1) for e0, e1, _ in ev)
    gat = sum(e1.elapsed_time(e2) for _, e1, e2 in ev)   # the exchange tail not hidden by compute

    # ---- end to end: pinned host slab -> device, tuned step + exchange, own band -> host -------
    e2e_rec = None
    if e2e:
        h_src = torch.empty((b.src_rows, W, 4), pin_memory=True)
        h_src.copy_(src)
        h_out = torch.empty((b.rows, W, 4), pin_memory=True)
        n_e2e = max(2, min(steps, 4))
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier(group=group)
        t0 = time.perf_counter()
        for _ in range(n_e2e):
            src.copy_(h_src, non_blocking=True)
            one_step()
            h_out.copy_(out[:b.rows], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        e2e_rec = [dt, float(b.src_rows * W * 16), float(b.rows * W * 16), n_e2e]
        del h_src, h_out
    t = torch.tensor([tot, comp, gat] + ([e2e_rec[0]] if e2e_rec else [0.0]), device=dev)
    final, it = tuner.final()
    chosen = [variants.level(final).ctas_per_sm if final >= 0 else -1, it,
              variants.level(min(range(nlev), key=lambda k: ms[k])).ctas_per_sm, b.row_begin, b.row_end]
    byts = torch.tensor([e2e_rec[1], e2e_rec[2]] if e2e_rec else [0.0, 0.0], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        dist.all_reduce(byts, op=dist.ReduceOp.SUM, group=group)
        allc = [None] * world
        dist.all_gather_object(allc, chosen, group=group)
    else:
        allc = [chosen]
    tot, comp, gat, e2e_dt = (float(x) for x in t.tolist())
    rec = None
    if rank == 0:
        kernel_ms = comp / steps
        roof = _roofline(kernel, wl, b.rows * W, kernel_ms)
        roof["note"] = "per rank: rank 0's band of rows per kernel millisecond"
        rec = {
            "metric": METRIC, "value": H * W * steps / (tot * 1e-3) / 1e6, "unit": "Mpix/s", "n_gpus": world,
            "steps": steps, "warmup": warmup, "ms_per_step": tot / steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": wl["name"], "baseline_config_index": 4, "kernel": kernel, "width": W, "height": H,
                       "rows_per_rank": b.rows_per_rank, "halo_rows": 6,
                       "collective": ("kernel fan-out stores into every rank's symmetric-memory image over NVLink "
                                      "+ device barrier" if mode == "fanout" else
                                      f"all_gather of {chunks} row chunks on a side stream, overlapped with the "
                                      f"next chunk's kernel" if mode == "gather" else "none (P=1)")
                       if world > 1 or mode in ("fanout", "gather") else "none (P=1)",
                       "collective_note": fan_note, "l2": "4 GiB frame >> L2",
                       "parallelism": f"row-sharded x{world}",
                       "backend": backend_name() if world > 1 or mode != "none" else None},
            "compute_only": {"value": H * W * steps / (comp * 1e-3) / 1e6, "unit": "Mpix/s",
                             "ms_per_step": comp / steps},
            "exchange_ms_per_step": gat / steps,
            "roofline": roof,
            "per_rank": [{"rank": r, "final_k": c[0], "iterations_to_final": c[1], "sweep_best_k": c[2],
                          "rows": [c[3], c[4]]} for r, c in enumerate(allc)],
            "sweep_rank0": [{"k": variants.level(i).ctas_per_sm, "ms": round(ms[i], 4)} for i in range(nlev)],
            "regret_rank0": (ms[final] / min(ms) - 1.0) if final >= 0 else None,
            "gpu_launches": launches, "clocks": dict(clk.summary(), remeasured=remeasured), "energy": clk.energy(steps),
            "e2e": ({"value": H * W * e2e_rec[3] / e2e_dt / 1e6, "unit": "Mpix/s",
                     "h2d_bytes_per_step": float(byts[0]), "d2h_bytes_per_step": float(byts[1]),
                     "steps": e2e_rec[3],
                     "api": "per rank: pinned host slab (+ halo) -> device, orion_tune_step + exchange, "
                            "own output band -> pinned host; bytes summed over ranks"} if e2e_rec else None),
            "cpu_baseline": None,
        }
    tuner.close()
    variants.close()
    del src, out, full, fan
    torch.cuda.empty_cache()
    return rec


# ---- C3 row-sharded: the thermal stencil with a halo exchange per launch ------------------------
def measure_c3_sharded(args, *, world: int, rank: int, local: int, steps: int, warmup: int, group=None,
                       size: int = 0, e2e: bool = True):
    """The 8192^2 thermal stencil row-sharded over the `world` ranks (strong scaling; SURVEY 8(e)'s
    NEXT item): each rank runs its tuner on its band (+ 4 halo rows per side) with `hotspot4h_f32`,
    whose launches store their first / last 4 rows into the neighbours' next slabs (symmetric memory
    over NVLink; fallback: an all-gather of the boundary rows); one device barrier per launch.
    A step = one 4-step launch on every rank + the exchange."""
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_hayeslcsz16_b200 import orion as O
    from paper_conf_middleware_hayeslcsz16_b200 import shard

    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    sp = stream.cuda_stream
    wl = WORKLOADS["c3"]
    kernel = "hotspot4h_f32"
    S = O.STEPS_PER_LAUNCH[kernel]
    W = H = size or wl["W"]
    bands = [shard.band(r, world, H, S) for r in range(world)]
    b = bands[rank]
    if world > 1 and min(x.rows for x in bands if x.rows) < S:
        raise SystemExit("bench.py: C3 bands must hold at least 4 rows")
    rows_max = max(x.src_rows for x in bands)
    # initial grid and power map: the generator's whole grid, this rank's slab copied out (untimed)
    full_t = torch.empty((H, W), device=dev)
    full_p = torch.empty((H, W), device=dev)
    O.generate_thermal(local, full_t.data_ptr(), full_p.data_ptr(), W, H, seed=1, stream=sp)
    pw = full_p[b.src_begin:b.src_end].clone()
    t0_slab = full_t[b.src_begin:b.src_end].clone()
    del full_t, full_p
    mode, note, slabs = "none", None, None
    if world > 1:
        try:
            if backend_name() != "nccl":
                raise RuntimeError("symmetric memory needs the nccl backend")
            slabs = shard.SymmetricSlabs(rows_max, W, dev, group)
            bufs = slabs.tensors
            mode = "fanout"
        except Exception as ex:
            mode, note = "gather", f"symmetric memory unavailable ({type(ex).__name__}: {ex}); all-gather of halo rows"
    if slabs is None:
        bufs = [torch.empty((rows_max, W), device=dev) for _ in range(2)]
    bufs[0][:b.src_rows].copy_(t0_slab)
    variants, res = O.build_all_levels(local, kernel, mode=O.REALISE_MIN_CARVEOUT if args.realise == "min"
                                       else O.REALISE_MAX_SMEM)
    nlev = len(variants)
    up, down = shard.halo_neighbours(rank, world, bands)

    def launch_args(n):
        cur, nxt = n % 2, (n + 1) % 2
        a = O.hotspot_args(bufs[cur].data_ptr(), bufs[nxt].data_ptr(), pw.data_ptr(), W, H, b.row_begin, b.row_end,
                           src_row_begin=b.src_begin, src_row_end=b.src_end, dst_row_begin=b.src_begin)
        if mode == "fanout":
            a = O.with_fanout(a, [shard.global_row_ptr(slabs.ptrs[nxt][up], bands[up], W) if up is not None else None,
                                  shard.global_row_ptr(slabs.ptrs[nxt][down], bands[down], W)
                                  if down is not None else None])
        return a

    ms = variants.sweep(launch_args(0), sp, rounds=max(3, args.rounds // 3))
    # the sweep wrote slab 1 from slab 0 (and, in fan-out mode, halo rows of the neighbours' slab 1):
    # restart from the initial grid
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier(group=group)
    bufs[0][:b.src_rows].copy_(t0_slab)
    tuner = O.Tuner(variants, O.default_cfg(samples_per_level=args.samples))
    n = 0

    def one_step(ev=None):
        nonlocal n
        tuner.step(launch_args(n), sp)
        if ev is not None:
            ev[1].record(stream)
        if mode == "fanout":
            slabs.barrier()                  # every rank's halo stores have landed
        elif mode == "gather":
            shard.exchange_halos_gather(bufs[(n + 1) % 2][:b.src_rows], b, bands, S, group)
        n += 1

    def all_settled():
        ok = torch.tensor([1 if tuner.final()[0] >= 0 else 0], device=dev)
        if world > 1:
            dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
        return bool(ok.item())

    done = 0
    while done < warmup or (done < warmup + 500 and not all_settled()):
        one_step()
        done += 1
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier(group=group)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
           torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    n0 = O.launch_count()
    with ClockSampler(local) as clk:
        for e in ev:
            e[0].record(stream)
            one_step(e)
            e[2].record(stream)
        torch.cuda.synchronize()
        clk.mark_end()
    launches = O.launch_count() - n0
    tot = ev[0][0].elapsed_time(ev[-1][2])
    comp = sum(e0.elapsed_time(e1) for e0, e1, _ in ev)
    exch = sum(e1.elapsed_time(e2) for _, e1, e2 in ev)
    # ---- end to end: pinned host slabs (T0 + P) -> device, 25 launches = 100 steps, band -> host ----
    e2e_dt = 0.0
    h2d = d2h = 0
    n_e2e = 100 // S
    if e2e:
        h_t = t0_slab.cpu().pin_memory()
        h_p = pw.cpu().pin_memory()
        h_o = torch.empty((b.rows, W), pin_memory=True)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier(group=group)
        t0 = time.perf_counter()
        n = 0
        bufs[0][:b.src_rows].copy_(h_t, non_blocking=True)
        pw.copy_(h_p, non_blocking=True)
        for _ in range(n_e2e):
            one_step()
        h_o.copy_(bufs[n % 2][b.row_begin - b.src_begin:b.row_end - b.src_begin], non_blocking=True)
        torch.cuda.synchronize()
        e2e_dt = time.perf_counter() - t0
        h2d, d2h = 2 * b.src_rows * W * 4, b.rows * W * 4
    t = torch.tensor([tot, comp, exch, e2e_dt], device=dev)
    byts = torch.tensor([float(h2d), float(d2h)], device=dev, dtype=torch.float64)
    final, it = tuner.final()
    chosen = [variants.level(final).ctas_per_sm if final >= 0 else -1, it,
              variants.level(min(range(nlev), key=lambda k: ms[k])).ctas_per_sm, b.row_begin, b.row_end]
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        dist.all_reduce(byts, op=dist.ReduceOp.SUM, group=group)
        allc = [None] * world
        dist.all_gather_object(allc, chosen, group=group)
    else:
        allc = [chosen]
    tot, comp, exch, e2e_dt = (float(x) for x in t.tolist())
    rec = None
    if rank == 0:
        units = H * W * S
        rec = {
            "metric": METRIC, "value": units * steps / (tot * 1e-3) / 1e6, "unit": "Mcell-steps/s",
            "n_gpus": world, "steps": steps, "warmup": warmup, "ms_per_step": tot / steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "thermal stencil 8192x8192 fp32 row-sharded, halo exchange per 4-step launch",
                       "baseline_config_index": 2, "kernel": kernel, "width": W, "height": H,
                       "rows_per_rank": b.rows_per_rank, "halo_rows": S,
                       "exchange": ("kernel stores of the first / last 4 rows into the neighbours' symmetric-memory "
                                    "slabs over NVLink + device barrier" if mode == "fanout" else
                                    "all_gather of the boundary rows" if mode == "gather" else "none (P=1)"),
                       "exchange_note": note, "parallelism": f"row-sharded x{world}",
                       "backend": backend_name() if world > 1 else None, "l2": "grids (3 x 256 MiB / P) vs L2"},
            "compute_only": {"value": units * steps / (comp * 1e-3) / 1e6, "unit": "Mcell-steps/s",
                             "ms_per_step": comp / steps},
            "exchange_ms_per_step": exch / steps,
            "per_rank": [{"rank": r, "final_k": c[0], "iterations_to_final": c[1], "sweep_best_k": c[2],
                          "rows": [c[3], c[4]]} for r, c in enumerate(allc)],
            "sweep_rank0": [{"k": variants.level(i).ctas_per_sm, "ms": round(ms[i], 4)} for i in range(nlev)],
            "gpu_launches": launches, "clocks": clk.summary(), "energy": clk.energy(steps),
            "e2e": ({"value": units * n_e2e / e2e_dt / 1e6, "unit": "Mcell-steps/s",
                     "h2d_bytes_per_step": float(byts[0]) / n_e2e, "d2h_bytes_per_step": float(byts[1]) / n_e2e,
                     "steps": n_e2e, "api": "per rank: pinned host T0 + P slabs -> device, 25 tuned launches "
                                            "(100 steps) with the halo exchange, own band -> pinned host"}
                    if e2e else None),
            "cpu_baseline": None,
        }
    tuner.close()
    variants.close()
    del bufs, slabs
    torch.cuda.empty_cache()
    return rec


# ---- drivers ------------------------------------------------------------------------------------
def run_single(args):
    """N = 1: the headline configuration and (unless --only) every other one as a sub-record."""
    import torch
    world, rank, local = dist_env()
    if not torch.cuda.is_available():
        raise SystemExit("bench.py: no CUDA device (the product has no CPU path)")
    local = init_dist(world, local)
    key = args.workload
    wl = WORKLOADS[key]
    steps = args.steps or wl["steps"]
    if key == "c5":
        if args.c5_mode in ("fanout", "gather") and not dist_initialized():
            # a one-rank NCCL group: the symmetric-memory fan-out path, or the chunked NCCL
            # all-gather overlapped with compute, exercised on one GPU
            import torch.distributed as dist
            dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{free_port()}", world_size=1, rank=0,
                                    device_id=torch.device("cuda", local))
        line = measure_c5(args, world=1, rank=0, local=local, steps=steps, warmup=args.warmup, size=args.size,
                          mode_req=args.c5_mode, chunks_req=args.c5_chunks)
        print(json.dumps(line), flush=True)
        return
    t0 = time.perf_counter()
    line = measure_single(key, args, steps=steps, warmup=args.warmup, rounds=args.rounds,
                          cpu_seconds=0 if args.no_cpu_baseline else args.cpu_seconds,
                          carveout_axis=not args.no_carveout_axis, kernel=args.kernel or None, select=args.select,
                          local=local)
    line["seconds"] = round(time.perf_counter() - t0, 1)
    if not args.only:
        subs = {}
        for sub in SUB_RECORDS:
            if sub == key:
                continue
            t1 = time.perf_counter()
            try:
                if sub == "c5":
                    r = measure_c5(args, world=1, rank=0, local=local, steps=WORKLOADS["c5"]["steps"], warmup=3)
                else:
                    r = measure_single(sub, args, steps=WORKLOADS[sub]["steps"], warmup=max(args.warmup, 12),
                                       rounds=5 if sub == "c4" else args.rounds,
                                       cpu_seconds=0 if args.no_cpu_baseline else args.sub_cpu_seconds,
                                       carveout_axis=sub != "c4", select="fastest", local=local)
                r["seconds"] = round(time.perf_counter() - t1, 1)
            except Exception as ex:                           # reported, never silently dropped
                r = {"error": f"{type(ex).__name__}: {ex}"}
            subs[sub] = r
        line["configs"] = subs
        if not args.no_energy:
            nx = {}
            for sub, kern in (("c2", "nlm_f4_w"), ("srad", "srad_f32hs"), ("c3", "hotspot_f32"), ("c1", "knn_f4"),
                              ("c4", "nlm_f4_regheavy")):
                try:
                    nx[f"{sub}:{kern}"] = measure_energy(sub, args, kern, local=local)
                except Exception as ex:
                    nx[f"{sub}:{kern}"] = {"error": f"{type(ex).__name__}: {ex}"}
            line["next3_energy"] = nx
            # the headline's own timed region is shorter than NVML's energy window: its energy is the
            # tuned (FASTEST) level replayed over a >= 1.2 s window of the same workload
            fa = nx.get(f"{args.workload}:{WORKLOADS[args.workload]['kernel']}", {}).get("levels", {}).get("fastest")
            if fa and (line.get("energy") or {}).get("joules_per_step") is None:
                line["energy"] = {"joules_per_step": fa["joules_per_iteration"], "mean_watts": fa["mean_watts"],
                                  "source": "nvml total energy",
                                  "note": f"the tuned level (k = {fa['k']}) replayed as a CUDA graph over "
                                          f"{fa['window_s']:.2f} s (next3_energy); the timed region itself is "
                                          f"shorter than the counter's window"}
    line["seconds_total"] = round(time.perf_counter() - t0, 1)
    print(json.dumps(line), flush=True)


def run_multi(args):
    """N > 1 (one process per GPU): C5 row-sharded over every rank, with C5 at P = 1 (rank 0
    alone, the curve's anchor) in the same line."""
    import torch
    import torch.distributed as dist
    world, rank, local = dist_env()
    if args.gpus and args.gpus != world:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    local = init_dist(world, local)
    if args.workload == "c3":      # the stencil row-sharded with a halo exchange per launch
        measure, key, extra = measure_c3_sharded, "c3", {}
    else:                          # C5: the NLM frame row-sharded + the output exchange
        measure, key, extra = measure_c5, "c5", {"mode_req": args.c5_mode, "chunks_req": args.c5_chunks}
    steps = args.steps or WORKLOADS[key]["steps"]
    anchor = None
    if not args.no_anchor:
        if rank == 0:
            anchor = measure(args, world=1, rank=0, local=local, steps=steps, warmup=3, size=args.size, e2e=False)
        dist.barrier()
    line = measure(args, world=world, rank=rank, local=local, steps=steps, warmup=args.warmup, size=args.size,
                   **extra)
    if rank == 0:
        if anchor is not None:
            line[f"{key}_p1_anchor"] = {k: anchor[k] for k in ("value", "ms_per_step", "compute_only", "per_rank",
                                                                "clocks")}
            line["speedup_vs_p1"] = line["value"] / anchor["value"]
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def run_plumbing_check(args):
    """CPU-only check of the multi-rank plumbing (tests/test_bench_host.py, gloo): the spawn, the
    row bands + halos, the gather and the max-over-ranks reduction, with the per-band compute
    replaced by a COPY of the band's own input rows (a stand-in, not the method: no kernel runs,
    nothing is measured).  Rank 0 prints one JSON line saying whether the gathered image equals
    the generated one."""
    import numpy as np
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_middleware_hayeslcsz16_b200 import shard
    world, rank, _ = dist_env()
    if world > 1:
        dist.init_process_group("gloo")
    W, H = 23, args.size or 37
    b = shard.band(rank, world, H, 6)
    slab = torch.from_numpy(synth.noisy_rgba(W, H, seed=5, row_begin=b.src_begin, row_end=b.src_end))
    out = torch.zeros((b.rows_per_rank, W, 4))
    out[:b.rows] = slab[b.row_begin - b.src_begin:b.row_end - b.src_begin]     # stand-in for the kernel
    full = torch.empty((world * b.rows_per_rank, W, 4))
    t0 = time.perf_counter()
    if world > 1:
        if args.c5_chunks > 1:   # the chunked gather of the C5 measurement (uneven last band included)
            for r0, r1, _, _ in shard.chunk_plan(b, args.c5_chunks):
                shard.gather_rows(out, full, b.rows_per_rank, r0, r1)
        else:
            shard.gather_bands(out, full)
    else:
        full = out
    dt = torch.tensor([time.perf_counter() - t0 + rank * 1e-3])
    if world > 1:
        dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        allb = [None] * world
        dist.all_gather_object(allb, [b.row_begin, b.row_end, b.src_begin, b.src_end])
    else:
        allb = [[b.row_begin, b.row_end, b.src_begin, b.src_end]]
    if rank == 0:
        ok = bool(np.array_equal(full[:H].numpy(), synth.noisy_rgba(W, H, seed=5)))
        print(json.dumps({"plumbing_check": True, "n_gpus": world, "ok": ok, "bands": allb,
                          "max_over_ranks_s": float(dt.item()), "spawned": os.environ.get("ORION_BENCH_SPAWNED")}),
              flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=0, help="timed steps (0: the workload's default)")
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=sorted(WORKLOADS), default="c2")
    ap.add_argument("--only", action="store_true", help="the headline workload alone (no sub-records)")
    ap.add_argument("--rounds", type=int, default=11, help="interleaved rounds of the exhaustive sweep")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--sub-cpu-seconds", type=float, default=3.0)
    ap.add_argument("--no-energy", action="store_true", help="skip the NEXT-3 energy record")
    ap.add_argument("--no-chain", action="store_true",
                    help="stencils: launch every iteration grid-wide ordered (no orion_chain)")
    ap.add_argument("--no-anchor", action="store_true", help="N > 1: skip C5 at P = 1 on rank 0")
    ap.add_argument("--size", type=int, default=0, help="override the C5 image side (tests)")
    ap.add_argument("--kernel", default="", help="override the headline workload's kernel id (same family)")
    ap.add_argument("--batch", type=int, default=0,
                    help="denoisers: frames per launch / step of the headline workload (0: the workload's default "
                         "-- C1 256, the others 1)")
    ap.add_argument("--c5-chunks", type=int, default=4, help="C5: row chunks per band whose all-gathers overlap compute")
    ap.add_argument("--c5-mode", default="auto", choices=("auto", "fanout", "gather"),
                    help="C5 exchange: kernel fan-out into symmetric memory (auto: when available) or all-gather")
    ap.add_argument("--graph", default="auto", choices=("auto", "on", "native", "off"),
                    help="on: replay the K timed iterations as one CUDA graph (orion_tuner_capture); native: "
                         "issue them in one library call (orion_tune_steps); off: one Python call per "
                         "iteration; auto = on for the launch-bound C1 frames, off otherwise")
    ap.add_argument("--async-timing", type=int, default=0, choices=(0, 1),
                    help="1: the tuner reads its event pairs without host synchronisation")
    ap.add_argument("--samples", type=int, default=2,
                    help="timed launches per explored level, the fastest kept (paper: 1; reading R-A11)")
    ap.add_argument("--select", choices=["fastest", "lowest"], default="fastest",
                    help="final-kernel rule: fastest measured, or lowest occupancy within 2%% (resource saving)")
    ap.add_argument("--realise", choices=["max", "min"], default="min",
                    help="level realisation: max = pad against 228 KB smem; min = smallest carveout (more L1)")
    ap.add_argument("--no-carveout-axis", action="store_true", help="skip the sweep of the other realisation")
    ap.add_argument("--plumbing-check", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args(argv)
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        if not args.plumbing_check and backend_name() == "nccl":
            import torch
            if torch.cuda.device_count() < args.gpus:
                raise SystemExit(f"bench.py: --gpus {args.gpus} but {torch.cuda.device_count()} CUDA device(s)")
        sys.exit(spawn(args.gpus, argv))
    if args.plumbing_check:
        run_plumbing_check(args)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.impl == "reference":
        run_reference(args)
    elif world > 1:
        run_multi(args)
    else:
        run_single(args)


if __name__ == "__main__":
    main()
