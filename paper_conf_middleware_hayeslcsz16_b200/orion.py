"""Thin ctypes binding of liborion (include/orion.h) -- argument marshalling only.

Every step of the hot path runs inside liborion.so and its sm_100a kernels; this
module only converts Python values to the C structs and raises ``OrionError`` on a
negative status.  There is no fallback: if liborion.so is missing the import of
``lib()`` raises, and on a machine without a GPU the device entry points return
ORION_E_CUDA (host-only entry points -- levels, probe, replay -- still work).

Device buffers are passed as integer device pointers (e.g. ``tensor.data_ptr()``) and
streams as integer CUstream handles (``torch.cuda.current_stream().cuda_stream``).
"""
from __future__ import annotations

import ctypes
import math
import os
import threading
from dataclasses import dataclass

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ORION_LIB") or os.path.join(_HERE, "liborion.so")  # ORION_LIB: A/B experiments

ORION_OK = 0
STATUS = {0: "ORION_OK", -1: "ORION_E_INVALID", -2: "ORION_E_CAPACITY", -3: "ORION_E_INFEASIBLE",
          -4: "ORION_E_COMPILE", -5: "ORION_E_CUDA", -6: "ORION_E_OCCUPANCY_MISMATCH", -7: "ORION_E_STATE"}
LIM_REGS, LIM_SMEM, LIM_WARPS, LIM_BLOCKS = 1, 2, 4, 8
DIR_DECREASING, DIR_INCREASING = -1, 1
SELECT_FASTEST, SELECT_LOWEST_WITHIN_TOL = 0, 1

HALO = {"knn_f4": 3, "knn_f4_p1": 3, "knn_f4_t16": 3, "nlm_f4": 6, "nlm_f4_w": 6, "nlm_f4_direct": 6,
        "nlm_f4_regheavy": 6, "hotspot_f32": 1, "hotspot2h_f32": 2, "hotspot4h_f32": 4, "srad_f32": 2,
        "srad_f32h": 2, "srad_f32hs": 2, "srad_f32_tile": 2}
# stencil steps one launch advances (temporal blocking); every other kernel: 1
STEPS_PER_LAUNCH = {"hotspot2h_f32": 2, "hotspot4h_f32": 4}
KERNELS = tuple(HALO)
# families whose launches take an orion_chain (tile-level waits between iterations)
CHAINABLE = ("hotspot4h_f32", "srad_f32hs")


class OrionError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        super().__init__(f"{where}: {STATUS.get(status, status)}: {msg}")
        self.status = status


class DeviceLimits(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in (
        "cc_major", "cc_minor", "sm_count", "warp_size", "regs_per_sm", "regs_per_block",
        "max_regs_per_thread", "reg_alloc_unit", "num_subpartitions", "max_threads_per_sm",
        "max_threads_per_block", "max_blocks_per_sm", "smem_per_sm", "smem_per_block_optin",
        "smem_reserved_per_block", "smem_alloc_unit")]


class KernelResources(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in (
        "block_threads", "regs_per_thread", "static_smem_bytes", "dyn_smem_bytes", "min_reg_cap")]


class Level(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in (
        "ctas_per_sm", "warps_per_sm", "occupancy_permille", "reg_cap", "smem_pad_bytes", "limiter",
        "carveout_kb")]

    def as_tuple(self):
        return tuple(getattr(self, n) for n, _ in self._fields_)

    def __repr__(self):
        return ("Level(k=%d, warps=%d, occ=%.3f, cap=%d, pad=%d, lim=%d, carveout=%dKB)"
                % (self.ctas_per_sm, self.warps_per_sm, self.occupancy_permille / 1000.0,
                   self.reg_cap, self.smem_pad_bytes, self.limiter, self.carveout_kb))


REALISE_MAX_SMEM, REALISE_MIN_CARVEOUT = 0, 1


class Args(ctypes.Structure):
    _fields_ = [("src", ctypes.c_void_p), ("dst", ctypes.c_void_p), ("aux", ctypes.c_void_p),
                ("width", ctypes.c_int), ("height", ctypes.c_int),
                ("row_begin", ctypes.c_int), ("row_end", ctypes.c_int),
                ("src_row_begin", ctypes.c_int), ("src_row_end", ctypes.c_int),
                ("dst_row_begin", ctypes.c_int), ("fparam", ctypes.c_float * 8),
                ("fanout", ctypes.c_void_p * 8), ("n_fanout", ctypes.c_int), ("flags", ctypes.c_int),
                ("chain", ctypes.c_void_p), ("batch", ctypes.c_int)]


ARGS_INDEPENDENT = 1       # orion.h ORION_ARGS_INDEPENDENT


def with_fanout(a: Args, ptrs) -> Args:
    """Add fan-out outputs (full-image device pointers, e.g. every rank's gather buffer) to a."""
    ptrs = list(ptrs)
    if len(ptrs) > 8:
        raise ValueError("at most 8 fan-out buffers")
    for i, p in enumerate(ptrs):
        a.fanout[i] = p
    a.n_fanout = len(ptrs)
    return a


class TunerCfg(ctypes.Structure):
    _fields_ = [("maxlive_threshold", ctypes.c_int), ("samples_per_level", ctypes.c_int),
                ("select_mode", ctypes.c_int), ("allow_direction_switch", ctypes.c_int),
                ("slowdown_tol", ctypes.c_float), ("worse_eps", ctypes.c_float),
                ("expected_iterations", ctypes.c_int), ("async_timing", ctypes.c_int)]


class StepReport(ctypes.Structure):
    _fields_ = [("iteration", ctypes.c_int), ("level_idx", ctypes.c_int), ("phase", ctypes.c_int),
                ("final_level_idx", ctypes.c_int), ("ms", ctypes.c_float)]


_lock = threading.Lock()
_lib = None


def lib() -> ctypes.CDLL:
    """Load liborion.so (building it first if it is missing and nvcc is available)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                from . import build as _build
                _build.build()
            L = ctypes.CDLL(LIB_PATH)
            P, I, V = ctypes.POINTER, ctypes.c_int, ctypes.c_void_p
            sig = {
                "orion_b200_limits": [P(DeviceLimits)],
                "orion_query_limits": [I, P(DeviceLimits)],
                "orion_ctas_per_sm": [P(DeviceLimits), I, I, I, I, P(I), P(I)],
                "orion_levels": [P(DeviceLimits), P(KernelResources), P(Level), I, P(I)],
                "orion_levels_ex": [P(DeviceLimits), P(KernelResources), I, P(Level), I, P(I)],
                "orion_ctas_per_sm_carveout": [P(DeviceLimits), I, I, I, I, I, P(I), P(I)],
                "orion_kernel_probe": [ctypes.c_char_p, I, P(KernelResources)],
                "orion_compile_info": [ctypes.c_char_p, I, I, P(I), P(I), P(I), P(I)],
                "orion_build_variants": [I, ctypes.c_char_p, I, P(Level), I, P(V)],
                "orion_variants_count": [V, P(I)],
                "orion_variant_level": [V, I, P(Level)],
                "orion_variant_info": [V, I, P(I), P(I), P(I), P(I), P(I)],
                "orion_variants_resources": [V, P(KernelResources)],
                "orion_launch": [V, I, P(Args), V],
                "orion_sweep": [V, P(Args), V, I, P(ctypes.c_float)],
                "orion_tuner_default_cfg": [P(TunerCfg)],
                "orion_tuner_create": [V, P(TunerCfg), P(V)],
                "orion_tune_step": [V, P(Args), V, P(StepReport)],
                "orion_tune_steps": [V, P(Args), I, V, P(StepReport)],
                "orion_tune_step_host": [V, P(Args), V, V, V, V, P(StepReport), P(ctypes.c_longlong),
                                         P(ctypes.c_longlong)],
                "orion_tune_split": [V, P(Args), I, V, P(StepReport)],
                "orion_tuner_capture": [V, P(Args), I, P(V)],
                "orion_tuner_resume": [V, I],
                "orion_graph_launch": [V, V],
                "orion_tune_run_host": [V, P(Args), I, V, V, V, P(I), V, P(ctypes.c_longlong),
                                        P(ctypes.c_longlong)],
                "orion_host_pipe_create": [V, I, I, I, P(V)],
                "orion_host_pipe_submit": [V, P(Args), P(StepReport), P(ctypes.c_longlong), P(ctypes.c_longlong)],
                "orion_host_pipe_drain": [V],
                "orion_tuner_ladder": [V, P(I), P(I), I, P(I)],
                "orion_tuner_final": [V, P(I), P(I)],
                "orion_tuner_tried": [V, P(ctypes.c_float), I],
                "orion_set_pdl": [I, P(I)],
                "orion_default_params": [ctypes.c_char_p, P(ctypes.c_float), I],
                "orion_tuner_replay": [P(TunerCfg), P(Level), I, I, P(ctypes.c_float), I, P(I), P(I), P(I)],
                "orion_generate_rgba": [I, V, I, I, I, I, ctypes.c_uint, ctypes.c_float, V],
                "orion_generate_thermal": [I, V, V, I, I, ctypes.c_uint, V],
                "orion_flush_l2": [I, V, ctypes.c_longlong, V],
                "orion_srad_roi_stats": [I, V, I, I, I, I, I, I, V, V],
                "orion_srad_stats_init": [I, V, I, I, I, I, I, I, V],
                "orion_chain_create": [V, I, I, P(V)],
                "orion_chain_info": [V, P(ctypes.c_uint), P(I), P(I)],
            }
            for name, args in sig.items():
                f = getattr(L, name)
                f.argtypes = args
                f.restype = ctypes.c_int
            for name in ("orion_variants_destroy", "orion_tuner_destroy", "orion_host_pipe_destroy",
                         "orion_graph_destroy", "orion_chain_destroy"):
                getattr(L, name).argtypes = [V]
                getattr(L, name).restype = None
            L.orion_status_str.restype = ctypes.c_char_p
            L.orion_status_str.argtypes = [I]
            L.orion_last_error.restype = ctypes.c_char_p
            L.orion_last_error.argtypes = []
            L.orion_launch_count.restype = ctypes.c_longlong
            L.orion_version.restype = ctypes.c_char_p
            _lib = L
    return _lib


def _check(status: int, where: str):
    if status != ORION_OK:
        raise OrionError(status, where, lib().orion_last_error().decode(errors="replace"))


def _s(stream) -> ctypes.c_void_p:
    return ctypes.c_void_p(int(stream) if stream else 0)


# ---- levels (host-only) -------------------------------------------------------------------
def b200_limits() -> DeviceLimits:
    d = DeviceLimits()
    _check(lib().orion_b200_limits(ctypes.byref(d)), "orion_b200_limits")
    return d


def query_limits(device: int = 0) -> DeviceLimits:
    d = DeviceLimits()
    _check(lib().orion_query_limits(device, ctypes.byref(d)), "orion_query_limits")
    return d


def ctas_per_sm(dev: DeviceLimits, T: int, regs: int, smem_static: int = 0, smem_dyn: int = 0,
                carveout_pct: int = -1):
    c, lim = ctypes.c_int(), ctypes.c_int()
    _check(lib().orion_ctas_per_sm_carveout(ctypes.byref(dev), T, regs, smem_static, smem_dyn, carveout_pct,
                                            ctypes.byref(c), ctypes.byref(lim)), "orion_ctas_per_sm_carveout")
    return c.value, lim.value


def resources(block_threads: int, regs: int, static_smem: int = 0, dyn_smem: int = 0,
              min_reg_cap: int = 16) -> KernelResources:
    return KernelResources(block_threads, regs, static_smem, dyn_smem, min_reg_cap)


def levels(dev: DeviceLimits, res: KernelResources, mode: int = REALISE_MAX_SMEM) -> list[Level]:
    n = ctypes.c_int()
    st = lib().orion_levels_ex(ctypes.byref(dev), ctypes.byref(res), mode, None, 0, ctypes.byref(n))
    if st not in (ORION_OK, -2):
        _check(st, "orion_levels_ex")
    arr = (Level * max(1, n.value))()
    _check(lib().orion_levels_ex(ctypes.byref(dev), ctypes.byref(res), mode, arr, n.value, ctypes.byref(n)),
           "orion_levels_ex")
    return [arr[i] for i in range(n.value)]


def kernel_probe(kernel_id: str, block_threads: int = 0) -> KernelResources:
    r = KernelResources()
    _check(lib().orion_kernel_probe(kernel_id.encode(), block_threads, ctypes.byref(r)), "orion_kernel_probe")
    return r


def compile_info(kernel_id: str, block_threads: int, reg_cap: int) -> dict:
    v = [ctypes.c_int() for _ in range(4)]
    _check(lib().orion_compile_info(kernel_id.encode(), block_threads, reg_cap, *[ctypes.byref(x) for x in v]),
           "orion_compile_info")
    return dict(regs=v[0].value, spill_store=v[1].value, spill_load=v[2].value, local_bytes=v[3].value)


# ---- launch arguments ----------------------------------------------------------------------
def denoise_args(kernel_id: str, src: int, dst: int, width: int, height: int, row_begin: int = 0,
                 row_end: int | None = None, src_row_begin: int = 0, src_row_end: int | None = None,
                 dst_row_begin: int | None = None, params=None, independent: bool = False, batch: int = 1) -> Args:
    """Arguments of one denoiser launch.  independent: ORION_ARGS_INDEPENDENT -- the caller asserts
    the launch touches nothing the stream's previous kernel writes (e.g. the next frame, in its own
    buffers), so with PDL it need not wait for that kernel.  batch: B > 1 whole frames stacked in
    src / dst (frame f at f * width * height pixels), one launch."""
    row_end = height if row_end is None else row_end
    src_row_end = height if src_row_end is None else src_row_end
    dst_row_begin = row_begin if dst_row_begin is None else dst_row_begin
    p = params or default_params(kernel_id)[:4]
    a = Args(src, dst, None, width, height, row_begin, row_end, src_row_begin, src_row_end, dst_row_begin)
    for i, x in enumerate(p):
        a.fparam[i] = x
    a.flags = ARGS_INDEPENDENT if independent else 0
    a.batch = batch
    return a


def default_params(kernel_id: str) -> tuple:
    """orion_default_params: the kernel family's method parameters (fparam[0..8)) as liborion
    defines them -- SDK imageDenoising (Noise, lerpC, wthr, lthr), Rodinia hotspot (sdc, rx, ry,
    rz, amb) or SRAD (lambda)."""
    buf = (ctypes.c_float * 8)()
    _check(lib().orion_default_params(kernel_id.encode(), buf, 8), "orion_default_params")
    return tuple(buf)


def hotspot_args(t_in: int, t_out: int, power: int, width: int, height: int, row_begin: int = 0,
                 row_end: int | None = None, consts=None, src_row_begin: int = 0, src_row_end: int | None = None,
                 dst_row_begin: int = 0, chain: "Chain | None" = None) -> Args:
    """Arguments of one thermal-stencil launch.  Whole grid by default; a row band of a sharded
    grid: t_in / power hold global rows [src_row_begin, src_row_end), t_out from dst_row_begin.
    chain: the orion_chain this whole-grid launch continues (tile-level waits, orion.h)."""
    row_end = height if row_end is None else row_end
    src_row_end = height if src_row_end is None else src_row_end
    a = Args(t_in, t_out, power, width, height, row_begin, row_end, src_row_begin, src_row_end, dst_row_begin)
    for i, x in enumerate(consts or default_params("hotspot_f32")[:5]):
        a.fparam[i] = x
    a.chain = chain.h if chain is not None else None
    return a


# ---- the multi-version binary --------------------------------------------------------------
@dataclass
class VariantInfo:
    level: Level
    regs: int
    spill_store: int
    spill_load: int
    local_bytes: int
    verified_ctas: int


class Variants:
    """orion_build_variants handle: one sm_100a variant per occupancy level."""

    def __init__(self, device: int, kernel_id: str, lv: list[Level], block_threads: int = 0):
        self.kernel_id = kernel_id
        self.device = device
        arr = (Level * len(lv))(*lv)
        h = ctypes.c_void_p()
        _check(lib().orion_build_variants(device, kernel_id.encode(), block_threads, arr, len(lv), ctypes.byref(h)),
               "orion_build_variants")
        self.h = h
        self.planned = list(lv)

    def __len__(self):
        n = ctypes.c_int()
        _check(lib().orion_variants_count(self.h, ctypes.byref(n)), "orion_variants_count")
        return n.value

    def level(self, i: int) -> Level:
        L = Level()
        _check(lib().orion_variant_level(self.h, i, ctypes.byref(L)), "orion_variant_level")
        return L

    def info(self, i: int) -> VariantInfo:
        v = [ctypes.c_int() for _ in range(5)]
        _check(lib().orion_variant_info(self.h, i, *[ctypes.byref(x) for x in v]), "orion_variant_info")
        return VariantInfo(self.level(i), *[x.value for x in v])

    def resources(self) -> KernelResources:
        r = KernelResources()
        _check(lib().orion_variants_resources(self.h, ctypes.byref(r)), "orion_variants_resources")
        return r

    def launch(self, i: int, args: Args, stream=None):
        _check(lib().orion_launch(self.h, i, ctypes.byref(args), _s(stream)), "orion_launch")

    def sweep(self, args: Args, stream=None, rounds: int = 5) -> list[float]:
        ms = (ctypes.c_float * len(self))()
        _check(lib().orion_sweep(self.h, ctypes.byref(args), _s(stream), rounds, ms), "orion_sweep")
        return list(ms)

    def close(self):
        if getattr(self, "h", None):
            lib().orion_variants_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def build_all_levels(device: int, kernel_id: str, block_threads: int = 0, dev: DeviceLimits | None = None,
                     mode: int = REALISE_MAX_SMEM):
    """Convenience: probe -> orion_levels_ex -> orion_build_variants (every feasible level)."""
    res = kernel_probe(kernel_id, block_threads)
    dev = dev or query_limits(device)
    lv = levels(dev, res, mode)
    return Variants(device, kernel_id, lv, block_threads), res


def default_cfg(**kw) -> TunerCfg:
    c = TunerCfg()
    _check(lib().orion_tuner_default_cfg(ctypes.byref(c)), "orion_tuner_default_cfg")
    for k, v in kw.items():
        setattr(c, k, v)
    return c


class Tuner:
    """orion_tuner handle: Fig. 8 ladder + Fig. 9 walk across iterations."""

    def __init__(self, variants: Variants, cfg: TunerCfg | None = None, trace: str | None = None):
        """trace: optional JSONL path -- one record per orion_tune_step (iteration, level index,
        its CTAs/SM, phase, measured ms, final level): the tuner's per-iteration log."""
        self.variants = variants
        h = ctypes.c_void_p()
        _check(lib().orion_tuner_create(variants.h, ctypes.byref(cfg or default_cfg()), ctypes.byref(h)),
               "orion_tuner_create")
        self.h = h
        self._trace = open(trace, "a") if trace else None

    def step(self, args: Args, stream=None) -> StepReport:
        r = StepReport()
        _check(lib().orion_tune_step(self.h, ctypes.byref(args), _s(stream), ctypes.byref(r)), "orion_tune_step")
        if self._trace is not None:
            import json
            self._trace.write(json.dumps({"iteration": r.iteration, "level_idx": r.level_idx,
                                          "ctas_per_sm": self.variants.level(r.level_idx).ctas_per_sm,
                                          "phase": "explore" if r.phase == 0 else "final",
                                          "ms": r.ms if r.ms >= 0 else None,
                                          "final_level_idx": r.final_level_idx}) + "\n")
        return r

    def steps(self, args_list: list, stream=None) -> StepReport:
        """orion_tune_steps: len(args_list) iterations issued by the library in one call."""
        arr = (Args * len(args_list))(*args_list)
        r = StepReport()
        _check(lib().orion_tune_steps(self.h, arr, len(args_list), _s(stream), ctypes.byref(r)), "orion_tune_steps")
        return r

    def split(self, args: Args, bands: int, stream=None) -> list[StepReport]:
        reps = (StepReport * bands)()
        _check(lib().orion_tune_split(self.h, ctypes.byref(args), bands, _s(stream), reps), "orion_tune_split")
        return [reps[i] for i in range(bands)]

    def step_host(self, args: Args, dev_src: int, dev_dst: int, dev_aux: int | None = None, stream=None):
        r = StepReport()
        hi, ho = ctypes.c_longlong(), ctypes.c_longlong()
        _check(lib().orion_tune_step_host(self.h, ctypes.byref(args), ctypes.c_void_p(dev_src),
                                          ctypes.c_void_p(dev_dst), ctypes.c_void_p(dev_aux or 0), _s(stream),
                                          ctypes.byref(r), ctypes.byref(hi), ctypes.byref(ho)),
               "orion_tune_step_host")
        return r, hi.value, ho.value

    def run_host(self, args: Args, iterations: int, dev_a: int, dev_b: int, dev_aux: int, roi=None, stream=None):
        """orion_tune_run_host: a whole stencil run from host grids (copy in, iterate, copy out)."""
        hi, ho = ctypes.c_longlong(), ctypes.c_longlong()
        r = (ctypes.c_int * 4)(*roi) if roi is not None else None
        _check(lib().orion_tune_run_host(self.h, ctypes.byref(args), iterations, ctypes.c_void_p(dev_a),
                                         ctypes.c_void_p(dev_b), ctypes.c_void_p(dev_aux), r, _s(stream),
                                         ctypes.byref(hi), ctypes.byref(ho)), "orion_tune_run_host")
        return hi.value, ho.value

    def resume(self, final_level_idx: int):
        """orion_tuner_resume: adopt a final level recorded by an earlier run (skip exploration)."""
        _check(lib().orion_tuner_resume(self.h, final_level_idx), "orion_tuner_resume")

    def capture(self, args_list: list, stream=None) -> "Graph":
        """orion_tuner_capture: the settled kernel's launches for args_list[i] as one CUDA graph."""
        return Graph(self, args_list)

    def ladder(self):
        d, n = ctypes.c_int(), ctypes.c_int()
        buf = (ctypes.c_int * 64)()
        _check(lib().orion_tuner_ladder(self.h, ctypes.byref(d), buf, 64, ctypes.byref(n)), "orion_tuner_ladder")
        return d.value, [buf[i] for i in range(n.value)]

    def tried(self) -> list[float]:
        """orion_tuner_tried: the per-level table Fig. 9 observed (ns per output element; -1 = not run)."""
        n = len(self.variants)
        buf = (ctypes.c_float * n)()
        _check(lib().orion_tuner_tried(self.h, buf, n), "orion_tuner_tried")
        return [buf[i] for i in range(n)]

    def final(self):
        f, it = ctypes.c_int(), ctypes.c_int()
        _check(lib().orion_tuner_final(self.h, ctypes.byref(f), ctypes.byref(it)), "orion_tuner_final")
        return f.value, it.value

    def close(self):
        if getattr(self, "_trace", None) is not None:
            self._trace.close()
            self._trace = None
        if getattr(self, "h", None):
            lib().orion_tuner_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Graph:
    """orion_graph handle: replay n settled iterations with one host call."""

    def __init__(self, tuner: "Tuner", args_list: list):
        self.tuner = tuner
        arr = (Args * len(args_list))(*args_list)
        h = ctypes.c_void_p()
        _check(lib().orion_tuner_capture(tuner.h, arr, len(args_list), ctypes.byref(h)), "orion_tuner_capture")
        self.h, self.n = h, len(args_list)

    def launch(self, stream=None):
        _check(lib().orion_graph_launch(self.h, _s(stream)), "orion_graph_launch")

    def close(self):
        if getattr(self, "h", None):
            lib().orion_graph_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class HostPipe:
    """orion_host_pipe handle: pipelined iterations from pinned host buffers."""

    def __init__(self, tuner: Tuner, width: int, max_rows: int, depth: int = 2):
        self.tuner = tuner
        h = ctypes.c_void_p()
        _check(lib().orion_host_pipe_create(tuner.h, width, max_rows, depth, ctypes.byref(h)),
               "orion_host_pipe_create")
        self.h = h

    def submit(self, args: Args):
        r = StepReport()
        hi, ho = ctypes.c_longlong(), ctypes.c_longlong()
        _check(lib().orion_host_pipe_submit(self.h, ctypes.byref(args), ctypes.byref(r), ctypes.byref(hi),
                                            ctypes.byref(ho)), "orion_host_pipe_submit")
        return r, hi.value, ho.value

    def drain(self):
        _check(lib().orion_host_pipe_drain(self.h), "orion_host_pipe_drain")

    def close(self):
        if getattr(self, "h", None):
            lib().orion_host_pipe_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def tuner_replay(cfg: TunerCfg, lv: list[Level], natural_regs: int, ms_of_level, iterations: int):
    n = len(lv)
    arr = (Level * n)(*lv)
    ms = (ctypes.c_float * n)(*[float(x) for x in ms_of_level])
    ran = (ctypes.c_int * max(1, iterations))()
    f, fi = ctypes.c_int(), ctypes.c_int()
    _check(lib().orion_tuner_replay(ctypes.byref(cfg), arr, n, natural_regs, ms, iterations, ran, ctypes.byref(f),
                                    ctypes.byref(fi)), "orion_tuner_replay")
    return [ran[i] for i in range(iterations)], f.value, fi.value


# ---- synthetic inputs (device generator) ----------------------------------------------------
def generate_rgba(device: int, dst: int, width: int, height: int, row_begin: int = 0, row_end: int | None = None,
                  seed: int = 1, sigma: float = 0.13, stream=None):
    row_end = height if row_end is None else row_end
    _check(lib().orion_generate_rgba(device, ctypes.c_void_p(dst), width, height, row_begin, row_end, seed,
                                     sigma, _s(stream)), "orion_generate_rgba")


def generate_thermal(device: int, t0: int, power: int, width: int, height: int, seed: int = 1, stream=None):
    _check(lib().orion_generate_thermal(device, ctypes.c_void_p(t0), ctypes.c_void_p(power), width, height, seed,
                                        _s(stream)), "orion_generate_thermal")


# "srad_f32hs": floats of ROI statistics slots behind every grid it reads or writes (orion.h)
SRAD_STATS_FLOATS = 256


def srad_args(j_in: int, j_out: int, q0: int, width: int, height: int, lam: float | None = None,
              roi=None, chain: "Chain | None" = None) -> Args:
    """Arguments of one SRAD iteration.  "srad_f32" / "srad_f32h" / "srad_f32_tile": q0 = device
    address of the float q0sqr (orion_srad_roi_stats).  "srad_f32hs": q0 unused (0), roi =
    (r1, r2, c1, c2) -- the statistics travel in the slots behind the grids.  lam None =
    liborion's default (orion_default_params)."""
    a = Args(j_in, j_out, q0 or None, width, height, 0, height, 0, height, 0)
    a.fparam[0] = default_params("srad_f32h")[0] if lam is None else lam
    if roi is not None:
        for i, v in enumerate(roi):
            a.fparam[1 + i] = float(v)
    a.chain = chain.h if chain is not None else None
    return a


class Chain:
    """orion_chain: consecutive whole-grid launches of one stencil family on one stream, each
    waiting for the previous one tile by tile (orion.h).  Pass it to hotspot_args / srad_args."""

    def __init__(self, variants: "Variants", width: int, height: int):
        self.h = ctypes.c_void_p()
        _check(lib().orion_chain_create(variants.h, width, height, ctypes.byref(self.h)), "orion_chain_create")

    def info(self) -> tuple[int, int, int]:
        """(launches so far, tiles_x, tiles_y)."""
        e, x, y = ctypes.c_uint(), ctypes.c_int(), ctypes.c_int()
        _check(lib().orion_chain_info(self.h, ctypes.byref(e), ctypes.byref(x), ctypes.byref(y)), "orion_chain_info")
        return e.value, x.value, y.value

    def close(self):
        if self.h:
            lib().orion_chain_destroy(self.h)
            self.h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def srad_stats_init(device: int, j: int, width: int, height: int, roi, stream=None):
    """orion_srad_stats_init: the statistics slots of grid j (the first "srad_f32hs" input)."""
    r1, r2, c1, c2 = roi
    _check(lib().orion_srad_stats_init(device, ctypes.c_void_p(j), width, height, r1, r2, c1, c2, _s(stream)),
           "orion_srad_stats_init")


def srad_roi_stats(device: int, j: int, width: int, height: int, roi, q0: int, stream=None):
    r1, r2, c1, c2 = roi
    _check(lib().orion_srad_roi_stats(device, ctypes.c_void_p(j), width, height, r1, r2, c1, c2, ctypes.c_void_p(q0),
                                      _s(stream)), "orion_srad_roi_stats")


def flush_l2(device: int, buf: int, nbytes: int, stream=None):
    _check(lib().orion_flush_l2(device, ctypes.c_void_p(buf), nbytes, _s(stream)), "orion_flush_l2")


def set_pdl(on: bool) -> bool:
    """orion_set_pdl: programmatic dependent launch on / off for later launches; returns the
    previous setting."""
    prev = ctypes.c_int()
    _check(lib().orion_set_pdl(1 if on else 0, ctypes.byref(prev)), "orion_set_pdl")
    return bool(prev.value)


def launch_count() -> int:
    return lib().orion_launch_count()


def version() -> str:
    return lib().orion_version().decode()


def occupancy(level: Level) -> float:
    return level.occupancy_permille / 1000.0


__all__ = [n for n in dir() if not n.startswith("_") and n not in ("annotations", "ctypes", "math", "os",
                                                                      "threading", "dataclass")]
