"""The CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously correct implementations of what the Orion hot path
computes, written from PAPER.md (and, where the paper is silent, from the
readings listed in DESIGN.md).  Nothing here is used by the product:

* only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
  ``cpu_baseline`` / ``--impl reference`` leg may import, call, link or
  execute anything under ``oracle/``;
* the product library (``paper_conf_middleware_hayeslcsz16_b200``) never
  imports this package, and this package never imports the product.  The two
  share no code; only ``synth`` (seeded input generator, no method arithmetic)
  serves both.

Parts:
  O1 ``oracle.occupancy``  occupancy calculator + feasible levels   (Eq. 1)
  O2 ``oracle/denoise.c``  KNN / NLM filters in double               (reading R-O2)
  O3 ``oracle/stencil.c``  thermal stencil in double + fp32 form    (reading R-O3)
  O4 ``oracle.tuner``      Fig. 8 prune + Fig. 9 selection + brute force
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SOURCES = [os.path.join(_HERE, "denoise.c"), os.path.join(_HERE, "stencil.c"), os.path.join(_HERE, "srad.c")]
_lock = threading.Lock()
_lib = None

# SDK imageDenoising constants (reading R-O2).
KNN = dict(noise=1.0 / (0.32 * 0.32), lerpc=0.2, wthr=0.02, lthr=0.79, R=3, B=0)
NLM = dict(noise=1.0 / (1.45 * 1.45), lerpc=0.2, wthr=0.10, lthr=0.10, R=3, B=3)
# Relative half-width of the "uncertain weight" band (reading R-AMB).
AMB_BAND = 1e-4


def build(force: bool = False) -> str:
    """Compile oracle/liboracle.so with gcc (-O2, no fast-math, no FP contraction)."""
    with _lock:
        newest = max(os.path.getmtime(s) for s in _SOURCES)
        if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < newest:
            tmp = _LIB_PATH + f".tmp{os.getpid()}"
            subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fPIC",
                                   "-shared", "-o", tmp, *_SOURCES, "-lm"])
            os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class _DnParams(ctypes.Structure):
    _fields_ = [("noise", ctypes.c_double), ("lerpc", ctypes.c_double), ("wthr", ctypes.c_double),
                ("lthr", ctypes.c_double), ("band", ctypes.c_double), ("R", ctypes.c_int),
                ("B", ctypes.c_int)]


class _HsParams(ctypes.Structure):
    _fields_ = [("sdc", ctypes.c_double), ("rx", ctypes.c_double), ("ry", ctypes.c_double),
                ("rz", ctypes.c_double), ("amb", ctypes.c_double)]


def _load():
    global _lib
    if _lib is None:
        # ORACLE_LIB_OVERRIDE: a deliberately mutated build, used only by
        # tests/test_oracle_mutations.py to show that the pins catch plausible mistakes
        override = os.environ.get("ORACLE_LIB_OVERRIDE")
        if not override:
            build()
        lib = ctypes.CDLL(override or _LIB_PATH)
        P = ctypes.c_void_p
        lib.oracle_denoise_rows.restype = ctypes.c_long
        lib.oracle_denoise_rows.argtypes = [P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                            ctypes.c_int, ctypes.c_int, ctypes.POINTER(_DnParams),
                                            ctypes.c_int, P, P, P]
        lib.oracle_denoise_points.restype = ctypes.c_long
        lib.oracle_denoise_points.argtypes = [P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                              P, P, ctypes.c_int, ctypes.POINTER(_DnParams),
                                              ctypes.c_int, P, P, P]
        lib.oracle_srad_f64.restype = ctypes.c_int
        lib.oracle_srad_f64.argtypes = [P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_double, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P]
        for name in ("oracle_hotspot_f64", "oracle_hotspot_f32"):
            f = getattr(lib, name)
            f.restype = ctypes.c_int
            f.argtypes = [P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(_HsParams), P]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _params(kind: str, overrides: dict | None) -> tuple[_DnParams, int]:
    base = dict(KNN if kind == "knn" else NLM)
    if overrides:
        base.update(overrides)
    band = base.pop("band", AMB_BAND)
    return _DnParams(base["noise"], base["lerpc"], base["wthr"], base["lthr"], band,
                     base["R"], base["B"]), (0 if kind == "knn" else 1)


def denoise(kind: str, img: np.ndarray, height: int | None = None, row0: int = 0,
            y_begin: int | None = None, y_end: int | None = None, params: dict | None = None):
    """Filter rows [y_begin, y_end) of an image (KNN or NLM, double precision).

    img: float32 (rows, W, 4) slab of global rows [row0, row0+rows) of a W x height image.
    Returns (out, alt, amb): out/alt float64 (n, W, 3), amb bool (n, W).
    """
    img = np.ascontiguousarray(img, dtype=np.float32)
    rows, W = img.shape[0], img.shape[1]
    H = rows if height is None else height
    yb = row0 if y_begin is None else y_begin
    ye = row0 + rows if y_end is None else y_end
    n = ye - yb
    p, nlm = _params(kind, params)
    out = np.zeros((n, W, 3), np.float64)
    alt = np.zeros((n, W, 3), np.float64)
    amb = np.zeros((n, W), np.int32)
    _load().oracle_denoise_rows(_ptr(img), W, H, row0, rows, yb, ye, ctypes.byref(p), nlm,
                                _ptr(out), _ptr(alt), _ptr(amb))
    return out, alt, amb.astype(bool)


def denoise_points(kind: str, img: np.ndarray, xs, ys, height: int | None = None, row0: int = 0,
                   params: dict | None = None):
    """Filter an explicit list of pixels; returns (out (n,3), alt (n,3), amb (n,))."""
    img = np.ascontiguousarray(img, dtype=np.float32)
    rows, W = img.shape[0], img.shape[1]
    H = rows if height is None else height
    xs = np.ascontiguousarray(xs, dtype=np.int32)
    ys = np.ascontiguousarray(ys, dtype=np.int32)
    n = xs.shape[0]
    p, nlm = _params(kind, params)
    out = np.zeros((n, 3), np.float64)
    alt = np.zeros((n, 3), np.float64)
    amb = np.zeros((n,), np.int32)
    _load().oracle_denoise_points(_ptr(img), W, H, row0, rows, _ptr(xs), _ptr(ys), n, ctypes.byref(p),
                                  nlm, _ptr(out), _ptr(alt), _ptr(amb))
    return out, alt, amb.astype(bool)


# Rodinia hotspot constants at a fixed cell size (reading R-A15): the 512x512 grid's
# 16 mm chip cell (31.25 um) is kept for every N, so the scheme stays stable.
def hotspot_constants(cell: float = 0.016 / 512) -> dict:
    t_chip, k_si, spec_heat_si, factor_chip, max_pd, precision = 0.0005, 100.0, 1.75e6, 0.5, 3.0e6, 0.001
    cap = factor_chip * spec_heat_si * t_chip * cell * cell
    rx = cell / (2.0 * k_si * t_chip * cell)
    ry = cell / (2.0 * k_si * t_chip * cell)
    rz = t_chip / (k_si * cell * cell)
    max_slope = max_pd / (factor_chip * t_chip * spec_heat_si)
    step = precision / max_slope
    return dict(sdc=step / cap, rx=1.0 / rx, ry=1.0 / ry, rz=1.0 / rz, amb=80.0)


def hotspot(t0: np.ndarray, power: np.ndarray, steps: int, consts: dict | None = None,
            precision: str = "f64") -> np.ndarray:
    """`steps` explicit thermal steps.  f64: inputs taken as float64, returns float64;
    f32: inputs rounded to float32, returns float32 (H, W)."""
    c = consts or hotspot_constants()
    p = _HsParams(c["sdc"], c["rx"], c["ry"], c["rz"], c["amb"])
    H, W = t0.shape
    if precision == "f64":
        t0 = np.ascontiguousarray(t0, dtype=np.float64)
        power = np.ascontiguousarray(power, dtype=np.float64)
        out = np.zeros((H, W), np.float64)
        rc = _load().oracle_hotspot_f64(_ptr(t0), _ptr(power), W, H, steps, ctypes.byref(p), _ptr(out))
    else:
        t0 = np.ascontiguousarray(t0, dtype=np.float32)
        power = np.ascontiguousarray(power, dtype=np.float32)
        out = np.zeros((H, W), np.float32)
        rc = _load().oracle_hotspot_f32(_ptr(t0), _ptr(power), W, H, steps, ctypes.byref(p), _ptr(out))
    if rc != 0:
        raise MemoryError("oracle hotspot allocation failed")
    return out


def srad(j0: np.ndarray, iters: int, lam: float = 0.5, roi=(0, 127, 0, 127)):
    """`iters` SRAD iterations (O5, reading R-SRAD) in double.  roi = (r1, r2, c1, c2)
    inclusive.  Returns (J float64 (H, W), q0sqr per iteration)."""
    j0 = np.ascontiguousarray(j0, dtype=np.float64)
    H, W = j0.shape
    r1, r2, c1, c2 = roi
    out = np.zeros((H, W), np.float64)
    q0 = np.zeros(max(1, iters), np.float64)
    if _load().oracle_srad_f64(_ptr(j0), W, H, iters, lam, r1, r2, c1, c2, _ptr(out), _ptr(q0)) != 0:
        raise MemoryError("oracle srad allocation failed")
    return out, q0[:iters]
