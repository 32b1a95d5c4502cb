"""Seeded synthetic inputs shared by the tests, the oracle and bench.py.

This module holds NO arithmetic of the method (no denoising, no stencil, no
occupancy or tuner logic).  It only draws the synthetic workloads whose recipe
DESIGN.md §"Input recipe" states (SURVEY.md §8(d) "Generator"):

* a counter-based hash (splitmix64 of ``(seed, pixel, channel)``) so that any
  pixel of any image can be regenerated independently — which is what makes a
  row-sharded image (config C5) bit-identical to the full one;
* every floating-point step is either exact or ONE IEEE fp32 rounding in a
  fixed order, so the GPU twin of this generator
  (``paper_conf_middleware_hayeslcsz16_b200/csrc/kernels/gen.cu``, a separate
  implementation of the same counter-based generator) produces the same bits.

Noisy RGBA image (SDK imageDenoising stand-in; PAPER.md gives no inputs,
P:L85-91 only names the benchmark):

    clean(x, y) = background gradient overwritten by 12 random boxes
                  r = 0.25 + 0.5*((x & 1023)/1024), g = 0.25 + 0.5*((y & 1023)/1024), b = 0.5
                  box colour channel = ((h >> 16c) % 820 + 102) / 1024      (all exact in fp32)
    a = splitmix64(key(seed, y*W + x, c)) >> 41                           (23-bit integer)
    u = (a - 2**22) * 2**-22                   in [-1, 1), exact
    v = clamp(clean + u * s, 0, 1),  s = fp32(sqrt(3) * sigma)           (two roundings)
    alpha = 1

Thermal stencil inputs (Rodinia hotspot stand-in):

    T0 = 323.15f + (a * 2**-23) * 20f          (two roundings)
    P  = (a' * 2**-23) * 0.05f                 (one rounding)
"""
from __future__ import annotations

import math

import numpy as np

__all__ = [
    "splitmix64",
    "noise_scale",
    "noisy_rgba",
    "thermal_inputs",
    "NBOXES",
]

NBOXES = 12
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """splitmix64 finaliser of ``x + golden`` (wrapping uint64 arithmetic)."""
    with np.errstate(over="ignore"):
        z = np.asarray(x, dtype=np.uint64) + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _key(seed: int, idx, chan: int):
    return (np.uint64(seed) << np.uint64(40)) + np.asarray(idx, dtype=np.uint64) * np.uint64(4) + np.uint64(chan)


def _box_key(seed: int, b: int, k: int):
    return (np.uint64(seed) << np.uint64(40)) | (np.uint64(1) << np.uint64(39)) | np.uint64(b * 8 + k)


def boxes(seed: int, width: int, height: int):
    """The 12 axis-aligned boxes: list of (x0, y0, w, h, (r, g, b)) with exact fp32 colours."""
    out = []
    for b in range(NBOXES):
        h = [int(splitmix64(_box_key(seed, b, k))) for k in range(5)]
        x0 = h[0] % width
        y0 = h[1] % height
        bw = 1 + h[2] % max(1, width // 4)
        bh = 1 + h[3] % max(1, height // 4)
        col = tuple(np.float32(((h[4] >> (16 * c)) % 820 + 102) / 1024.0) for c in range(3))
        out.append((x0, y0, bw, bh, col))
    return out


def noise_scale(sigma: float) -> np.float32:
    """fp32 amplitude s of uniform noise u*s with std sigma (u uniform on [-1,1))."""
    return np.float32(math.sqrt(3.0) * sigma)


def noisy_rgba(width: int, height: int, seed: int = 1, sigma: float = 0.13,
               row_begin: int = 0, row_end: int | None = None) -> np.ndarray:
    """Rows [row_begin, row_end) of the W x H noisy RGBA image, float32 (rows, W, 4)."""
    if row_end is None:
        row_end = height
    row_begin = max(0, row_begin)
    row_end = min(height, row_end)
    ys = np.arange(row_begin, row_end, dtype=np.int64)[:, None]
    xs = np.arange(width, dtype=np.int64)[None, :]
    rows = row_end - row_begin
    clean = np.empty((rows, width, 3), dtype=np.float32)
    clean[..., 0] = np.float32(0.25) + np.float32(0.5) * ((xs & 1023).astype(np.float32) / np.float32(1024.0))
    clean[..., 1] = np.float32(0.25) + np.float32(0.5) * ((ys & 1023).astype(np.float32) / np.float32(1024.0))
    clean[..., 2] = np.float32(0.5)
    for (x0, y0, bw, bh, col) in boxes(seed, width, height):
        m = (xs >= x0) & (xs < x0 + bw) & (ys >= y0) & (ys < y0 + bh)
        for c in range(3):
            clean[..., c] = np.where(m, col[c], clean[..., c])
    s = noise_scale(sigma)
    idx = (ys * width + xs).astype(np.uint64)
    out = np.empty((rows, width, 4), dtype=np.float32)
    for c in range(3):
        a = (splitmix64(_key(seed, idx, c)) >> np.uint64(41)).astype(np.int64)
        u = (a - (1 << 22)).astype(np.float32) * np.float32(2.0 ** -22)
        v = clean[..., c] + u * s
        out[..., c] = np.clip(v, np.float32(0.0), np.float32(1.0))
    out[..., 3] = np.float32(1.0)
    return out


def thermal_inputs(width: int, height: int, seed: int = 1):
    """(T0, P) float32 (H, W) arrays for the thermal stencil."""
    ys = np.arange(height, dtype=np.int64)[:, None]
    xs = np.arange(width, dtype=np.int64)[None, :]
    idx = (ys * width + xs).astype(np.uint64)
    a = (splitmix64(_key(seed, idx, 0)) >> np.uint64(41)).astype(np.float32) * np.float32(2.0 ** -23)
    b = (splitmix64(_key(seed, idx, 1)) >> np.uint64(41)).astype(np.float32) * np.float32(2.0 ** -23)
    t0 = np.float32(323.15) + a * np.float32(20.0)
    p = b * np.float32(0.05)
    return t0.astype(np.float32), p.astype(np.float32)
