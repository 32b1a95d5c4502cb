"""Test infrastructure: the UNCHANGED oracle (oracle.denoise / oracle.srad / oracle.hotspot)
called on row chunks from several host threads at once (ctypes releases the GIL inside the C
oracle), so whole configured-size frames can be checked element by element in seconds.
No arithmetic of the method lives here: only the partition of rows over threads."""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

import oracle


def threads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:
        return os.cpu_count() or 1


def denoise_rows(kind: str, img: np.ndarray, height: int, row0: int, y_begin: int, y_end: int,
                 chunk: int = 8):
    """oracle.denoise over global rows [y_begin, y_end) of the slab `img` (global rows
    [row0, row0 + len(img))), split into `chunk`-row calls on every host thread."""
    n = y_end - y_begin
    W = img.shape[1]
    out = np.empty((n, W, 3), np.float64)
    alt = np.empty((n, W, 3), np.float64)
    amb = np.empty((n, W), bool)

    def one(y):
        y1 = min(y_end, y + chunk)
        o, a, m = oracle.denoise(kind, img, height=height, row0=row0, y_begin=y, y_end=y1)
        out[y - y_begin:y1 - y_begin], alt[y - y_begin:y1 - y_begin], amb[y - y_begin:y1 - y_begin] = o, a, m

    with ThreadPoolExecutor(threads()) as ex:
        list(ex.map(one, range(y_begin, y_end, chunk)))
    return out, alt, amb


def map_threads(fn, items):
    with ThreadPoolExecutor(threads()) as ex:
        return list(ex.map(fn, items))
