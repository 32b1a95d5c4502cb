"""B200-native (sm_100a) occupancy-tuned hot path of Orion (Hayes et al., Middleware '16).

The product is liborion.so (C ABI in include/orion.h): occupancy levels, the
multi-version binary, level-realising launches and the Fig. 8/9 tuner, plus the
hand-written sm_100a kernels (KNN / NLM imageDenoising, register-heavy NLM,
thermal stencil).  ``orion`` is a thin ctypes binding of that ABI.
"""
from . import orion  # noqa: F401
from .orion import *  # noqa: F401,F403
