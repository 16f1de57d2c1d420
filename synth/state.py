"""Seeded BP states for injected-state parity tests (no method arithmetic).

S^p values are a counter-based function of the (row edge, column edge) pair,
sp_value(e, f, seed), so that the CUDA path (which needs the whole S^p in its
CSR order) and the oracle (which evaluates sampled rows by the definition of S)
draw the SAME value for the same nonzero without either side handing its
layout to the other.  splitmix64 on (seed, e, f) -> uniform in [-lo, hi).
"""
from __future__ import annotations

import numpy as np

_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_G = np.uint64(0x9E3779B97F4A7C15)


def _splitmix64(x):
    x = (x + _G).astype(np.uint64)
    x = ((x ^ (x >> np.uint64(30))) * _M1).astype(np.uint64)
    x = ((x ^ (x >> np.uint64(27))) * _M2).astype(np.uint64)
    return (x ^ (x >> np.uint64(31))).astype(np.uint64)


def sp_value(e, f, seed: int = 1, lo: float = -4.0, hi: float = 2.0):
    """S^p value of the nonzero (e, f): deterministic in (seed, e, f)."""
    e = np.asarray(e, dtype=np.uint64)
    f = np.asarray(f, dtype=np.uint64)
    with np.errstate(over="ignore"):
        key = (e << np.uint64(32)) | f
        r = _splitmix64(key ^ _splitmix64(np.full(key.shape, seed, dtype=np.uint64)))
    u = (r >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)  # [0, 1)
    return lo + (hi - lo) * u


def edge_values(m: int, seed: int = 2, scale: float = 3.0):
    """A seeded y^p- or z^p-like vector over the m edges."""
    return np.random.default_rng(seed).normal(size=m) * scale
