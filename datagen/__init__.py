"""Seeded synthetic workloads for the MDMC skycube (shared by the oracle tests and the GPU path).

This module holds NO skycube arithmetic: it only draws numbers.  It is the one module that both
``oracle/`` and the CUDA path (through tests and bench.py) may use, so that both sides see the same
bytes.

Workloads (§7.1 "Datasets"): the benchmark generator of Börzsönyi et al. [5]
with anticorrelated (A), independent (I) and correlated (C) dimensions, n in {1,2.5,5,7.5,10}x1e5,
d in {4..16}.  The generator itself is not in the paper; the reconstruction below is the one stated
in SURVEY.md §8(d) (reading Q13 in DESIGN.md).  A Covertype-shaped tie-heavy stand-in (Table 2,
L1106: CT 581,012 x 10, |S+| = 432,253) is added as "ct".

All values are drawn in float64 with numpy PCG64 and rounded to float32 (round-to-nearest-even);
the rounding creates exact ties at large n, which the method must handle (Def. 1).
"""
from __future__ import annotations

import hashlib
from dataclasses import dataclass

import numpy as np

__all__ = ["generate", "CONFIGS", "Config", "config", "digest", "distinct_columns",
           "chain", "antichain2d"]


def _peak(rng, lo, hi, k, size):
    """Börzsönyi RandomPeak: mean of k uniforms scaled to [lo, hi) (approximately normal)."""
    u = rng.random(size + (k,)).sum(axis=-1) / k
    return lo + (hi - lo) * u


def _independent(rng, n, d):
    return rng.random((n, d))


def _correlated(rng, n, d):
    out = np.empty((n, d))
    filled = 0
    while filled < n:
        m = max(1024, int(1.6 * (n - filled)))
        v = _peak(rng, 0.0, 1.0, d, (m,))              # RandomPeak(0,1,dim)
        x = np.repeat(v[:, None], d, axis=1)
        l = np.minimum(v, 1.0 - v)
        for i in range(d):                              # h = RandomNormal(0, l) = peak(-l, l, 12)
            h = _peak(rng, -l, l, 12, (m,))
            x[:, i] += h
            x[:, (i + 1) % d] -= h
        ok = np.all((x >= 0.0) & (x <= 1.0), axis=1)
        x = x[ok]
        take = min(n - filled, x.shape[0])
        out[filled:filled + take] = x[:take]
        filled += take
    return out


def _anticorrelated(rng, n, d):
    out = np.empty((n, d))
    filled = 0
    while filled < n:
        m = max(1024, int(1.6 * (n - filled)))
        v = _peak(rng, 0.25, 0.75, 12, (m,))            # RandomNormal(0.5, 0.25)
        x = np.repeat(v[:, None], d, axis=1)
        l = np.minimum(v, 1.0 - v)
        for i in range(d):                              # h = RandomEqual(-l, l)
            h = rng.uniform(-l, l)
            x[:, i] += h
            x[:, (i + 1) % d] -= h
        ok = np.all((x >= 0.0) & (x <= 1.0), axis=1)
        x = x[ok]
        take = min(n - filled, x.shape[0])
        out[filled:filled + take] = x[:take]
        filled += take
    return out


# Covertype-like numeric attribute cardinalities (calibrated to |S+|/n ~ 74%).
CT_CARDINALITIES = (1978, 361, 67, 551, 700, 5785, 207, 185, 255, 5827)


def _covertype_like(rng, n, d):
    cards = [CT_CARDINALITIES[i % len(CT_CARDINALITIES)] for i in range(d)]
    out = np.empty((n, d))
    for i, c in enumerate(cards):
        level = np.floor(rng.random(n) * c)
        level[rng.random(n) < 0.12] = 0.0               # skew to the optimum (Table 2 CT, L1106/L1130)
        out[:, i] = level / (c - 1)
    return out


_DISTS = {"I": _independent, "C": _correlated, "A": _anticorrelated, "ct": _covertype_like}


def generate(dist: str, n: int, d: int, seed: int) -> np.ndarray:
    """Return a C-contiguous float32 (n, d) array; row = point id, column i = dimension i = bit i."""
    if dist not in _DISTS:
        raise ValueError(f"unknown distribution {dist!r}")
    rng = np.random.default_rng(seed)
    x = _DISTS[dist](rng, int(n), int(d)) if n > 0 else np.empty((0, d))
    return np.ascontiguousarray(x.astype(np.float32))


def distinct_columns(n: int, d: int, seed: int) -> np.ndarray:
    """Per-dimension random permutations of 0..n-1: the distinct-value condition of L184 holds."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(
        np.stack([rng.permutation(n) for _ in range(d)], axis=1).astype(np.float32))


def chain(n: int, d: int) -> np.ndarray:
    """p_i = (i, ..., i): a total order, only p_0 is in any skyline."""
    return np.ascontiguousarray(np.repeat(np.arange(n, dtype=np.float32)[:, None], d, axis=1))


def antichain2d(n: int) -> np.ndarray:
    """(i, n-1-i): every point in S_3; only the extremes in S_1 / S_2."""
    i = np.arange(n, dtype=np.float32)
    return np.ascontiguousarray(np.stack([i, n - 1 - i], axis=1))


def small_int_grid(n: int, d: int, levels: int, seed: int) -> np.ndarray:
    """Tie-heavy tiny datasets: values in {0..levels-1}."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(rng.integers(0, levels, size=(n, d)).astype(np.float32))


@dataclass(frozen=True)
class Config:
    name: str
    dist: str
    n: int
    d: int
    seed: int

    def data(self) -> np.ndarray:
        return generate(self.dist, self.n, self.d, self.seed)


# BASELINE.json configs (seeds from BASELINE.md §3).  H = the headline metric workload.
CONFIGS = {
    "C1": Config("C1", "I", 1_000, 4, 1),
    "C2": Config("C2", "I", 100_000, 8, 2),
    "C3C": Config("C3C", "C", 500_000, 12, 3),
    "C3A": Config("C3A", "A", 500_000, 12, 4),
    "C3I": Config("C3I", "I", 500_000, 12, 5),
    "C4": Config("C4", "A", 1_000_000, 16, 6),
    "H": Config("H", "A", 1_000_000, 12, 7),
    "C5": Config("C5", "ct", 581_012, 10, 8),
}


def config(name: str) -> Config:
    return CONFIGS[name]


def digest(x: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(x).tobytes()).hexdigest()
