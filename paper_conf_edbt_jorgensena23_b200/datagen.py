"""Seeded synthetic inputs shaped like the paper's workloads.

This module holds NO arithmetic of the method (no neighbourhoods, no Eq.1,
no grid). It is the one piece shared by the CUDA path's tests/bench and the
oracle's tests: both sides draw their inputs from here and nothing else.

Recipe (§5 "Synthetic data"; L290 / L70 min/max normalisation):
Gaussian clusters in [-100, 100]^d with standard deviation 5.0, optional
uniform noise in the same range, then per-dimension min/max normalisation to
[0, 1].  The generator of Beer et al. [4] is not available, so the draw order
is fixed here (numpy PCG64 via ``default_rng(seed)``, fp64 throughout):

1. centres ~ U[-100, 100]^{k x d}
2. m = n - round(noise * n) clustered points; cluster sizes m // k, the first
   m % k clusters get one extra point
3. clustered points ~ N(centre, 5.0^2 I), cluster by cluster
4. noise points ~ U[-100, 100]^d
5. per-dimension min/max normalisation to [0, 1]
6. shuffle rows with rng.permutation(n)
7. cast to float32 and clip to [0, 1]
"""
from __future__ import annotations

import dataclasses

import numpy as np

__all__ = ["Config", "CONFIGS", "blobs", "make_config"]


@dataclasses.dataclass(frozen=True)
class Config:
    """One BASELINE.json workload."""

    name: str
    n: int
    d: int
    k: int
    noise: float
    eps: float
    std: float = 5.0

    def generate(self, seed: int = 0) -> np.ndarray:
        return blobs(self.n, self.d, self.k, noise=self.noise, std=self.std, seed=seed)


#: BASELINE.json ``configs`` (C1..C5) plus the paper's Table-1 workload (T1).
CONFIGS = {
    "C1": Config("C1", 1_000, 2, 5, 0.0, 0.05),
    "C2": Config("C2", 70_000, 5, 10, 0.0, 0.05),
    "C3": Config("C3", 1_000_000, 10, 20, 0.05, 0.1),
    "C5": Config("C5", 10_000_000, 3, 10, 0.0, 0.05),
    "T1": Config("T1", 1_024_000, 2, 5, 0.0, 0.05),
}


def make_config(name: str) -> Config:
    """``C4-d<dim>`` gives the dimension-sweep point (n=100k, k=5, eps=0.05)."""
    if name.startswith("C4-d"):
        return Config(name, 100_000, int(name[4:]), 5, 0.0, 0.05)
    return CONFIGS[name]


def blobs(n: int, d: int, k: int, *, noise: float = 0.0, std: float = 5.0,
          seed: int = 0, lo: float = -100.0, hi: float = 100.0) -> np.ndarray:
    """Return an (n, d) float32 C-contiguous array in [0, 1]^d."""
    if n < 1 or d < 1 or k < 1:
        raise ValueError("n, d, k must be >= 1")
    rng = np.random.default_rng(seed)
    centres = rng.uniform(lo, hi, size=(k, d))
    m = n - int(round(noise * n))
    sizes = [m // k + (1 if c < m % k else 0) for c in range(k)]
    parts = [rng.normal(centres[c], std, size=(sizes[c], d)) for c in range(k)]
    if n - m > 0:
        parts.append(rng.uniform(lo, hi, size=(n - m, d)))
    x = np.concatenate(parts, axis=0)
    mn = x.min(axis=0)
    span = x.max(axis=0) - mn
    span[span == 0.0] = 1.0
    x = (x - mn) / span
    x = x[rng.permutation(n)]
    return np.ascontiguousarray(np.clip(x.astype(np.float32), 0.0, 1.0))


def uniform(n: int, d: int, seed: int = 0) -> np.ndarray:
    """Uniform [0,1]^d points (edge-case tests: no cluster structure)."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(rng.random((n, d)).astype(np.float32))


def bridge(m: int = 200, b: int = 3, seed: int = 0) -> np.ndarray:
    """Fig 1 (L89) shaped input: two tight 2-D clusters of m points (std 0.002) at x = 0.40
    and 0.48 (0.08 apart, more than eps = 0.05) and a small bridge of b points at x = 0.44,
    within eps of both.  Used with eps = 0.05 to show lambda-termination stopping early."""
    rng = np.random.default_rng(seed)
    a = np.c_[rng.normal(0.40, 0.002, m), rng.normal(0.5, 0.002, m)]
    c = np.c_[rng.normal(0.48, 0.002, m), rng.normal(0.5, 0.002, m)]
    br = np.c_[np.full(b, 0.44) + rng.normal(0, 0.001, b), np.full(b, 0.5)]
    return np.ascontiguousarray(np.vstack([a, c, br]).astype(np.float32))
