"""Seeded synthetic inputs shared by the tests, smoke() and bench.py.

This module holds NO arithmetic of the PROCLUS method: it only generates
data matrices.  It follows the paper's description of its synthetic
workload: points in ``d`` dimensions with values in
[0, 100], ``n_clusters`` Gaussian clusters each living in a random
``subspace_dim``-dimensional subspace with standard deviation ``sd`` (5.0 by
default), uniform values in the other dimensions, plus a fraction of
uniform noise points (``noise``, our choice: the paper is silent, north_star
says "plus uniform noise").  Every dimension is then min-max normalised to
[0, 1] in fp64 and cast to fp32.  The recipe is restated in
DESIGN.md section 4.
"""
from __future__ import annotations

import numpy as np

# The configurations of BASELINE.json (C1..C4) and the large-n workload L8.
CONFIGS = {
    "C1": dict(n=4_000, d=15, n_clusters=5, subspace_dim=3, k=5, l=3),
    "C2": dict(n=64_000, d=15, n_clusters=10, subspace_dim=5, k=10, l=5),
    "C3": dict(n=1_000_000, d=15, n_clusters=10, subspace_dim=5, k=10, l=5),
    "C4": dict(n=256_000, d=100, n_clusters=20, subspace_dim=10, k=20, l=10),
    # the paper's large-n workload (Fig 3e, > 8M points)
    "L8": dict(n=8_000_000, d=15, n_clusters=10, subspace_dim=5, k=10, l=5),
}


def generate(n: int, d: int, n_clusters: int = 10, subspace_dim: int = 5,
             sd: float = 5.0, noise: float = 0.05, seed: int = 1,
             normalize: bool = True) -> np.ndarray:
    """Return an (n, d) C-contiguous float32 matrix (row-major, point-major)."""
    if n < 1 or d < 1:
        raise ValueError("n and d must be positive")
    rng = np.random.default_rng(np.random.SeedSequence([0x50524F43, seed]))
    n_noise = int(round(noise * n)) if n_clusters > 0 else n
    n_clust = n - n_noise
    out = np.empty((n, d), dtype=np.float64)
    # uniform background everywhere, then overwrite each cluster's subspace
    out[:] = rng.uniform(0.0, 100.0, size=(n, d))
    if n_clusters > 0 and n_clust > 0:
        s = min(subspace_dim, d)
        sizes = np.full(n_clusters, n_clust // n_clusters, dtype=np.int64)
        sizes[: n_clust % n_clusters] += 1
        start = 0
        for c in range(n_clusters):
            dims = rng.permutation(d)[:s]
            centre = rng.uniform(0.0, 100.0, size=s)
            m = int(sizes[c])
            out[start:start + m][:, dims] = centre + sd * rng.standard_normal((m, s))
            start += m
    out = out[rng.permutation(n)]
    if normalize:
        lo = out.min(axis=0)
        hi = out.max(axis=0)
        span = np.where(hi > lo, hi - lo, 1.0)
        out = (out - lo) / span
    return np.ascontiguousarray(out.astype(np.float32))


def config_data(name: str, seed: int = 1) -> tuple[np.ndarray, dict]:
    cfg = dict(CONFIGS[name])
    data = generate(cfg["n"], cfg["d"], cfg["n_clusters"], cfg["subspace_dim"], seed=seed)
    return data, cfg
