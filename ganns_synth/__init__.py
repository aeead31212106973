"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no distance, no search, no
graph construction).  It only draws random numbers with numpy's PCG64 and
shapes them like the paper's workloads (Table I):

* integer-grid point sets (stored as fp32) drawn from a low-rank Gaussian
  mixture -- SURVEY.md §8(d) recipe, restated in DESIGN.md "Input recipe";
* uniformly random fixed-degree adjacency arrays (distinct neighbours, no
  self loop, ragged rows padded with -1 as a suffix) used as *input graphs*
  for search parity at full size;
* the reconstructed Fig. 1 graph G1 fixture lives in tests/golden/, not here.

Both the CUDA path and the oracle consume exactly these arrays.
"""
from __future__ import annotations

import dataclasses
import numpy as np

CHUNK = 1_000_000  # rows per independently seeded chunk


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    index: int          # seed component
    n: int
    d: int
    lo: int
    hi: int
    n_centers: int
    spread: float
    rank: int
    noise: float
    metric: str          # "l2" | "ip" | "cosine"
    nq: int
    degree: int          # d_max; d_min = degree // 2
    k: int = 10
    zipf: float = 0.0    # cluster-weight skew (0 = uniform weights)
    shards: int = 1


# BASELINE.json "configs" C1..C5 (SURVEY.md §8 table, §8(d) generator table)
CONFIGS = {
    "C1": Config("C1", 1, 10_000, 128, 0, 255, 32, 0.25, 16, 0.03, "l2", 100, 16),
    "C2": Config("C2", 2, 1_000_000, 128, 0, 255, 32, 0.25, 16, 0.03, "l2", 10_000, 32),
    "C3": Config("C3", 3, 1_000_000, 960, 0, 127, 32, 0.25, 20, 0.03, "l2", 1_000, 32),
    "C4": Config("C4", 4, 1_183_514, 200, -127, 127, 256, 0.25, 24, 0.03, "cosine", 10_000, 32,
                 zipf=1.1),
    "C5": Config("C5", 5, 100_000_000, 96, -127, 127, 1024, 0.25, 16, 0.03, "l2", 10_000, 32,
                 shards=8),
}


def _structure(cfg: Config):
    """Shared mixture structure: centers, projection and weights (seed [2022, cfg, 99])."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, cfg.index, 99])))
    span = float(cfg.hi - cfg.lo)
    mid = (cfg.hi + cfg.lo) / 2.0
    centers = mid + cfg.spread * span * rng.standard_normal((cfg.n_centers, cfg.d)) / 4.0
    W = rng.standard_normal((cfg.rank, cfg.d)) / np.sqrt(cfg.rank)
    if cfg.zipf > 0:
        w = 1.0 / np.arange(1, cfg.n_centers + 1) ** cfg.zipf
    else:
        w = np.ones(cfg.n_centers)
    return centers.astype(np.float32), W.astype(np.float32), (w / w.sum())


def _draw_rows(cfg: Config, m: int, rng: np.random.Generator, structure) -> np.ndarray:
    centers, W, pi = structure
    span = float(cfg.hi - cfg.lo)
    z = rng.choice(cfg.n_centers, size=m, p=pi)
    g = rng.standard_normal((m, cfg.rank), dtype=np.float32)
    x = centers[z]
    x += (0.15 * span) * (g @ W)
    x += (cfg.noise * span) * rng.standard_normal((m, cfg.d), dtype=np.float32)
    np.rint(x, out=x)
    np.clip(x, cfg.lo, cfg.hi, out=x)
    return np.ascontiguousarray(x, dtype=np.float32)


def with_size(cfg: Config, n: int | None = None, nq: int | None = None, **kw) -> Config:
    """Same distribution, different sizes (parity cases smaller than the config)."""
    return dataclasses.replace(cfg, n=cfg.n if n is None else n,
                               nq=cfg.nq if nq is None else nq, **kw)


def points(cfg: Config, start: int = 0, stop: int | None = None) -> np.ndarray:
    """Base rows [start, stop) -- each 1M-row chunk has its own seed [2022, cfg, 0, chunk],
    so any shard or chunk regenerates alone."""
    stop = cfg.n if stop is None else stop
    assert 0 <= start <= stop <= cfg.n
    st = _structure(cfg)
    out = np.empty((stop - start, cfg.d), dtype=np.float32)
    c0, c1 = start // CHUNK, (stop + CHUNK - 1) // CHUNK
    for c in range(c0, c1):
        lo, hi = c * CHUNK, min((c + 1) * CHUNK, cfg.n)
        rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, cfg.index, 0, c])))
        rows = _draw_rows(cfg, hi - lo, rng, st)
        a, b = max(lo, start), min(hi, stop)
        if a < b:
            out[a - start:b - start] = rows[a - lo:b - lo]
    return out


def queries(cfg: Config, nq: int | None = None) -> np.ndarray:
    """Query rows, same mixture, seed [2022, cfg, 1]."""
    nq = cfg.nq if nq is None else nq
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, cfg.index, 1])))
    return _draw_rows(cfg, nq, rng, _structure(cfg))


def normalize_rows(x: np.ndarray) -> np.ndarray:
    """Input preparation for the cosine config (Table I "Cosine Similarity"):
    rows scaled to unit L2 norm in fp32.  Both sides receive the same array."""
    nrm = np.sqrt((x.astype(np.float64) ** 2).sum(1, keepdims=True))
    nrm[nrm == 0] = 1.0
    return (x / nrm).astype(np.float32)


def random_graph(n: int, d_max: int, seed: int, min_degree: int | None = None) -> np.ndarray:
    """Uniform random fixed-degree digraph as an int32 [n, d_max] adjacency array.

    Row v holds deg(v) ~ U[min_degree, d_max] distinct neighbours != v, then -1
    padding (a suffix).  Used as an *input* for search parity: the search
    semantics do not depend on how the graph was made.
    """
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, 7, seed])))
    min_degree = d_max if min_degree is None else min_degree
    assert 0 <= min_degree <= d_max and d_max <= n - 1
    if n <= 4 * d_max:
        adj = np.stack([rng.permutation(n - 1)[:d_max] for _ in range(n)]).astype(np.int64)
    else:
        adj = rng.integers(0, n - 1, size=(n, d_max), dtype=np.int64)
        while True:
            s = np.sort(adj, axis=1)
            bad = np.nonzero((s[:, 1:] == s[:, :-1]).any(1))[0]
            if bad.size == 0:
                break
            adj[bad] = rng.integers(0, n - 1, size=(bad.size, d_max), dtype=np.int64)
    v = np.arange(n, dtype=np.int64)[:, None]
    adj = adj + (adj >= v)                       # skip the self id
    deg = rng.integers(min_degree, d_max + 1, size=n)
    adj[np.arange(d_max)[None, :] >= deg[:, None]] = -1
    return adj.astype(np.int32)


def random_int_points(n: int, d: int, lo: int, hi: int, seed: int) -> np.ndarray:
    """Small tie-heavy integer-grid point sets for oracle pins and edge cases."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, 8, seed])))
    return rng.integers(lo, hi + 1, size=(n, d)).astype(np.float32)


def hnsw_levels(n: int, d_min: int, seed: int) -> np.ndarray:
    """Top layer of every point for the HNSW extension ("a subset ... randomly
    selected", the higher the fewer): level = floor(-ln(U) * mL), U ~ U(0, 1],
    mL = 1 / ln(d_min) (the standard HNSW normalisation, so each layer keeps about
    1/d_min of the one below).  A seeded input, identical for the oracle and the GPU."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([2022, 9, seed])))
    u = 1.0 - rng.random(n)                      # (0, 1]
    lv = np.floor(-np.log(u) / np.log(d_min)).astype(np.int64)
    return np.minimum(lv, 15).astype(np.int8)
