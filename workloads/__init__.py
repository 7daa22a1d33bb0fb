"""Seeded synthetic inputs shared by the oracle tests, the parity tests and bench.py.

This module holds NO arithmetic of the self-join method (no distances, no grid,
no cell ids): only the random point generators and the frozen configurations
(point count, dimensionality, distribution, epsilon) of SURVEY.md §8.0.  Both the
CPU oracle (``oracle/``) and the CUDA path (``paper_conf_ipps_galletg19_b200``)
consume the arrays it returns; neither side imports the other.

Distributions follow the paper's workloads (§IV-A):
  * uniform          -- "synthetically generated with a uniform ... distribution",
                        read as U[0,1)^n (reading c16);
  * exponential      -- "an exponential distribution with lambda = 40", read as
                        i.i.d. Exp(rate 40) per coordinate (reading c15);
  * sw (space-weather shaped) -- the SW datasets are "latitude and longitude"
                        (PAPER.md:208); the real data [31] is unavailable, so a
                        clustered (lon, lat) mixture stands in (recipe below).
Epsilon is chosen from a target mean neighbour count K by the closed forms of
SURVEY.md §8.0 (boundary effects ignored), because the paper's epsilons refer to
an unstated data scale (reading c15).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

__all__ = [
    "Config", "CONFIGS", "get_config", "gen_points", "eps_for_k",
    "uniform", "exponential", "sw_shaped", "lattice", "duplicates", "clusters",
]


def uniform(n: int, dim: int, seed: int) -> np.ndarray:
    """U[0,1)^dim, float64, C-contiguous (N, dim)."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(rng.random((n, dim), dtype=np.float64))


def exponential(n: int, dim: int, seed: int, lam: float = 40.0) -> np.ndarray:
    """i.i.d. Exp(rate=lam) per coordinate (mean 1/lam) -- PAPER.md:208."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(rng.exponential(1.0 / lam, size=(n, dim)).astype(np.float64))


def sw_shaped(n: int, seed: int, n_clusters: int = 60, frac_clustered: float = 0.9) -> np.ndarray:
    """2-D (lon, lat) in degrees, shaped like GNSS-TEC receiver density.

    90 % of the points come from ``n_clusters`` anisotropic Gaussian clusters
    (centres lat ~ U[-55, 70], lon ~ U[-180, 180]; sigma_lat ~ U[1, 8] deg,
    sigma_lon ~ U[1.5, 12] deg; Zipf(1.2) cluster weights); 10 % are uniform on
    the sphere.  lat is clipped to [-90, 90], lon wrapped to [-180, 180), and the
    rows are shuffled.
    """
    rng = np.random.default_rng(seed)
    n_cl = int(round(n * frac_clustered))
    n_un = n - n_cl
    c_lat = rng.uniform(-55.0, 70.0, n_clusters)
    c_lon = rng.uniform(-180.0, 180.0, n_clusters)
    s_lat = rng.uniform(1.0, 8.0, n_clusters)
    s_lon = rng.uniform(1.5, 12.0, n_clusters)
    w = 1.0 / np.arange(1, n_clusters + 1, dtype=np.float64) ** 1.2
    w /= w.sum()
    which = rng.choice(n_clusters, size=n_cl, p=w)
    lat = c_lat[which] + s_lat[which] * rng.standard_normal(n_cl)
    lon = c_lon[which] + s_lon[which] * rng.standard_normal(n_cl)
    u_lon = rng.uniform(-180.0, 180.0, n_un)
    u_lat = np.degrees(np.arcsin(rng.uniform(-1.0, 1.0, n_un)))
    lat = np.clip(np.concatenate([lat, u_lat]), -90.0, 90.0)
    lon = np.concatenate([lon, u_lon])
    lon = (lon + 180.0) % 360.0 - 180.0
    pts = np.stack([lon, lat], axis=1)
    pts = pts[rng.permutation(n)]
    return np.ascontiguousarray(pts, dtype=np.float64)


def lattice(g: int, dim: int, spacing: float = 1.0) -> np.ndarray:
    """The integer lattice {0..g-1}^dim scaled by ``spacing`` (closed-form pins)."""
    axes = [np.arange(g, dtype=np.float64) * spacing] * dim
    mesh = np.meshgrid(*axes, indexing="ij")
    return np.ascontiguousarray(np.stack([m.ravel() for m in mesh], axis=1))


def duplicates(n: int, dim: int, value: float = 0.25) -> np.ndarray:
    """n copies of the same point (every i != j pair is at distance 0)."""
    return np.full((n, dim), value, dtype=np.float64)


def clusters(centres, per_cluster: int, sigma: float, seed: int) -> np.ndarray:
    """Gaussian clusters (isotropic sigma) of ``per_cluster`` points around each row of
    ``centres`` (k, dim), shuffled: sparse grids whose non-empty cells are few and far apart
    (the hashed lid -> cell lookup, 64-bit cell keys)."""
    rng = np.random.default_rng(seed)
    c = np.asarray(centres, dtype=np.float64)
    pts = np.repeat(c, per_cluster, axis=0) + sigma * rng.standard_normal((c.shape[0] * per_cluster, c.shape[1]))
    return np.ascontiguousarray(pts[rng.permutation(pts.shape[0])])


def eps_for_k(dist: str, n: int, dim: int, k: float, lam: float = 40.0) -> float:
    """Epsilon giving a mean of ~k neighbours (SURVEY.md §8.0 closed forms, no boundary effects).

    uniform on [0,1)^dim: k = n * V_dim * eps^dim with V_dim the unit-ball volume.
    exponential (rate lam): the density at the origin corner region is
    approximated as in SURVEY.md §8.0 by n * V_dim * (lam/2)^dim * eps^dim.
    """
    v = math.pi ** (dim / 2.0) / math.gamma(dim / 2.0 + 1.0)
    if dist == "uniform":
        return (k / (n * v)) ** (1.0 / dim)
    if dist == "exponential":
        return (k / (n * v * (lam / 2.0) ** dim)) ** (1.0 / dim)
    raise ValueError(dist)


@dataclass(frozen=True)
class Config:
    name: str
    dist: str            # uniform | exponential | sw
    n: int
    dim: int
    eps: float
    seed: int
    k: int = 8           # threads per query point
    note: str = ""
    extra: dict = field(default_factory=dict, compare=False, hash=False)

    def points(self) -> np.ndarray:
        return gen_points(self.dist, self.n, self.dim, self.seed)

    def scaled(self, n: int, name: str | None = None) -> "Config":
        """Same distribution and expected neighbour count at a smaller n (parity sizes)."""
        if self.dist == "sw":
            eps = self.eps * math.sqrt(self.n / n)
        else:
            eps = self.eps * (self.n / n) ** (1.0 / self.dim)
        return Config(name or f"{self.name}@{n}", self.dist, n, self.dim, eps, self.seed + 1000, self.k,
                      f"scaled from {self.name}")


def gen_points(dist: str, n: int, dim: int, seed: int) -> np.ndarray:
    if dist == "uniform":
        return uniform(n, dim, seed)
    if dist == "exponential":
        return exponential(n, dim, seed)
    if dist == "sw":
        if dim != 2:
            raise ValueError("sw-shaped data is 2-D (lon, lat)")
        return sw_shaped(n, seed)
    raise ValueError(dist)


def _build() -> dict:
    c = {}
    c["c1"] = Config("c1", "uniform", 10_000, 2, eps_for_k("uniform", 10_000, 2, 32), 1, 8,
                     "2-D uniform, 10^4 points, ~32 neighbours (BASELINE.json configs[0])")
    for kk in (16, 32, 64, 128, 256):
        c[f"c2k{kk}"] = Config(f"c2k{kk}", "uniform", 2_000_000, 2, eps_for_k("uniform", 2_000_000, 2, kk), 2, 8,
                               f"2-D uniform, 2M points, ~{kk} neighbours (configs[1] sweep)")
    for kk in (16, 64, 256):
        c[f"c3k{kk}"] = Config(f"c3k{kk}", "exponential", 2_000_000, 3,
                               eps_for_k("exponential", 2_000_000, 3, kk), 3, 8,
                               f"3-D exponential lambda=40, 2M points, ~{kk} neighbours (configs[2])")
    for kk in (8, 32, 128):
        c[f"c4k{kk}"] = Config(f"c4k{kk}", "uniform", 2_000_000, 6, eps_for_k("uniform", 2_000_000, 6, kk), 4, 8,
                               f"6-D uniform, 2M points, ~{kk} neighbours, k=8 (configs[3])")
    c["c5"] = Config("c5", "sw", 5_000_000, 2, 0.1, 5, 8,
                     "2-D space-weather-shaped, 5M points, eps=0.1 deg, > 1 batch (configs[4])")
    c["c5e02"] = Config("c5e02", "sw", 5_000_000, 2, 0.2, 5, 8, "C5 stress, eps=0.2 deg (~19 batches)")
    # primary aliases (SURVEY.md §8.0 bold rows)
    c["c2"] = c["c2k64"]
    c["c3"] = c["c3k64"]
    c["c4"] = c["c4k32"]
    return c


CONFIGS = _build()


def get_config(name: str) -> Config:
    try:
        return CONFIGS[name]
    except KeyError:
        raise KeyError(f"unknown config {name!r}; known: {sorted(CONFIGS)}") from None
