"""Seeded synthetic workloads for PSB kNN (inputs only — no kNN arithmetic here).

This module is the ONE thing shared by the oracle (`oracle/`) and the CUDA path
(`paper_conf_icpp_namkn16_b200/`): it produces the point sets and query batches
both sides consume, byte for byte. It holds none of the method's arithmetic
(no distances, no bounding boxes, no selection).

Recipe (DESIGN.md §3 "Input recipe"):

* ``u24(seed, i) = (mix64(seed + (i + 1) * GAMMA) >> 40) * 2**-24`` — a
  counter-based SplitMix64 stream; every value is an exact binary32 in [0, 1).
* Uniform points: ``x[i][j] = u24(seed, i*d + j)``.
* Clustered points (paper's workload shape, §IV-D "1M points =
  100 normal distributions x 10,000", L817-823 §V-A, L841-843 §V-B): C = 100
  Gaussian clusters; centre ``c[m][j] = float32(1e4 * u24(seed ^ 0xC1, m*d + j))``;
  point i belongs to cluster ``m = i // ceil(n / C)``;
  ``x[i][j] = float32(c[m][j] + sigma * g)``, g standard normal by Box-Muller in
  float64 from the same counter stream.  sigma = 160 by default (the paper's
  Fig. 6 setting).
* Queries follow the points' distribution with a different seed; clustered
  queries reuse the points' centres (cluster ``m = mix64(qseed ^ i) % C``) so
  queries land inside the data, as the paper's queries do.

Seeds: points ``0x5053420000 + cfg``, queries ``0x5053510000 + cfg``.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_CHUNK = 1 << 24  # values per vectorised chunk (bounds temporaries to ~0.5 GB)


def mix64(z: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on a uint64 array (wrapping arithmetic)."""
    z = z.astype(np.uint64, copy=True)
    z ^= z >> np.uint64(30)
    z *= _M1
    z ^= z >> np.uint64(27)
    z *= _M2
    z ^= z >> np.uint64(31)
    return z


def _u24_range(seed: int, start: int, count: int) -> np.ndarray:
    """u24(seed, i) for i in [start, start+count) as float64 (exact 24-bit values)."""
    with np.errstate(over="ignore"):
        i = np.arange(start + 1, start + count + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + i * GAMMA
        return (mix64(z) >> np.uint64(40)).astype(np.float64) * (2.0 ** -24)


def u24(seed: int, start: int, count: int) -> np.ndarray:
    out = np.empty(count, dtype=np.float64)
    for s in range(0, count, _CHUNK):
        c = min(_CHUNK, count - s)
        out[s:s + c] = _u24_range(seed, start + s, c)
    return out


def gen_uniform(n: int, d: int, seed: int, row0: int = 0) -> np.ndarray:
    """Rows [row0, row0+n) of the uniform set: n x d float32, coordinates u24 in [0, 1)."""
    out = np.empty(n * d, dtype=np.float32)
    for s in range(0, n * d, _CHUNK):
        c = min(_CHUNK, n * d - s)
        out[s:s + c] = _u24_range(seed, row0 * d + s, c).astype(np.float32)
    return out.reshape(n, d)


def _normals(seed: int, start: int, count: int) -> np.ndarray:
    """Standard normals g[t], t in [start, start+count): Box-Muller on u24 pairs."""
    u = _u24_range(seed, 2 * start, 2 * count)
    u1 = u[0::2] + 2.0 ** -25          # (0, 1): log never sees 0
    u2 = u[1::2]
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * math.pi * u2)


def cluster_centres(d: int, seed: int, clusters: int = 100) -> np.ndarray:
    return (1e4 * u24(seed ^ 0xC1, 0, clusters * d)).astype(np.float32).reshape(clusters, d)


def gen_clustered(n: int, d: int, seed: int, sigma: float = 160.0,
                  clusters: int = 100, row0: int = 0, n_total: int | None = None) -> np.ndarray:
    """Rows [row0, row0+n) of an n_total-point set (default n): `clusters` Gaussian
    blobs, contiguous id blocks per cluster."""
    n_total = n if n_total is None else n_total
    c = cluster_centres(d, seed, clusters).astype(np.float64)
    per = -(-n_total // clusters)
    out = np.empty((n, d), dtype=np.float32)
    rows = max(1, _CHUNK // d)
    for s in range(0, n, rows):
        r = min(rows, n - s)
        m = np.arange(row0 + s, row0 + s + r) // per
        g = _normals(seed, (row0 + s) * d, r * d).reshape(r, d)
        out[s:s + r] = (c[m] + sigma * g).astype(np.float32)
    return out


def gen_clustered_queries(q: int, d: int, points_seed: int, qseed: int,
                          sigma: float = 160.0, clusters: int = 100) -> np.ndarray:
    """Queries drawn around the POINTS' centres (centre seed from the points seed)."""
    c = cluster_centres(d, points_seed, clusters).astype(np.float64)
    with np.errstate(over="ignore"):
        m = (mix64(np.uint64(qseed) ^ np.arange(q, dtype=np.uint64))
             % np.uint64(clusters)).astype(np.int64)
    g = _normals(qseed, 0, q * d).reshape(q, d)
    return (c[m] + sigma * g).astype(np.float32)


@dataclasses.dataclass(frozen=True)
class Config:
    """One BASELINE.json config."""
    name: str
    dist: str          # "uniform" | "clustered"
    n: int
    d: int
    fanout: int
    q: int
    k: int
    sigma: float = 160.0
    cfg_id: int = 0

    @property
    def points_seed(self) -> int:
        return 0x5053420000 + self.cfg_id

    @property
    def queries_seed(self) -> int:
        return 0x5053510000 + self.cfg_id

    def points(self, n: int | None = None, row0: int = 0) -> np.ndarray:
        """Rows [row0, row0+n) of this config's point set (all rows by default;
        a data-sharded rank asks for its slab)."""
        n = self.n - row0 if n is None else n
        if self.dist == "uniform":
            return gen_uniform(n, self.d, self.points_seed, row0)
        return gen_clustered(n, self.d, self.points_seed, self.sigma, row0=row0, n_total=self.n)

    def queries(self, q: int | None = None) -> np.ndarray:
        q = self.q if q is None else q
        if self.dist == "uniform":
            return gen_uniform(q, self.d, self.queries_seed)
        return gen_clustered_queries(q, self.d, self.points_seed, self.queries_seed, self.sigma)

    def describe(self) -> dict:
        return {"workload": self.name, "points": self.dist, "n": self.n, "d": self.d,
                "fanout": self.fanout, "q": self.q, "k": self.k,
                **({"sigma": self.sigma, "clusters": 100} if self.dist == "clustered" else {})}


# BASELINE.json "configs", in order (C1 is the oracle-in-seconds case).
CONFIGS = {
    "C1": Config("C1", "uniform", 10_000, 2, 32, 100, 8, cfg_id=1),
    "C2": Config("C2", "clustered", 1_000_000, 3, 64, 10_000, 32, cfg_id=2),
    "C3": Config("C3", "uniform", 4_000_000, 8, 128, 100_000, 16, cfg_id=3),
    "C4": Config("C4", "clustered", 16_000_000, 16, 128, 10_000, 64, cfg_id=4),
    "C5": Config("C5", "uniform", 512_000_000, 3, 128, 1_000_000, 32, cfg_id=5),
    # SURVEY.md §8(d) "ctx": the paper's own experiment shape (§V-B: 64-D
    # clustered points, 240 kNN queries), optional context, not a BASELINE config
    "CTX": Config("CTX", "clustered", 1_000_000, 64, 128, 240, 32, cfg_id=6),
}


def config(name: str, **over) -> Config:
    return dataclasses.replace(CONFIGS[name], **over) if over else CONFIGS[name]
