"""Seeded synthetic inputs shaped like the paper's workloads (shared by both sides).

This module holds NO arithmetic of the method (no reduce, scan, fold,
distance or combine): it only draws seeded random arrays.  It is the one
module both the oracle-side tests and the CUDA-side callers use, so that the
two sides see the same bytes.  Recipes:

  C1  i32 full range [-2^31, 2^31) (exercises wrap-around), n = 2^20, seed 1;
      small-range variant [-1000, 1000].                      (BASELINE configs[0])
  C2  Rodinia NN: base of 42,764 (lat, lng) records, lat ~ U[-90, 90),
      lng ~ U[-180, 180) f32, seed 2, duplicated 20 times
      -> 855,280 records; query (30, 90).                     (configs[1])
  C3  Rodinia K-means kdd_cup shape (L1634): n = 494,019, d = 34 points
      U[0,1) f32 (seed 3); membership keys for k = 5 drawn U{0..k-1}
      (seed 4), "clustered" (points = centre[key] + noise) or "skewed"
      (90% in cluster 0).                                     (configs[2])
  C4  U[0,1) f32, n = 2^28 (seed 5), segment-length sweep.    (configs[3])
  C5  k-means n = 2^26, d = 34, k = 32, shard r drawn with seed 5000 + r on
      the device; transpose input [2^14][2^14] U[0,1) f32 (seed 6). (configs[4])

Host arrays use ``numpy.random.default_rng(seed)``; device arrays (sizes too
large to draw on the host) use ``torch.Generator(device).manual_seed(seed)``.
The two generators give different bytes; every consumer of a device array
copies THAT array to the host for the oracle.
"""
from __future__ import annotations

import numpy as np

NN_BASE = 42_764
NN_REPS = 20
NN_QUERY = (30.0, 90.0)
KDD_N, KDD_D, KDD_K = 494_019, 34, 5
C4_N = 1 << 28
C5_N, C5_D, C5_K = 1 << 26, 34, 32
C5_T = 1 << 14
C4_SEGLENS = sorted(set([1 << j for j in range(29)] + [3, 7, 33, 1000, 4097, 65537, 1_000_003]))


def rng(seed: int) -> np.random.Generator:
    return np.random.default_rng(seed)


def ints(n: int, seed: int, low: int, high: int, dtype=np.int32) -> np.ndarray:
    """n integers uniform in [low, high)."""
    return rng(seed).integers(low, high, size=n, dtype=np.int64).astype(dtype)


def uniform(shape, seed: int, low: float = 0.0, high: float = 1.0, dtype=np.float32) -> np.ndarray:
    """Uniform [low, high) floats drawn in f64 then rounded to ``dtype``."""
    return (rng(seed).random(shape) * (high - low) + low).astype(dtype)


def mixed(shape, seed: int, dtype) -> np.ndarray:
    """Signed test data for any table dtype: ints in [-1000, 1000], floats in [-1, 1)."""
    dtype = np.dtype(dtype)
    n = int(np.prod(shape))
    if dtype.kind == "i":
        return ints(n, seed, -1000, 1001, dtype).reshape(shape)
    return uniform(shape, seed, -1.0, 1.0, dtype)


def full_range(shape, seed: int, dtype) -> np.ndarray:
    """Integers over the full range of ``dtype`` (wrap-around exercise), floats U[0,1)."""
    dtype = np.dtype(dtype)
    n = int(np.prod(shape))
    if dtype == np.int32:
        return ints(n, seed, -(1 << 31), 1 << 31, np.int32).reshape(shape)
    if dtype == np.int64:
        r = rng(seed)
        hi = r.integers(-(1 << 31), 1 << 31, size=n, dtype=np.int64)
        lo = r.integers(0, 1 << 32, size=n, dtype=np.int64)
        return ((hi << 32) | lo).astype(np.int64).reshape(shape)
    return uniform(shape, seed, dtype=dtype)


def c1(n: int = 1 << 20, seed: int = 1, small_range: bool = False) -> np.ndarray:
    if small_range:
        return ints(n, seed, -1000, 1001)
    return ints(n, seed, -(1 << 31), 1 << 31)


def c2_nn(base: int = NN_BASE, reps: int = NN_REPS, seed: int = 2):
    """(lat, lng, query): the base set tiled ``reps`` times (L1637 "duplicated 20 times")."""
    r = rng(seed)
    lat = (r.random(base) * 180.0 - 90.0).astype(np.float32)
    lng = (r.random(base) * 360.0 - 180.0).astype(np.float32)
    return np.tile(lat, reps), np.tile(lng, reps), NN_QUERY


def c3_kmeans(n: int = KDD_N, d: int = KDD_D, k: int = KDD_K, seed: int = 3, keys: str = "uniform"):
    """(points [n][d] f32, membership [n] i32)."""
    pts = uniform((n, d), seed)
    if keys == "uniform":
        mem = ints(n, seed + 1, 0, k)
    elif keys == "skewed":
        r = rng(seed + 1)
        mem = np.where(r.random(n) < 0.9, 0, r.integers(1, max(k, 2), size=n)).astype(np.int32)
        mem = np.minimum(mem, k - 1).astype(np.int32)
    elif keys == "clustered":
        r = rng(seed + 1)
        centres = r.random((k, d)).astype(np.float32)
        mem = r.integers(0, k, size=n).astype(np.int32)
        pts = (centres[mem] + (r.random((n, d)) * 0.1 - 0.05)).astype(np.float32)
    else:
        raise ValueError(keys)
    return pts, mem


def c4(n: int = C4_N, seed: int = 5) -> np.ndarray:
    return uniform(n, seed)


def device_uniform(shape, seed: int, device, low: float = 0.0, high: float = 1.0, dtype=None):
    """Uniform floats drawn directly on ``device`` (bench-scale inputs)."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    t = torch.rand(shape, generator=g, device=device, dtype=dtype or torch.float32)
    if low != 0.0 or high != 1.0:
        t.mul_(high - low).add_(low)
    return t


def device_ints(shape, seed: int, device, low: int, high: int, dtype=None):
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return torch.randint(low, high, shape, generator=g, device=device, dtype=dtype or torch.int32)


def c5_kmeans_shard(rank: int, device, n: int = C5_N, d: int = C5_D, k: int = C5_K):
    """Rank ``rank``'s shard: points [n][d] f32 U[0,1) and keys U{0..k-1}, seed 5000 + rank."""
    pts = device_uniform((n, d), 5000 + rank, device)
    mem = device_ints((n,), 7000 + rank, device, 0, k)
    return pts, mem
