"""Seeded synthetic inputs shaped like the paper's workloads.

Shared by the tests, the bench and smoke(): it holds NONE of the method's
arithmetic (no ordering, no keys, no sampling) -- only value generators, so
both the CUDA path and the CPU oracle see identical bits.

Recipe (§V.A):
  * "uniform distribution across a pre-defined set of d distinct values",
    d in {1, 16, 128, 1024, n}, n = 2^16 .. 2^28  -> :func:`distinct`
  * continuous distributions named by north_star: uniform U[0,1), normal
    N(0,1), exponential Exp(1) -> :func:`uniform`, :func:`normal`,
    :func:`exponential`
  * adversarial sets: all-equal, few-distinct, the permutation input whose
    answer has a closed form -> :func:`all_equal`, :func:`permutation`
  * integer data over the full range -> :func:`int_uniform`
  * special IEEE values (+-0, +-inf, NaNs with payloads) -> :func:`specials`
  * random ranks "chosen uniformly at random" (L596-597) -> :func:`rank`

Seeds: dataset seed = 1000 + 17*config_id + dataset_idx; the
rank for random-k runs comes from a separate generator seeded with seed + 1.
All generators are numpy PCG64 on the host.
"""
from __future__ import annotations

import numpy as np


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def dataset_seed(config_id: int, dataset_idx: int) -> int:
    return 1000 + 17 * config_id + dataset_idx


def uniform(n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    return rng(seed).random(n, dtype=np.dtype(dtype))


def normal(n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    return rng(seed).standard_normal(n, dtype=np.dtype(dtype))


def exponential(n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    return rng(seed).standard_exponential(n, dtype=np.dtype(dtype))


def distinct(n: int, d: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    """§V.A: n values drawn uniformly from d distinct values v_j = j."""
    idx = rng(seed).integers(0, d, size=n, dtype=np.int64)
    return idx.astype(np.dtype(dtype))


def all_equal(n: int, value=42.0, dtype=np.float32) -> np.ndarray:
    return np.full(n, value, dtype=np.dtype(dtype))


def permutation(n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    """d = n distinct values in random order.  float: bit patterns
    0x00800000 + pi(i) (distinct positive normals); int: pi(i).  The element
    of rank k then has bits 0x00800000 + k (float) or value k (int)."""
    pi = rng(seed).permutation(n).astype(np.int64)
    dt = np.dtype(dtype)
    if dt == np.float32:
        return (pi + 0x00800000).astype(np.uint32).view(np.float32)
    if dt == np.float64:
        return (pi + 0x0010000000000000).astype(np.uint64).view(np.float64)
    return pi.astype(dt)


def int_uniform(n: int, dtype=np.int32, seed: int = 0) -> np.ndarray:
    dt = np.dtype(dtype)
    info = np.iinfo(dt)
    return rng(seed).integers(info.min, info.max, size=n, dtype=dt, endpoint=True)


def specials(n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    """A mix of ordinary values and IEEE special bit patterns: +-0, +-inf,
    quiet/signalling NaNs of both signs with payloads, denormals."""
    dt = np.dtype(dtype)
    g = rng(seed)
    base = g.standard_normal(n).astype(dt)
    if dt == np.float32:
        pats = np.array([0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000,
                         0xFFC00000, 0x7F800001, 0xFFFFFFFF, 0x7FFFFFFF, 0x00000001,
                         0x80000001, 0x007FFFFF], dtype=np.uint32).view(np.float32)
    else:
        pats = np.array([0, 0x8000000000000000, 0x7FF0000000000000, 0xFFF0000000000000,
                         0x7FF8000000000000, 0xFFF8000000000000, 0x7FF0000000000001,
                         0xFFFFFFFFFFFFFFFF, 0x7FFFFFFFFFFFFFFF, 1, 0x8000000000000001],
                        dtype=np.uint64).view(np.float64)
    mask = g.random(n) < 0.25
    base[mask] = pats[g.integers(0, pats.size, size=int(mask.sum()))]
    return base


def rank(n: int, seed: int) -> int:
    """A rank drawn uniformly at random in [0, n) (L596-597)."""
    return int(rng(seed + 1).integers(0, n))


def make(kind: str, n: int, dtype=np.float32, seed: int = 0) -> np.ndarray:
    """Dispatch by name: uniform, normal, exponential, distinct16, distinct128,
    distinct1024, equal, perm, specials, int (full range)."""
    if kind == "uniform":
        return uniform(n, dtype, seed)
    if kind == "normal":
        return normal(n, dtype, seed)
    if kind == "exponential":
        return exponential(n, dtype, seed)
    if kind.startswith("distinct"):
        return distinct(n, int(kind[len("distinct"):]), dtype, seed)
    if kind == "equal":
        return all_equal(n, 42, dtype)
    if kind == "perm":
        return permutation(n, dtype, seed)
    if kind == "specials":
        return specials(n, dtype, seed)
    if kind == "int":
        return int_uniform(n, dtype, seed)
    raise ValueError(f"unknown input kind {kind!r}")
