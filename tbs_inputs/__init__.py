"""Seeded synthetic inputs shared by the oracle, the tests and the bench.

This module holds NONE of the method's arithmetic: it only produces the input
bytes (AoS ``float32[n][dim]`` point sets) that both the oracle and the CUDA path
consume. Everything is integer-only (splitmix64, 24-bit fixed point) so the bytes
are identical on any host. Workload recipes follow the paper's "uniformly
distributed" synthetic particles plus the clustered
and lattice sets of SURVEY.md §8(d); the exact recipe is restated in DESIGN.md
§Inputs.

splitmix64 is used in counter form: draw k (k = 0, 1, ...) of stream ``seed`` is
``mix(seed + (k + 1) * GAMMA)``, so any slice of the stream is computed directly
and the generators are vectorised with numpy.
"""
from __future__ import annotations

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
TWO_M24 = np.float32(2.0 ** -24)

# Clustered-set constants (SURVEY §8(d) generator spec).
CLUSTER_K = 1024                      # parents
CLUSTER_BG_THRESH = 1677722           # background if (v >> 40) < 10% of 2^24
CLUSTER_S = 18162                     # round(0.01 * sqrt(3) * 2^20): sigma_c = 0.01


def splitmix64(seed: int, start: int, count: int) -> np.ndarray:
    """Draws ``start .. start+count-1`` of the splitmix64 stream ``seed`` (uint64)."""
    with np.errstate(over="ignore"):
        k = np.arange(start + 1, start + 1 + count, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + k * GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _u24(draws: np.ndarray) -> np.ndarray:
    return (draws >> np.uint64(40)).astype(np.int64)


def uniform(n: int, seed: int, dim: int = 3) -> np.ndarray:
    """n points uniform in [0,1)^dim, point-major (x, y, z per point), exact fp32."""
    u = _u24(splitmix64(seed, 0, n * dim))
    return (u.astype(np.float32) * TWO_M24).reshape(n, dim)


def clustered(n: int, seed: int, k_parents: int = CLUSTER_K) -> np.ndarray:
    """Clustered 3-D set: 90% children around K uniform parents, 10% background.

    Draws: 3K parent coordinates first; then 13 draws per point: v, then 12 u24.
    Background if (v >> 40) < CLUSTER_BG_THRESH, coordinates = the first three u24.
    Otherwise parent = v & (K-1) (low bits: the top bits were used by the
    background test) and each coordinate gets an Irwin-Hall(4) offset
    ((sum of 4 u24) - 2^25) * S >> 20 (std 0.01), wrapped mod 2^24.
    """
    assert k_parents & (k_parents - 1) == 0
    par = _u24(splitmix64(seed, 0, 3 * k_parents)).reshape(k_parents, 3)
    d = splitmix64(seed, 3 * k_parents, 13 * n).reshape(n, 13)
    v = d[:, 0]
    u = _u24(d[:, 1:]).reshape(n, 3, 4)
    background = _u24(v) < CLUSTER_BG_THRESH
    parent = (v & np.uint64(k_parents - 1)).astype(np.int64)
    off = ((u.sum(axis=2) - (1 << 25)) * CLUSTER_S) >> 20          # int64, arithmetic shift
    child = (par[parent] + off) & ((1 << 24) - 1)
    bg = u[:, :, 0]
    ci = np.where(background[:, None], bg, child)
    return ci.astype(np.float32) * TWO_M24


def lattice(L: int, seed: int) -> np.ndarray:
    """The full cubic lattice {0..L-1}^3 (integer-valued fp32) in a seeded random order.

    The permutation is the stable argsort of one splitmix64 draw per point.
    """
    a = np.arange(L, dtype=np.int64)
    g = np.stack(np.meshgrid(a, a, a, indexing="ij"), axis=-1).reshape(-1, 3)
    perm = np.argsort(splitmix64(seed, 0, L ** 3), kind="stable")
    return g[perm].astype(np.float32)


def make(kind: str, n: int, seed: int, dim: int = 3) -> np.ndarray:
    """Dispatch by name: 'uniform' | 'clustered' | 'lattice' (n must be a cube)."""
    if kind == "uniform":
        return uniform(n, seed, dim)
    if kind == "clustered":
        assert dim == 3
        return clustered(n, seed)
    if kind == "lattice":
        L = round(n ** (1.0 / 3.0))
        assert L ** 3 == n and dim == 3, "lattice needs n = L^3"
        return lattice(L, seed)
    raise ValueError(kind)
