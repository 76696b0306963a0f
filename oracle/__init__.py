"""CPU oracle for the 2-BS hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package. The product package
(``paper_conf_icpp_pitaksirianannt16_b200``) never imports it and shares no code
with it. The arithmetic lives in ``tbs_oracle.c`` (plain C + OpenMP, double
precision); this file only marshals numpy arrays through ctypes.

Functions and their pins (tests/test_oracle_pins.py):
  sdh            brute force (numpy pdist-style), mass, hand cases, cube closed form
  sdh_lattice    hand cases (edge ties), brute force, closed form lattice_closed
  pcf            brute force, cumulative-SDH identity, cube closed form
  pairmatrix     torch.cdist float64 (library routine), symmetry, diagonal
  lattice_closed brute force of sdh_lattice on permuted lattices
  kde            brute force (scipy pdist), closed form for coincident / two-point sets
  sdh_bands      = sdh (same loop) + the 5e-7 diagnostic band counts; band nesting, brute force
  rdf            unit-ball volumes vs scipy.special.gamma, hand-computed 2-point shells in dims
                 1-4, the uniform-hypercube covariogram law (Monte Carlo) in dims 1-4
  pairmatrix_hd  torch.cdist float64 on the decoded bf16 features, symmetry, diagonal
  knn            lexsort brute force, lattice neighbour shells (6/12/8), index tie-break, k > n-1
Parity status: no worked example in PAPER.md prints values, so every pin is a
mathematical one; see DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tbs_oracle.c")
_LIB = os.path.join(_HERE, "libtbs_oracle.so")
_lib = None

_u64p = ctypes.POINTER(ctypes.c_uint64)
_f32p = ctypes.POINTER(ctypes.c_float)
_f64p = ctypes.POINTER(ctypes.c_double)
_i64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2 -ffp-contract=off -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
                               "-std=c11", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_sdh.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_double, ctypes.c_int, _i64, _i64,
                                   _u64p, _u64p]
        lib.oracle_sdh_bands.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_double, ctypes.c_int, _i64, _i64,
                                         _u64p, _u64p, _u64p]
        lib.oracle_sdh_lattice.argtypes = [_f32p, _i64, ctypes.c_int, _i64, ctypes.c_int, ctypes.c_int,
                                           _i64, _i64, _u64p]
        lib.oracle_pcf.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_double, _i64, _i64, _u64p, _u64p]
        lib.oracle_pairmatrix.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_int, ctypes.c_double, _i64, _i64,
                                          _f64p]
        lib.oracle_lattice_closed.argtypes = [_i64, _i64, ctypes.c_int, ctypes.c_int, _u64p, _i64, _u64p]
        lib.oracle_kde.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_double, _i64, _i64, _f64p]
        lib.oracle_rdf.argtypes = [_u64p, ctypes.c_int, ctypes.c_int, ctypes.c_double, ctypes.c_double,
                                   ctypes.c_double, _f64p]
        lib.oracle_pairmatrix_hd.argtypes = [ctypes.POINTER(ctypes.c_uint16), _i64, ctypes.c_int, ctypes.c_int,
                                             ctypes.c_double, _i64, _i64, _f64p]
        lib.oracle_knn.argtypes = [_f32p, _i64, ctypes.c_int, ctypes.c_int, _i64, _i64,
                                   ctypes.POINTER(ctypes.c_int64), _f64p]
        lib.oracle_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _pts(points):
    p = np.ascontiguousarray(points, dtype=np.float32)
    if p.ndim == 1:
        p = p.reshape(-1, 1)
    return p, p.shape[0], p.shape[1]


def _ptr(a, t):
    return a.ctypes.data_as(t)


def _rows(rows, n):
    return (0, n) if rows is None else (int(rows[0]), int(rows[1]))


def num_threads() -> int:
    return _load().oracle_num_threads()


def sdh(points, bucket_width, nbuckets, rows=None, with_amb=True):
    """Float-mode SDH. ``bucket_width`` is rounded to fp32 first (the API's type).

    Returns (hist uint64[nb], amb uint64[nb+1]) — amb[e] counts pairs within 1e-6
    relative of edge e (e = 1..nb-1).
    """
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    hist = np.zeros(nbuckets, np.uint64)
    amb = np.zeros(nbuckets + 1, np.uint64)
    w = float(np.float32(bucket_width))
    rc = _load().oracle_sdh(_ptr(p, _f32p), n, dim, w, int(nbuckets), rb, re, _ptr(hist, _u64p),
                            _ptr(amb, _u64p) if with_amb else None)
    if rc:
        raise ValueError(f"oracle_sdh: status {rc}")
    return hist, amb


def sdh_lattice(points, m, j, nbuckets, rows=None):
    """Exact-lattice SDH, bucket width w = m * 2^-j (integer-valued coordinates)."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    hist = np.zeros(nbuckets, np.uint64)
    rc = _load().oracle_sdh_lattice(_ptr(p, _f32p), n, dim, int(m), int(j), int(nbuckets), rb, re,
                                    _ptr(hist, _u64p))
    if rc:
        raise ValueError(f"oracle_sdh_lattice: status {rc}")
    return hist


def pcf(points, radius, rows=None):
    """2PCF count #{i<j : d < r} and its ambiguity count (|d - r| <= 1e-6 r)."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    c = np.zeros(1, np.uint64)
    a = np.zeros(1, np.uint64)
    rc = _load().oracle_pcf(_ptr(p, _f32p), n, dim, float(np.float32(radius)), rb, re, _ptr(c, _u64p),
                            _ptr(a, _u64p))
    if rc:
        raise ValueError(f"oracle_pcf: status {rc}")
    return int(c[0]), int(a[0])


def pairmatrix(points, gamma, rows=None, ktype=0):
    """Pair matrix rows [rb, re) x n in float64; ktype 0 Gaussian, 1 squared distance, 2 distance."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    out = np.zeros((re - rb, n), np.float64)
    rc = _load().oracle_pairmatrix(_ptr(p, _f32p), n, dim, int(ktype), float(np.float32(gamma)), rb, re,
                                   _ptr(out, _f64p))
    if rc:
        raise ValueError(f"oracle_pairmatrix: status {rc}")
    return out


def lattice_closed(L, m, j, nbuckets, r2=-1):
    """Closed-form lattice SDH of {0..L-1}^3 (and 2PCF count s < r2 if r2 >= 0)."""
    hist = np.zeros(nbuckets, np.uint64)
    c = np.zeros(1, np.uint64)
    rc = _load().oracle_lattice_closed(int(L), int(m), int(j), int(nbuckets), _ptr(hist, _u64p), int(r2),
                                       _ptr(c, _u64p))
    if rc:
        raise ValueError(f"oracle_lattice_closed: status {rc}")
    return hist, int(c[0])


def kde(points, gamma, rows=None):
    """Gaussian kernel pair sum S = sum_{i<j} exp(-gamma d_ij^2) in float64."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    out = np.zeros(1, np.float64)
    rc = _load().oracle_kde(_ptr(p, _f32p), n, dim, float(np.float32(gamma)), rb, re, _ptr(out, _f64p))
    if rc:
        raise ValueError(f"oracle_kde: status {rc}")
    return float(out[0])


def sdh_bands(points, bucket_width, nbuckets, rows=None):
    """Float-mode SDH with both ambiguity bands: (hist, amb (1e-6), amb_diag (5e-7)), each
    amb array uint64[nb+1] indexed by edge e = 1..nb-1 (SURVEY §8(c) diagnostic band)."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    hist = np.zeros(nbuckets, np.uint64)
    amb = np.zeros(nbuckets + 1, np.uint64)
    amb2 = np.zeros(nbuckets + 1, np.uint64)
    w = float(np.float32(bucket_width))
    rc = _load().oracle_sdh_bands(_ptr(p, _f32p), n, dim, w, int(nbuckets), rb, re, _ptr(hist, _u64p),
                                  _ptr(amb, _u64p), _ptr(amb2, _u64p))
    if rc:
        raise ValueError(f"oracle_sdh_bands: status {rc}")
    return hist, amb, amb2


def pairs_of_rows(n, rows=None):
    """Pairs an anchor-row range [b, e) counts: sum_{i=b}^{e-1} (n - 1 - i)."""
    b, e = _rows(rows, n)
    return (e - b) * (2 * n - b - e - 1) // 2


def rdf(hist, bucket_width, volume, dim=3, *, pairs):
    """RDF g[k] = hist[k] / (pairs shell_k / volume) for the len(hist) real shells (R6)."""
    h = np.ascontiguousarray(hist, dtype=np.uint64)
    g = np.zeros(len(h), np.float64)
    rc = _load().oracle_rdf(_ptr(h, _u64p), len(h), int(dim), float(np.float32(bucket_width)), float(pairs),
                            float(volume), _ptr(g, _f64p))
    if rc:
        raise ValueError(f"oracle_rdf: status {rc}")
    return g


def rdf_points(points, bucket_width, nbuckets, volume, rows=None, lattice=None):
    """The RDF pipeline of reading R6 on the oracle: SDH with nbuckets + 1 buckets (bucket nb
    takes every d >= nb w), its first nb counts normalised by the pairs the rows count.
    lattice=(m, j): exact-lattice SDH instead of float mode. Returns (g, hist[nb+1], amb)."""
    p, n, dim = _pts(points)
    if lattice is None:
        h, amb = sdh(p, bucket_width, nbuckets + 1, rows=rows)
    else:
        h, amb = sdh_lattice(p, lattice[0], lattice[1], nbuckets + 1, rows=rows), None
    return rdf(h[:nbuckets], bucket_width, volume, dim, pairs=pairs_of_rows(n, rows)), h, amb


def pairmatrix_hd(features_bf16_bits, gamma, rows=None, ktype=0):
    """High-dimensional pair matrix from bf16 features given as uint16 bit patterns [n][d]."""
    x = np.ascontiguousarray(features_bf16_bits, dtype=np.uint16)
    n, d = x.shape
    rb, re = _rows(rows, n)
    out = np.zeros((re - rb, n), np.float64)
    rc = _load().oracle_pairmatrix_hd(x.ctypes.data_as(ctypes.POINTER(ctypes.c_uint16)), n, d, int(ktype),
                                      float(np.float32(gamma)), rb, re, _ptr(out, _f64p))
    if rc:
        raise ValueError(f"oracle_pairmatrix_hd: status {rc}")
    return out


def knn(points, k, rows=None):
    """All-point kNN: (idx int64 [rows, k], dist float64 [rows, k]) in (distance, index) order."""
    p, n, dim = _pts(points)
    rb, re = _rows(rows, n)
    idx = np.zeros((re - rb, k), np.int64)
    dist = np.zeros((re - rb, k), np.float64)
    rc = _load().oracle_knn(_ptr(p, _f32p), n, dim, int(k), rb, re, idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                            _ptr(dist, _f64p))
    if rc:
        raise ValueError(f"oracle_knn: status {rc}")
    return idx, dist
