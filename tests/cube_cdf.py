"""Distance distribution of two independent uniform points in the unit cube.

Test helper (a pin for the oracle, SURVEY §8(c) "closed form (cube line
picking)"). Per axis, |X_c - Y_c| has density g(u) = 2(1 - u) on [0, 1] and CDF
G(t) = 2t - t^2, so

    F(r) = P(|X - Y| < r) = int_0^1 g(x) int_0^1 g(y) G(sqrt(r^2 - x^2 - y^2)) dy dx

(G = 0 for a negative argument, 1 above 1). For r <= 1 this equals the textbook
closed form F(r) = (4 pi / 3) r^3 - (3 pi / 2) r^4 + (8/5) r^5 - r^6 / 6, which the
tests use to pin the quadrature; the mean distance is Robbins' constant.
"""
from __future__ import annotations

import math

from scipy import integrate

ROBBINS = 0.66170718226717623515583113324841358174640013579095


def F_closed_le1(r: float) -> float:
    return 4 * math.pi / 3 * r ** 3 - 1.5 * math.pi * r ** 4 + 1.6 * r ** 5 - r ** 6 / 6


def _G(t2: float) -> float:
    if t2 <= 0.0:
        return 0.0
    if t2 >= 1.0:
        return 1.0
    t = math.sqrt(t2)
    return 2 * t - t * t


def _H(q: float) -> float:
    """int_0^1 2(1-y) G(sqrt(q - y^2)) dy."""
    if q <= 0.0:
        return 0.0
    pts = [p for p in (math.sqrt(q) if q < 1 else None, math.sqrt(q - 1) if 1 < q < 2 else None)
           if p is not None and 0 < p < 1]
    val, _ = integrate.quad(lambda y: 2 * (1 - y) * _G(q - y * y), 0.0, 1.0, points=pts or None,
                            epsabs=1e-13, epsrel=1e-12, limit=200)
    return val


def F(r: float) -> float:
    if r <= 0:
        return 0.0
    if r * r >= 3.0:
        return 1.0
    r2 = r * r
    pts = [p for p in (r, math.sqrt(max(r2 - 1, 0)), math.sqrt(max(r2 - 2, 0))) if 0 < p < 1]
    val, _ = integrate.quad(lambda x: 2 * (1 - x) * _H(r2 - x * x), 0.0, 1.0, points=pts or None,
                            epsabs=1e-12, epsrel=1e-11, limit=200)
    return val
