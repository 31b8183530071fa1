"""Shared test helpers: tolerances derived from the fp32 arithmetic (DESIGN.md
"Tolerances") and small utilities.  No method arithmetic lives here."""
from __future__ import annotations

import numpy as np

from synth import ACKLEY, EASOM, GRIEWANK, RASTRIGIN, ROSENBROCK, SPHERE

EPS = 2.0 ** -24  # fp32 unit roundoff

# north_star: single step from identical state within relative 1e-5
RTOL = {SPHERE: 1e-5, RASTRIGIN: 1e-5, ROSENBROCK: 1e-5, GRIEWANK: 1e-5, ACKLEY: 1e-5,
        EASOM: 2e-4}


def fit_atol(obj: int, X: np.ndarray) -> np.ndarray:
    """Per-row absolute tolerance for the GPU's fp32 fitness vs the oracle's
    fp64 fitness rounded to fp32 (derivations in DESIGN.md)."""
    X = np.atleast_2d(np.asarray(X, dtype=np.float64))
    m, d = X.shape
    if obj == GRIEWANK:
        # product of d cosines: each factor's argument y = x*rsqrt(k) carries <= 3 eps
        # relative error and t = y/(2 pi) 2 more; cos = 1 - 2 sin^2(pi t) is within
        # ~10 eps absolute of cos(t 2 pi) -> |dP| <= eps * sum(5 |y| + 10) + d eps
        k = np.arange(1, d + 1, dtype=np.float64)
        return 2.0 ** -21 * (np.abs(X) / np.sqrt(k)).sum(axis=1) + 2.0 ** -20 * d
    if obj == ACKLEY:
        # C/d carries <= (32 + log2 d + 4) eps absolute; times e
        return np.full(m, np.e * (36.0 + np.log2(max(d, 2))) * EPS * 2)
    if obj == EASOM:
        return np.full(m, 1e-30)
    return np.zeros(m)  # sums of nonnegative terms: relative bound only


def fit_tol(obj: int, X: np.ndarray, f_ref: np.ndarray) -> np.ndarray:
    return RTOL[obj] * np.abs(np.asarray(f_ref, dtype=np.float64)) + fit_atol(obj, X)


def bits(a: np.ndarray) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


def assert_bitwise(a, b, what=""):
    a, b = np.asarray(a, np.float32), np.asarray(b, np.float32)
    assert a.shape == b.shape, (what, a.shape, b.shape)
    ne = bits(a) != bits(b)
    if ne.any():
        idx = np.argwhere(ne)[:5]
        raise AssertionError(f"{what}: {int(ne.sum())} of {ne.size} differ, e.g. "
                             + ", ".join(f"{tuple(i)}: {a[tuple(i)]!r} vs {b[tuple(i)]!r}" for i in idx))


def assert_fitness_close(obj, X, got, ref, what="fitness"):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    tol = fit_tol(obj, X, ref)
    bad = np.abs(got - ref) > tol
    if bad.any():
        i = int(np.argmax(bad))
        raise AssertionError(f"{what}: {int(bad.sum())} rows outside tolerance, e.g. row {i}: "
                             f"{got[i]!r} vs {ref[i]!r} (tol {tol[i]:.3g})")
