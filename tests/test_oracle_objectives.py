"""Pins for the oracle's objectives (Sec 3.2; definitions P:L287-305;
Rastrigin / Rosenbrock / Ackley from [20] Molga & Smutnicki).

Each pin is a closed form, a special case that reduces to a library routine
(numpy dot, scipy.optimize.rosen), or a known optimum — chosen so that a
dropped term, a wrong sign or an off-by-one dimension index fails.
"""
import math

import numpy as np
import pytest
from scipy.optimize import rosen

import oracle as orc

RNG = np.random.default_rng(12345)


def f32(a):
    return np.asarray(a, dtype=np.float32)


# ------------------------------------------------------------------ Sphere
def test_sphere_closed_forms():
    assert orc.objective(orc.SPHERE, [1, 2, 3]) == 14.0
    assert orc.objective(orc.SPHERE, np.zeros(17)) == 0.0
    x = f32(RNG.uniform(-5.12, 5.12, 1000))
    ref = float(np.dot(x.astype(np.float64), x.astype(np.float64)))
    assert orc.objective_f64(orc.SPHERE, x) == pytest.approx(ref, rel=1e-13)


# --------------------------------------------------------------- Rastrigin
def test_rastrigin_optimum_and_lattice():
    assert orc.objective_f64(orc.RASTRIGIN, np.zeros(50)) == pytest.approx(0.0, abs=1e-12)
    # at integer points cos(2 pi k) = 1, so f = sum x_k^2
    x = f32(RNG.integers(-5, 6, 64))
    assert orc.objective_f64(orc.RASTRIGIN, x) == pytest.approx(float(np.sum(x.astype(np.float64) ** 2)),
                                                                 abs=1e-9)
    # at half-integers cos = -1, so each term is x^2 + 20
    h = f32(RNG.integers(-5, 5, 40) + 0.5)
    ref = float(np.sum(h.astype(np.float64) ** 2)) + 20.0 * h.size
    assert orc.objective_f64(orc.RASTRIGIN, h) == pytest.approx(ref, rel=1e-13)


def test_rastrigin_nonnegative():
    X = f32(RNG.uniform(-5.12, 5.12, (64, 33)))
    assert (orc.objective_rows(orc.RASTRIGIN, X) >= 0).all()


# -------------------------------------------------------------- Rosenbrock
def test_rosenbrock_matches_scipy_rosen():
    for d in [2, 3, 10, 257]:
        x = f32(RNG.uniform(-2.048, 2.048, d))
        assert orc.objective_f64(orc.ROSENBROCK, x) == pytest.approx(rosen(x.astype(np.float64)), rel=1e-12)


def test_rosenbrock_closed_forms():
    assert orc.objective(orc.ROSENBROCK, np.ones(30)) == 0.0
    assert orc.objective(orc.ROSENBROCK, np.zeros(30)) == 29.0  # d - 1
    assert orc.objective(orc.ROSENBROCK, [-1.0, 1.0]) == 4.0
    assert orc.objective(orc.ROSENBROCK, [1.7]) == 0.0  # d = 1: empty sum
    # neighbour orientation: x_{k+1} - x_k^2, not x_k - x_{k+1}^2
    assert orc.objective(orc.ROSENBROCK, [2.0, 4.0]) == 1.0
    assert orc.objective(orc.ROSENBROCK, [4.0, 2.0]) == 100.0 * 14.0 ** 2 + 9.0


# ---------------------------------------------------------------- Griewank
def test_griewank_optimum():
    assert orc.objective(orc.GRIEWANK, np.zeros(200)) == 0.0


def test_griewank_product_term_index_base():
    # 1-based k (reading 18): x_k = 2 pi sqrt(k) makes every cosine 1, so
    # f = sum x^2 / 4000 exactly up to the fp32 rounding of x.
    d = 12
    k = np.arange(1, d + 1, dtype=np.float64)
    x = f32(2.0 * math.pi * np.sqrt(k))
    ref = float(np.sum(x.astype(np.float64) ** 2)) / 4000.0
    assert orc.objective_f64(orc.GRIEWANK, x) == pytest.approx(ref, abs=1e-5)
    # with a 0-based index the first factor would be cos(x_1 / 0) -> nonsense
    # x_1 = pi: factor cos(pi / sqrt 1) = -1 -> f = 1 + pi^2/4000 + 1
    assert orc.objective_f64(orc.GRIEWANK, [math.pi]) == pytest.approx(2.0 + math.pi ** 2 / 4000.0,
                                                                         rel=1e-7)
    # x_2 = pi sqrt(2)/2: factor cos(pi/2) = 0 -> product vanishes
    x2 = f32([0.0, math.pi * math.sqrt(2.0) / 2.0, 0.0])
    ref2 = 1.0 + float(np.sum(x2.astype(np.float64) ** 2)) / 4000.0
    assert orc.objective_f64(orc.GRIEWANK, x2) == pytest.approx(ref2, abs=1e-7)


# ------------------------------------------------------------------ Ackley
def test_ackley_optimum():
    assert abs(orc.objective(orc.ACKLEY, np.zeros(64))) <= 1e-6


def test_ackley_lattice_closed_forms():
    # integer point, all |x_k| = m: cos terms are 1 ->
    # f = -20 exp(-0.2 m) - e + 20 + e = 20 (1 - exp(-0.2 m))
    for m in [1, 3]:
        x = f32(np.where(RNG.random(40) < 0.5, -m, m))
        assert orc.objective_f64(orc.ACKLEY, x) == pytest.approx(20.0 * (1.0 - math.exp(-0.2 * m)), rel=1e-12)
    # half-integers +-0.5: cos = -1 -> f = -20 exp(-0.1) - exp(-1) + 20 + e
    h = f32(np.where(RNG.random(40) < 0.5, -0.5, 0.5))
    ref = -20.0 * math.exp(-0.1) - math.exp(-1.0) + 20.0 + math.e
    assert orc.objective_f64(orc.ACKLEY, h) == pytest.approx(ref, rel=1e-12)


# ------------------------------------------------------------------- Easom
def test_easom_optimum_sign():
    # -(-1)^d prod cos^2(x_k) exp(-sum (x_k - pi)^2): at x = pi, f = -(-1)^d (reading 17)
    assert orc.objective_f64(orc.EASOM, f32(np.full(4, math.pi))) == pytest.approx(-1.0, abs=1e-6)
    assert orc.objective_f64(orc.EASOM, f32(np.full(3, math.pi))) == pytest.approx(1.0, abs=1e-6)
    assert orc.objective_f64(orc.EASOM, f32([math.pi, math.pi / 2])) == pytest.approx(0.0, abs=1e-6)


def test_rows_helper_equals_scalar():
    X = f32(RNG.uniform(-600, 600, (5, 19)))
    got = orc.objective_rows(orc.GRIEWANK, X)
    assert [float(v) for v in got] == [orc.objective(orc.GRIEWANK, r) for r in X]
