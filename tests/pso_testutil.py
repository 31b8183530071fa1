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
    with np.errstate(invalid="ignore"):  # inf - inf where both are +inf pbests
        bad = ~(got == ref) & ~(np.abs(got - ref) <= tol)
    if bad.any():
        i = int(np.argmax(bad))
        raise AssertionError(f"{what}: {int(bad.sum())} rows outside tolerance, e.g. row {i}: "
                             f"{got[i]!r} vs {ref[i]!r} (tol {tol[i]:.3g})")


# ------------------------------------------------------------------ oracle lockstep
def gather_rows(parts):
    """Concatenate per-rank row shards (rank order) of each state array."""
    return [np.concatenate(p, axis=0) for p in zip(*parts)]


def oracle_lockstep(make_oracle, obj, snaps, ops, what=""):
    """Check a sequence of GPU states against the oracle, one call at a time.

    ``snaps[0]`` is the GPU state after create / init, ``snaps[k]`` after
    ``ops[k-1]``; a snapshot is a dict with X, V, PB, pf (whole swarm, dense),
    t, f, i (gbest) and G.  ``ops`` items are ("step", k) or ("set_state",
    (X, V, PB, pf, t)).  ``make_oracle(create)`` returns a fresh OracleSwarm
    (for a multi-rank run: ``nshards`` = world, so the oracle merges virtual
    shards exactly as SURVEY 8(e) prescribes).

    Each call is replayed by the oracle from the GPU's state before it (the
    oracle's re-selection of the gbest from that state must give the GPU's
    incumbent), one iteration at a time.  A pbest decision whose margin is
    inside the fitness tolerance is *ambiguous* (reading 23): such rows are
    excluded; when the gbest decision of an iteration before the call's last
    one is ambiguous the state can legitimately diverge and the call is only
    checked for G == PB[gi]; an ambiguous decision in the last iteration skips
    only the gbest comparison.  Returns (calls whose state was skipped, calls
    whose gbest was skipped)."""
    def compare(c, s, amb_rows, label):
        ok = ~amb_rows
        assert s["t"] == c.t, (label, s["t"], c.t)
        assert_bitwise(s["X"][ok], c.X[ok], f"{label}: X")
        assert_bitwise(s["V"][ok], c.V[ok], f"{label}: V")
        assert_bitwise(s["PB"][ok], c.PB[ok], f"{label}: PB")
        assert_fitness_close(obj, c.PB[ok], s["pf"][ok], c.pf[ok], f"{label}: pf")

    def gbest_ok(c, s, label):
        assert s["i"] == c.gi, (label, s["i"], c.gi)
        tol = fit_tol(obj, c.G[None, :], np.array([c.gf]))[0]
        assert abs(float(s["f"]) - float(c.gf)) <= tol or s["f"] == c.gf, (label, s["f"], c.gf)
        assert_bitwise(s["G"], c.G, f"{label}: G")

    n = snaps[0]["X"].shape[0]
    c = make_oracle(True)
    tol = fit_tol(obj, c.X, c.pf)
    amb_init = np.abs(c.pf.astype(np.float64) - c.gf) <= tol + fit_tol(obj, c.G[None, :], [c.gf])[0]
    compare(c, snaps[0], np.zeros(n, bool), f"{what} init")
    if amb_init.sum() <= 1:
        gbest_ok(c, snaps[0], f"{what} init")
    skipped_state = skipped_gbest = 0
    for k, (op, arg) in enumerate(ops):
        prev, cur = snaps[k], snaps[k + 1]
        label = f"{what} op {k} {op} {arg if op == 'step' else ''}"
        c = make_oracle(False)
        if op == "set_state":
            X, V, PB, pf, t = arg
            c.set_state(X, V, PB, pf, t=t)
            compare(c, cur, np.zeros(n, bool), label)
            gbest_ok(c, cur, label)
            continue
        c.set_state(prev["X"], prev["V"], prev["PB"], prev["pf"], t=prev["t"])
        assert c.gi == prev["i"], (label, "GPU incumbent != re-selection", c.gi, prev["i"])
        amb_rows = np.zeros(n, bool)
        amb_g_early = amb_g_last = False
        for it in range(arg):
            pf0, gf0 = c.pf.copy(), c.gf
            c.step(1)
            tol = fit_tol(obj, c.X, c.f)
            amb_rows |= np.abs(c.f.astype(np.float64) - pf0.astype(np.float64)) <= tol
            # the gbest decision: any candidate near the incumbent or near the winner
            near = (np.abs(c.f.astype(np.float64) - gf0) <= tol) | \
                   (np.abs(c.f.astype(np.float64) - c.gf) <= tol)
            amb = int(near.sum()) > (1 if c.gf != gf0 else 0)
            if it + 1 < arg:
                amb_g_early |= amb
            else:
                amb_g_last = amb
        assert_bitwise(cur["G"], cur["PB"][cur["i"]], f"{label}: G == PB[gi]")
        if amb_g_early:
            skipped_state += 1
            continue
        compare(c, cur, amb_rows, label)
        if amb_g_last:
            skipped_gbest += 1
            continue
        gbest_ok(c, cur, label)
    return skipped_state, skipped_gbest


# ------------------------------------------------------------------ crafted decision states
def crafted_state(case: str, n: int, d: int):
    """States for the decision pins of readings 9-11, to run on a FROZEN swarm
    (w = c1 = c2 = 0: x' = x), so every fitness is exact in fp32 on both sides.
    Returns (objective, lo, hi, X, V, PB, pf, a, b) where a < b are the rows
    the case is about (far apart: different CTAs, and different ranks of any
    particle split with world <= n / 3).

    ties  Sphere: rows a and b reach f = 1 on the next step (the lower index
          wins, later equal values never replace it); every other row sits at
          f = 4d > 9 = its pbest; row 0's pbest is NaN (read as +inf).
    zero  Easom, even d, x = -50: every f = -0.  pbest +0 at row a, -0 at
          row b, +inf elsewhere: -0 ties +0 (the incumbent a stays).
    minf  Sphere: a -inf pbest at row b wins and nothing beats it; row 0
          reaches f = +0.
    """
    a, b = 1, n - 2
    if case == "ties":
        X = np.full((n, d), 2.0, np.float32)
        X[a] = 0.0
        X[a, 0] = 1.0
        X[b] = 0.0
        X[b, d - 1] = -1.0
        pf = np.full(n, 9.0, np.float32)
        pf[0] = np.nan
        obj, lo, hi = SPHERE, -5.12, 5.12
    elif case == "zero":
        assert d % 2 == 0
        X = np.full((n, d), -50.0, np.float32)
        pf = np.full(n, np.inf, np.float32)
        pf[a] = 0.0
        pf[b] = -0.0
        obj, lo, hi = EASOM, -100.0, 100.0
    elif case == "minf":
        X = np.full((n, d), 1.0, np.float32)
        X[0] = 0.0
        pf = np.full(n, 5.0 * d, np.float32)
        pf[b] = -np.inf
        obj, lo, hi = SPHERE, -5.12, 5.12
    else:
        raise ValueError(case)
    return obj, lo, hi, X, np.zeros_like(X), X.copy(), pf, a, b


def crafted_expect(case: str, n: int, d: int, after_steps: int):
    """The gbest index (and value) the case must produce."""
    a, b = 1, n - 2
    if case == "ties":
        return (1, 9.0) if after_steps == 0 else (a, 1.0)
    if case == "zero":
        return a, 0.0
    return b, -np.inf
