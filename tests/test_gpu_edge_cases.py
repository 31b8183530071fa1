"""GPU twins of the oracle's decision pins (readings 9-11 of DESIGN.md 3):
strict < and the lowest global index among equal minima (Alg. 1 lines 7-12,
P:L91-93), NaN pbest read as +inf, -0 == +0 in the packed gbest key, and -inf
as a legal winner -- on every kernel path that takes these decisions: the
register and TMA streaming kernels, the CTA-resident and grid-resident
latency kernels, the thread-block cluster and the column split.

The states are crafted and injected with set_state; the swarm is frozen
(w = c1 = c2 = 0, so x' = x) and each case is run by the oracle on the same
state.  Fitness values here are exact in fp32 on both sides (sums of 0, 1
and 4, or an underflowed Easom), so every pf, decision and gbest must be
identical, not merely within tolerance.
"""
import numpy as np
import pytest

import oracle as orc
import paper_conf_icpp_liuwc21_b200 as fp
from pso_testutil import assert_bitwise, crafted_expect, crafted_state

pytestmark = pytest.mark.gpu

# path -> (n, d, environment, constructor keywords, expected pso_info check)
PATHS = {
    "reg": (700, 14, {"PSO_RESIDENT": "0"}, {}, lambda i: i["tma_pipeline"] == 0 and not i["resident"]),
    "tma": (700, 1000, {"PSO_RESIDENT": "0"}, {}, lambda i: i["tma_pipeline"] == 1 and not i["resident"]),
    "tma-eager": (700, 1000, {"PSO_RESIDENT": "0", "PSO_LAZY_PB": "0"}, {},
                  lambda i: i["tma_pipeline"] == 1 and not i["lazy_pb"]),
    "cta-resident": (32, 10, {}, {}, lambda i: i["resident"] == 1),
    "grid-resident": (600, 1000, {}, {}, lambda i: i["resident"] == 2),
    "cluster": (300, 1000, {"PSO_CLUSTER": "2"}, {}, lambda i: i["cluster"] == 2),
    "column-split": (300, 1000, {}, {"column_split": True}, lambda i: i["column_split"] == 1),
}


def _pair(path, obj, lo, hi, monkeypatch, seed=5):
    n, d, env, kw, check = PATHS[path]
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    g = fp.Swarm(n, d, 0.0, 0.0, 0.0, lo, hi, obj, seed, device=0, **kw)
    assert check(g.info()), g.info()
    c = orc.OracleSwarm(n, d, 0.0, 0.0, 0.0, lo, hi, obj, seed, create=False)
    return g, c, n, d


def _compare(g, c, what):
    X, V, PB, pf, t = g.get_state()
    gf, gi, G = g.gbest()
    assert t == c.t, what
    assert_bitwise(X, c.X, f"{what}: X")
    assert_bitwise(V, c.V, f"{what}: V")
    assert_bitwise(PB, c.PB, f"{what}: PB")
    assert_bitwise(pf, c.pf, f"{what}: pf")
    assert gi == c.gi, (what, gi, c.gi)
    assert gf == c.gf, (what, gf, c.gf)  # IEEE equality: the GPU key stores -0 as +0
    assert_bitwise(G, PB[gi], f"{what}: G == PB[gi]")
    assert_bitwise(G, c.G, f"{what}: G")
    return gi, gf, pf


CASES = ["ties", "zero", "minf"]


@pytest.mark.parametrize("case", CASES)
@pytest.mark.parametrize("path", sorted(PATHS))
def test_decisions_on_every_path(path, case, monkeypatch):
    """ties: rows a < b far apart (different CTAs; the serpentine order visits
    b first on odd iterations) reach the same fitness 1 on the same step -- the
    lower index wins, and on the next step the incumbent is kept (strict <); a
    NaN pbest is +inf after set_state and is improved on by any fitness.
    zero: Easom with even d far from pi gives f = -0 on every row: against the
    +0 pbest / gbest of row a it is a tie, even with a -0 pbest at row b, and
    only +inf pbests improve (to -0).  minf: an injected -inf pbest at a high
    index is the gbest and no fitness -- not even an exact +0 -- beats it.
    Both iteration parities (both row orders) are run."""
    n, d = PATHS[path][0], PATHS[path][1]
    obj, lo, hi, X, V, PB, pf, a, b = crafted_state(case, n, d)
    g, c, _, _ = _pair(path, obj, lo, hi, monkeypatch)
    for t0 in (0, 1):
        g.set_state(X, V, PB, pf, t=t0)
        c.set_state(X, V, PB, pf, t=t0)
        gi, gf, gpf = _compare(g, c, f"{path}/{case} set_state t={t0}")
        assert (gi, gf) == crafted_expect(case, n, d, 0)
        if case == "ties":
            assert gpf[0] == np.inf
        for k in (1, 2):
            g.step(1)
            c.step(1)
            gi, gf, gpf = _compare(g, c, f"{path}/{case} step {k} t={t0}")
            assert (gi, gf) == crafted_expect(case, n, d, k)
        if case == "ties":
            assert gpf[0] == np.float32(4 * d)
        if case == "zero":
            assert np.signbit(gpf[3]) and not np.signbit(gpf[a])
        if case == "minf":
            assert gpf[0] == 0.0
