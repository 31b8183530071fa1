"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Acceptance (north_star):
  * Philox words and init state: bit-exact
  * single step from identical injected state: X, V bit-exact (<= 1e-5 rel
    required); fitness within the derived tolerance; PB / pbest decisions
    equal except ambiguous rows (|f - pf| within tolerance); gbest index exact
    unless ambiguous
  * C1 after 100 iterations: gbest fitness within relative 1e-4
Sizes span several CTA tiles, ragged d (d % 4 != 0), every CTA shape
(VPT 1/2/4/8) and the degenerate n = 1, d = 1.
"""
import os

import numpy as np
import pytest

import oracle as orc
import paper_conf_icpp_liuwc21_b200 as fp
from synth import (ACKLEY, DOMAINS, EASOM, GRIEWANK, RASTRIGIN, ROSENBROCK, SPHERE, WORKLOADS,
                   random_state, sample_rows)
from pso_testutil import assert_bitwise, assert_fitness_close, fit_tol

pytestmark = pytest.mark.gpu

OBJS = [SPHERE, RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY, EASOM]
# (n, d): C1; ragged d over several tiles; VPT 1, 2, 4, 8 shapes; degenerate
SHAPES = [(32, 10), (257, 13), (300, 1000), (70, 2000), (9, 4096), (3, 8192), (1, 1), (5, 3),
          (40, 999)]


def gpu_swarm(n, d, obj, seed=2021, w=0.9, c1=2.0, c2=2.0, vmax=0.0, **kw):
    lo, hi = DOMAINS[obj]
    return fp.Swarm(n, d, w, c1, c2, lo, hi, obj, seed, vmax=vmax, device=0, **kw)


def cpu_swarm(n, d, obj, seed=2021, w=0.9, c1=2.0, c2=2.0, vmax=0.0, create=True):
    lo, hi = DOMAINS[obj]
    return orc.OracleSwarm(n, d, w, c1, c2, lo, hi, obj, seed, vmax=vmax, create=create)


def keep_cluster(monkeypatch, d):
    """Rows of d in (PSO_D_AUTO_COLSPLIT, 16384] take the column split on one
    GPU; tests that exercise the row kernels there (the cluster: lazy vs eager
    pbest, the exchanges against a single-GPU twin) switch the automatic
    column split off (PSO_COLSPLIT=0: the planner's own cluster)."""
    if fp.PSO_D_AUTO_COLSPLIT < d <= 16384:
        monkeypatch.setenv("PSO_COLSPLIT", "0")


# ------------------------------------------------------------------ Philox
@pytest.mark.parametrize("tag,t,i,j0,m", [(0, 1, 0, 0, 4096), (1, 7, 123456, 5, 1001),
                                          (2, 0, 2**32 - 1, 0, 64), (3, 0, 77, 8189, 3),
                                          (0, 2**32 - 1, 5, 1, 513)])
@pytest.mark.parametrize("seed", [0, 2021, 2**64 - 1])
def test_philox_words_bitexact(tag, t, i, j0, m, seed):
    ref = orc.words(seed, tag, t, i, j0, m)
    got = fp.debug_philox(seed, tag, t, i, j0, m, device=0)
    np.testing.assert_array_equal(got, ref)
    cur = fp.debug_philox(seed, tag, t, i, j0, m, use_curand=True, device=0)
    np.testing.assert_array_equal(cur, ref)  # NVIDIA's curand_Philox4x32_10, same counters


# ------------------------------------------------------------------ objectives
@pytest.mark.parametrize("obj", OBJS)
@pytest.mark.parametrize("d", [1, 2, 7, 64, 1000, 2000, 4096, 8192])
def test_objective_matches_oracle(obj, d):
    lo, hi = DOMAINS[obj]
    rng = np.random.default_rng(d * 10 + obj)
    X = rng.uniform(lo, hi, size=(17, d)).astype(np.float32)
    X[0] = 0.0
    X[1] = np.float32(1.0) if obj == ROSENBROCK else X[1]
    got = fp.debug_objective(obj, X, device=0)
    ref = orc.objective_rows(obj, X)
    assert_fitness_close(obj, X, got, ref)


def test_objective_closed_forms_on_gpu():
    assert fp.debug_objective(SPHERE, np.array([[1, 2, 3]], np.float32))[0] == 14.0
    assert fp.debug_objective(ROSENBROCK, np.ones((1, 33), np.float32))[0] == 0.0
    assert fp.debug_objective(ROSENBROCK, np.zeros((1, 33), np.float32))[0] == 32.0
    assert fp.debug_objective(RASTRIGIN, np.zeros((1, 100), np.float32))[0] == 0.0
    assert fp.debug_objective(GRIEWANK, np.zeros((1, 100), np.float32))[0] == 0.0
    assert abs(fp.debug_objective(ACKLEY, np.zeros((1, 100), np.float32))[0]) <= 1e-6
    x = np.arange(-5, 5, dtype=np.float32)[None, :]
    assert fp.debug_objective(RASTRIGIN, x)[0] == pytest.approx(float((x.astype(np.float64) ** 2).sum()),
                                                                 rel=1e-6)


# ------------------------------------------------------------------ init
@pytest.mark.parametrize("obj", OBJS)
@pytest.mark.parametrize("n,d", SHAPES)
def test_init_bitexact(obj, n, d):
    g = gpu_swarm(n, d, obj, seed=11 * n + d)
    c = cpu_swarm(n, d, obj, seed=11 * n + d)
    X, V, PB, pf, t = g.get_state()
    assert t == 0
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    assert_bitwise(PB, c.PB, "PB0")
    assert_fitness_close(obj, c.X, pf, c.pf, "pf0")
    gf, gi, G = g.gbest()
    assert_bitwise(G, PB[gi], "G == PB[gi]")
    assert pf[gi] == gf and gf == pf.min() and gi == int(np.argmin(pf))
    tol = fit_tol(obj, c.X, c.pf)
    ambiguous = np.abs(c.pf.astype(np.float64) - c.gf) <= tol + fit_tol(obj, c.X[[c.gi]], [c.gf])[0]
    if ambiguous.sum() <= 1:
        assert gi == c.gi
    else:
        assert ambiguous[gi]


# ------------------------------------------------------------------ single step
def _step_and_compare(obj, n, d, seed, pf_mode, t0=0, **kw):
    lo, hi = DOMAINS[obj]
    X, V, PB, pf = random_state(n, d, lo, hi, 1.0, seed, pf_mode="inf")
    if pf_mode == "mixed":
        # pf around the oracle's next f, +-50%: both pbest branches, clear margins
        probe = cpu_swarm(n, d, obj, seed=seed, create=False).set_state(X, V, PB, pf, t=t0)
        probe.step(1)
        rng = np.random.default_rng(seed + 1)
        pf = (probe.f * rng.choice([0.5, 1.5], size=n)).astype(np.float32)
        pf[probe.f < 0] = probe.f[probe.f < 0] * 0.5
    g = gpu_swarm(n, d, obj, seed=seed, **kw).set_state(X, V, PB, pf, t=t0)
    c = cpu_swarm(n, d, obj, seed=seed, create=False).set_state(X, V, PB, pf, t=t0)
    gf0, gi0, G0 = g.gbest()
    assert gi0 == c.gi and gf0 == c.gf
    assert_bitwise(G0, c.G, "G after set_state")
    g.step(1)
    c.step(1)
    gX, gV, gPB, gpf, gt = g.get_state()
    assert gt == t0 + 1 == c.t
    assert_bitwise(gX, c.X, "X")
    assert_bitwise(gV, c.V, "V")
    # pbest decisions: equal unless ambiguous
    tol = fit_tol(obj, c.X, c.f)
    amb = np.abs(c.f.astype(np.float64) - pf.astype(np.float64)) <= tol
    c_imp = c.f < pf
    g_imp = (gpf.view(np.uint32) != pf.view(np.uint32)) | (gPB != PB).any(axis=1)
    assert ((g_imp == c_imp) | amb).all(), np.argwhere((g_imp != c_imp) & ~amb)[:5]
    agree = (g_imp == c_imp) & ~amb
    assert_bitwise(gPB[agree], c.PB[agree], "PB")
    imp = agree & c_imp
    assert_fitness_close(obj, c.X[imp], gpf[imp], c.pf[imp], "pf (improved rows)")
    assert_bitwise(gpf[agree & ~c_imp], pf[agree & ~c_imp], "pf (kept rows)")
    gf, gi, G = g.gbest()
    assert_bitwise(G, gPB[gi], "G == PB[gi]")
    if not amb.any():
        assert gi == c.gi
    return g, c


@pytest.mark.parametrize("obj", OBJS)
@pytest.mark.parametrize("n,d", SHAPES)
def test_single_step_all_improve(obj, n, d):
    _step_and_compare(obj, n, d, seed=1000 + 7 * n + d, pf_mode="inf", t0=0)


@pytest.mark.parametrize("obj", [SPHERE, RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY])
@pytest.mark.parametrize("n,d", [(257, 13), (300, 1000), (70, 2000), (9, 4096)])
def test_single_step_mixed_pbest(obj, n, d):
    _step_and_compare(obj, n, d, seed=2000 + n + d, pf_mode="mixed", t0=41)


@pytest.mark.parametrize("kernel", ["reg", "tma"])
@pytest.mark.parametrize("obj", [RASTRIGIN, ROSENBROCK, GRIEWANK])
@pytest.mark.parametrize("n,d", [(300, 13), (301, 1000), (70, 2001), (9, 4096), (5, 8192)])
def test_single_step_both_kernels(kernel, obj, n, d, monkeypatch):
    """Both step-kernel variants (register streaming / TMA bulk-copy pipeline)
    on every CTA shape, with a shallow and the default pipeline depth."""
    monkeypatch.setenv("PSO_KERNEL", kernel)
    g, _ = _step_and_compare(obj, n, d, seed=3000 + n + d, pf_mode="mixed", t0=3)
    info = g.info()
    assert info["tma_pipeline"] == (1 if kernel == "tma" else 0) or (kernel == "tma" and d >= 8192)
    monkeypatch.setenv("PSO_STAGES", "2")
    _step_and_compare(obj, n, d, seed=3100 + n + d, pf_mode="inf", t0=9)


# ------------------------------------------------------------------ multi-step
def test_lockstep_c1_100_iterations():
    """C1 (Sphere 32x10): at every one of 100 iterations the oracle, restarted
    from the GPU's state, must reproduce the GPU's next state."""
    w = WORKLOADS["C1"]
    g = gpu_swarm(w.n, w.d, w.objective, seed=w.seed)
    c = cpu_swarm(w.n, w.d, w.objective, seed=w.seed)
    for it in range(w.iters):
        X, V, PB, pf, t = g.get_state()
        gf, gi, G = g.gbest()
        c.set_state(X, V, PB, pf, t=t)
        assert c.gi == gi
        g.step(1)
        c.step(1)
        X2, V2, PB2, pf2, _ = g.get_state()
        assert_bitwise(X2, c.X, f"X it={it}")
        assert_bitwise(V2, c.V, f"V it={it}")
        assert_fitness_close(SPHERE, c.PB, pf2, c.pf, f"pf it={it}")


def test_end_to_end_c1_100_iterations():
    w = WORKLOADS["C1"]
    g = gpu_swarm(w.n, w.d, w.objective, seed=w.seed)
    c = cpu_swarm(w.n, w.d, w.objective, seed=w.seed)
    g.step(w.iters)
    c.step(w.iters)
    gf, gi, G = g.gbest()
    assert gf == pytest.approx(c.gf, rel=1e-4)
    X, V, PB, pf, t = g.get_state()
    assert t == w.iters
    assert gi == c.gi
    assert_bitwise(X, c.X, "X after 100 iterations")


@pytest.mark.parametrize("obj", [RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY])
def test_end_to_end_independent_runs(obj):
    n, d, T = 64, 37, 50
    g = gpu_swarm(n, d, obj, seed=5)
    c = cpu_swarm(n, d, obj, seed=5)
    g.step(T)
    c.step(T)
    gf, gi, G = g.gbest()
    assert gf == pytest.approx(c.gf, rel=1e-4, abs=1e-5)


# ------------------------------------------------------------------ invariants
@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 1024, 1000), (ROSENBROCK, 500, 1001),
                                     (GRIEWANK, 300, 2000), (ACKLEY, 100, 4096)])
def test_invariants_over_run(obj, n, d):
    lo, hi = DOMAINS[obj]
    g = gpu_swarm(n, d, obj, seed=n)
    prev_pf, prev_gf = g.get_state()[3], g.gbest(pos=False)[0]
    for _ in range(10):
        g.step(3)
        X, V, PB, pf, t = g.get_state()
        gf, gi, G = g.gbest()
        assert (X >= np.float32(lo)).all() and (X <= np.float32(hi)).all()
        assert (np.abs(V) <= g.vmax).all()
        assert (pf <= prev_pf).all() and gf <= prev_gf
        assert gf == pf.min() and pf[gi] == gf
        assert_bitwise(G, PB[gi], "G == PB[gi]")
        prev_pf, prev_gf = pf, gf


# ------------------------------------------------------------------ API semantics
def test_step_splitting_and_determinism():
    a = gpu_swarm(200, 300, RASTRIGIN, seed=9)
    b = gpu_swarm(200, 300, RASTRIGIN, seed=9)
    a.step(7)
    b.step(3).step(0).step(4)
    for x, y in zip(a.get_state()[:4], b.get_state()[:4]):
        assert_bitwise(x, y, "split")
    assert a.gbest()[:2] == b.gbest()[:2]
    c = gpu_swarm(200, 300, RASTRIGIN, seed=10)
    assert not np.array_equal(a.get_state()[0], c.step(7).get_state()[0])


def test_launch_counter_and_improvements(monkeypatch):
    monkeypatch.setenv("PSO_RESIDENT", "0")  # one streaming launch per iteration
    g = gpu_swarm(1000, 256, SPHERE, seed=3, timing=True)
    g.reset_counters()
    g.step(20)
    info = g.info()
    assert info["launches"] == 20
    assert info["step_kernel_count"] == 20 and info["step_kernel_ms"] > 0
    assert 0 < info["improvements"] <= 20 * 1000


@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 600, 1000), (ROSENBROCK, 300, 2001),
                                     (ACKLEY, 40, 4096), (SPHERE, 700, 256)])
def test_pdl_and_timing_do_not_change_results(obj, n, d, monkeypatch):
    """Programmatic dependent launch (default) vs plain stream order, with and
    without the timing events: the same bits (PDL only moves the launch, every
    global read of a step kernel sits behind griddepcontrol.wait)."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    runs = []
    for pdl, timing in (("1", False), ("1", True), ("0", True)):
        monkeypatch.setenv("PSO_PDL", pdl)
        g = gpu_swarm(n, d, obj, seed=77, timing=timing)
        g.step(9)
        runs.append((g.get_state()[:4], g.gbest()))
        info = g.info()
        if timing:  # per-call events under PDL, one pair per launch without
            assert info["step_kernel_count"] == 9 and info["step_kernel_ms"] > 0
        g.close()
    (s0, b0) = runs[0]
    for s1, b1 in runs[1:]:
        for x, y in zip(s0, s1):
            assert_bitwise(x, y, "PDL / timing changed the state")
        assert b0[:2] == b1[:2]
        assert_bitwise(b0[2], b1[2], "G")


@pytest.mark.parametrize("d,vpt,threads,ctas,stages", [
    (1000, 2, 128 + 64, 4, 4),    # C3 shape: 4 CTAs x 4 compute warps
    (2000, 2, 256 + 64, 2, 4),    # NS / C4: 2 CTAs x 8 warps
    (4096, 2, 512 + 64, 1, 4),    # C5: the wide instantiation, 16 warps
])
def test_tma_launch_shape_rule(d, vpt, threads, ctas, stages, monkeypatch):
    """The planner's shape rule: 16 compute warps per SM with
    >= 3 stages, 2 float4 per thread preferred; it depends on d only."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    for n in (ctas * 148 + 5, 3):  # the shape must not depend on n
        g = gpu_swarm(n, d, GRIEWANK, seed=5)
        info = g.info()
        assert info["tma_pipeline"] == 1
        assert (info["vec_per_thread"], info["threads_per_cta"], info["pipeline_stages"]) == \
            (vpt, threads, stages), info
        if n > 3:
            assert info["ctas_per_sm"] == ctas
        g.close()


def test_errors_do_not_abort():
    with pytest.raises(fp.PsoError) as e:
        gpu_swarm(0, 10, SPHERE)
    assert e.value.status == 1
    with pytest.raises(fp.PsoError) as e:
        gpu_swarm(10, fp.PSO_D_MAX + 1, SPHERE)  # beyond the column split's limit
    assert e.value.status == 5
    g = gpu_swarm(10, 10, SPHERE)
    with pytest.raises(fp.PsoError):
        g.step(-1)
    with pytest.raises(ValueError):
        g.set_state(np.zeros((9, 10)), np.zeros((10, 10)), np.zeros((10, 10)), np.zeros(10))
    fp.lib().pso_destroy(None)


def test_iteration_counter_limit():
    """The device iteration counter (Philox ctr[2], record tags) is 32-bit:
    pso_step refuses to cross 2^32 instead of repeating random streams."""
    g = gpu_swarm(40, 300, RASTRIGIN)
    X, V, PB, pf, _ = g.get_state()
    g.set_state(X, V, PB, pf, t=2**32 - 3)
    g.step(2)  # reaches 2^32 - 1
    with pytest.raises(fp.PsoError) as e:
        g.step(1)
    assert e.value.status == 5
    assert g.get_state()[4] == 2**32 - 1  # not poisoned, nothing ran


@pytest.mark.parametrize("first,second", [(2000, 1600), (16384, 12288)])
def test_handles_sharing_a_kernel_keep_their_shared_memory(first, second, monkeypatch):
    """The dynamic shared memory limit is one attribute per kernel function:
    planning a second handle of the same instantiation with a smaller ring must
    not lower the limit the first one launches with (both keep stepping, each
    equal to a fresh single handle)."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    if first > fp.PSO_D_AUTO_COLSPLIT:  # the cluster kernel (the column split's ring is d-free)
        monkeypatch.setenv("PSO_CLUSTER", "4")
    a = gpu_swarm(300, first, RASTRIGIN, seed=1)
    b = gpu_swarm(300, second, RASTRIGIN, seed=2)
    ia, ib = a.info(), b.info()
    assert ia["smem_bytes"] > ib["smem_bytes"] and ia["vec_per_thread"] == ib["vec_per_thread"]
    a.step(3)
    b.step(3)
    a2 = gpu_swarm(300, first, RASTRIGIN, seed=1).step(3)
    for x, y in zip(a.get_state()[:4], a2.get_state()[:4]):
        assert_bitwise(x, y, "first handle after a smaller plan")


# ------------------------------------------------------------------ full size, sampled
@pytest.mark.parametrize("key", ["NS", "C4", "C3", "C2", "W16K", "W16K@cluster", "W64K", "C5",
                                 "C5_2900K"])
def test_full_size_sampled_rows(key, monkeypatch):
    """Bench configurations at full size in the bench's launch shape (NS / C4
    streaming 100k x 2000, C3 streaming with a neighbour functor, C2 on the
    grid-resident path, W16K and W64K on the automatic column split, W16K on
    4-CTA clusters too, C5 1M x 4096 on the wide 16-warp instantiation, and the
    capacity sweep's 2.9M x 4096 -- 142.5 GB of state): sampled rows read back with
    pso_get_rows are recomputed by the oracle exactly (rows are independent
    given G): init bit-exact, one iteration's X / V bit-exact, decisions as the
    oracle's; the gbest is min pf with the lowest index and G = PB[gi]."""
    if key.endswith("@cluster"):
        key = key.split("@")[0]
        monkeypatch.setenv("PSO_CLUSTER", "4")
    w = WORKLOADS[key]
    g = gpu_swarm(w.n, w.d, w.objective, seed=w.seed)
    assert g.info()["column_split"] == int(w.d > fp.PSO_D_AUTO_COLSPLIT and "PSO_CLUSTER" not in os.environ)
    idx = sample_rows(w.n, 48, seed=7)
    X0, V0, _, _ = g.get_rows(idx[:8])
    for k, i in enumerate(idx[:8]):  # init rows are bit-exact
        c = orc.OracleSwarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed,
                            row_begin=int(i), nrows=1, create=False)
        c.init_local()
        assert_bitwise(X0[k], c.X[0], f"X0 row {i}")
        assert_bitwise(V0[k], c.V[0], f"V0 row {i}")
    g.step(2)
    X, V, PB, pf = g.get_rows(idx)
    t = g.info()["t"]
    _, _, G = g.gbest()
    g.step(1)
    X2, V2, PB2, pf2s = g.get_rows(idx)
    pf2 = np.empty(w.n, np.float32)
    g.get_state(out=(None, None, None, pf2))
    gf, gi, G2 = g.gbest()
    c = cpu_swarm(w.n, w.d, w.objective, seed=w.seed, create=False)
    cX, cV, cPB, cpf, cf = c.rows_step(t + 1, G, idx, X, V, PB, pf)
    assert_bitwise(X2, cX, "X rows")
    assert_bitwise(V2, cV, "V rows")
    assert_bitwise(pf2s, pf2[idx], "pf rows (get_rows vs get_state)")
    tol = fit_tol(w.objective, cX, cf)
    amb = np.abs(cf.astype(np.float64) - pf.astype(np.float64)) <= tol
    ok = ~amb
    assert_bitwise(PB2[ok], cPB[ok], "PB rows")
    assert_fitness_close(w.objective, cPB[ok], pf2s[ok], cpf[ok], "pf rows")
    assert gf == pf2.min() and gi == int(np.argmin(pf2))
    Xg, _, PBg, _ = g.get_rows([gi])
    assert_bitwise(G2, PBg[0], "G == PB[gi]")
    g.close()


def test_get_rows_reads_without_changing_the_state(monkeypatch):
    """pso_get_rows returns exactly the rows pso_get_state returns (a deferred
    pbest read from x), and reading does not change the following iterations."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    a = gpu_swarm(500, 2000, GRIEWANK, seed=3)
    b = gpu_swarm(500, 2000, GRIEWANK, seed=3)
    assert a.info()["lazy_pb"] == 1
    a.step(4)
    b.step(4)
    idx = np.array([499, 0, 17, 17, 250])
    Xr, Vr, PBr, pfr = a.get_rows(idx)
    a.step(3)
    b.step(3)
    X, V, PB, pf, _ = b.get_state()
    Xa, Va, PBa, pfa, _ = a.get_state()
    for x, y in zip((Xa, Va, PBa, pfa), (X, V, PB, pf)):
        assert_bitwise(x, y, "a run read with get_rows equals one that was not")
    c = gpu_swarm(500, 2000, GRIEWANK, seed=3).step(4)
    Xc, Vc, PBc, pfc, _ = c.get_state()
    for got, ref in zip((Xr, Vr, PBr, pfr), (Xc[idx], Vc[idx], PBc[idx], pfc[idx])):
        assert_bitwise(got, ref, "get_rows vs get_state")
    with pytest.raises(fp.PsoError):
        a.get_rows([500])


# ------------------------------------------------------------------ exchange path
@pytest.mark.parametrize("mode", ["allgather", "allreduce", "allgather-eager", "allreduce-eager"])
@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 300, 1000), (GRIEWANK, 50, 13),
                                     (ROSENBROCK, 6, 10000)])
def test_exchange_path_with_single_rank_comm(obj, n, d, mode, monkeypatch):
    """The NCCL exchanges forced on a 1-rank communicator must give the
    single-GPU results bitwise: the all-gather of the (key, row) records, and
    north_star's allreduce-min of the key + sum-broadcast of the owner's row
    (PSO_FLAG_ALLREDUCE); both replayed as captured CUDA graphs of 4
    iterations, or launched eagerly (PSO_GRAPH=0)."""
    import torch  # noqa: F401  (loads the NCCL the library resolves)
    monkeypatch.setenv("PSO_FORCE_EXCHANGE", "1")
    keep_cluster(monkeypatch, d)
    if mode.endswith("-eager"):
        monkeypatch.setenv("PSO_GRAPH", "0")
    comm = fp.nccl_comm_init(1, fp.nccl_unique_id(), 0, 0)
    try:
        g = gpu_swarm(n, d, obj, seed=5, nccl_comm=comm,
                      allreduce_exchange=mode.startswith("allreduce"))
        ref = gpu_swarm(n, d, obj, seed=5)
        assert g.gbest()[:2] == ref.gbest()[:2]
        g.reset_counters()
        g.step(20)
        ref.step(20)
        # one step kernel per iteration (the exchange merge runs in the next
        # step's prologue) + one select kernel at the end of the call; the
        # allreduce exchange adds its owner-row kernel per iteration
        assert g.info()["launches"] == (41 if mode.startswith("allreduce") else 21)
        g.step(1).step(2)
        ref.step(3)
        for x, y in zip(g.get_state()[:4], ref.get_state()[:4]):
            assert_bitwise(x, y, "exchange path state")
        gf, gi, G = g.gbest()
        rf, ri, RG = ref.gbest()
        assert (gf, gi) == (rf, ri)
        assert_bitwise(G, RG, "G")
        X, V, PB, pf, t = g.get_state()
        g.set_state(X, V, PB, pf, t=t)  # rebest through the exchange
        assert g.gbest()[:2] == (rf, ri)
        g.close()
    finally:
        fp.nccl_comm_destroy(comm)


# ------------------------------------------------------------------ resident path (NEXT-1)
@pytest.mark.parametrize("obj,n,d", [(SPHERE, 32, 10), (ROSENBROCK, 100, 16), (GRIEWANK, 7, 13),
                                     (ACKLEY, 64, 128), (RASTRIGIN, 1, 1), (RASTRIGIN, 200, 40)])
def test_resident_path_bitwise_equals_streaming(obj, n, d, monkeypatch):
    """The single-CTA shared-memory path for tiny swarms gives the streaming
    kernel's results bit for bit (same per-row reduction order), in one launch
    per pso_step call."""
    a = gpu_swarm(n, d, obj, seed=31)
    assert a.info()["resident"] == 1
    monkeypatch.setenv("PSO_RESIDENT", "0")
    b = gpu_swarm(n, d, obj, seed=31)
    assert b.info()["resident"] == 0
    a.reset_counters()
    for k in (1, 7, 42):
        a.step(k)
        b.step(k)
        for x, y in zip(a.get_state()[:4], b.get_state()[:4]):
            assert_bitwise(x, y, f"resident vs streaming after +{k}")
        fa, ia, Ga = a.gbest()
        fb, ib, Gb = b.gbest()
        assert (fa, ia) == (fb, ib)
        assert_bitwise(Ga, Gb, "G")
    info = a.info()
    assert info["launches"] == 3 and info["t"] == 50
    assert info["improvements"] > 0


@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 1024, 1000), (ROSENBROCK, 300, 1001),
                                     (GRIEWANK, 70, 2000), (ACKLEY, 9, 4096), (SPHERE, 600, 256)])
def test_grid_resident_bitwise_equals_streaming(obj, n, d, monkeypatch):
    """Swarms that fit in the grid's shared memory run whole pso_step calls in
    one cooperative launch; results are the streaming TMA kernel's bit for bit."""
    a = gpu_swarm(n, d, obj, seed=41)
    assert a.info()["resident"] == 2
    monkeypatch.setenv("PSO_RESIDENT", "0")
    b = gpu_swarm(n, d, obj, seed=41)
    assert b.info()["resident"] == 0 and b.info()["tma_pipeline"] == 1
    a.reset_counters()
    for k in (1, 5, 14):
        a.step(k)
        b.step(k)
        for x, y in zip(a.get_state()[:4], b.get_state()[:4]):
            assert_bitwise(x, y, f"grid-resident vs streaming after +{k}")
        fa, ia, Ga = a.gbest()
        fb, ib, Gb = b.gbest()
        assert (fa, ia) == (fb, ib)
        assert_bitwise(Ga, Gb, "G")
    info = a.info()
    assert info["launches"] == 3 and info["t"] == 20
    assert info["improvements"] > 0


# ------------------------------------------------------------------ per-dimension bounds (NEXT-2)
def _dim_bounds(d, seed):
    rng = np.random.default_rng(seed)
    xlo = rng.uniform(-5, -0.5, d).astype(np.float32)
    xhi = (xlo + rng.uniform(0.5, 6, d)).astype(np.float32)
    vhi = rng.uniform(0.05, 2, d).astype(np.float32)
    vlo = (-rng.uniform(0.05, 2, d)).astype(np.float32)
    return np.stack([vlo, vhi, xlo, xhi])


@pytest.mark.parametrize("path", ["auto", "reg", "tma", "streaming"])
@pytest.mark.parametrize("obj,n,d", [(SPHERE, 32, 10), (RASTRIGIN, 300, 1000), (ROSENBROCK, 70, 2001),
                                     (GRIEWANK, 257, 13), (ACKLEY, 9, 4096)])
def test_per_dim_bounds_match_oracle(path, obj, n, d, monkeypatch):
    if path in ("reg", "tma"):
        monkeypatch.setenv("PSO_KERNEL", path)
    elif path == "streaming":
        monkeypatch.setenv("PSO_RESIDENT", "0")
    b = _dim_bounds(d, n + d)
    lo, hi = DOMAINS[obj]
    g = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 13, device=0, bounds=b)
    assert g.info()["bounds"] == 1
    c = orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 13, bounds=b)
    X, V, PB, pf, _ = g.get_state()
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    for _ in range(3):
        X, V, PB, pf, t = g.get_state()
        c.set_state(X, V, PB, pf, t=t)
        g.step(1)
        c.step(1)
        X2, V2, _, pf2, _ = g.get_state()
        assert_bitwise(X2, c.X, "X")
        assert_bitwise(V2, c.V, "V")
        assert (X2 >= b[2]).all() and (X2 <= b[3]).all()
        assert (V2 >= b[0]).all() and (V2 <= b[1]).all()
    b2 = _dim_bounds(d, 99)
    g.set_bounds(b2)
    g.step(2)
    X3, V3, _, _, _ = g.get_state()
    assert (V3 >= b2[0]).all() and (V3 <= b2[1]).all()


def test_set_bounds_requires_bounds_handle():
    g = gpu_swarm(10, 10, SPHERE)
    with pytest.raises(fp.PsoError) as e:
        g.set_bounds(_dim_bounds(10, 1))
    assert e.value.status == 5
    with pytest.raises(fp.PsoError) as e:
        bad = _dim_bounds(10, 1)
        bad[0, 3] = 5.0  # vlo > vhi
        gpu_swarm(10, 10, SPHERE, bounds=bad)
    assert e.value.status == 1


# ------------------------------------------------------------------ persistent streaming kernel
@pytest.mark.parametrize("obj,n,d,kw", [(ROSENBROCK, 3000, 1000, {}), (GRIEWANK, 2000, 2000, {}),
                                        (RASTRIGIN, 1500, 2000, {}), (SPHERE, 60, 2001, {}),
                                        (EASOM, 700, 999, {"bounds": True}), (ACKLEY, 5000, 256, {})])
def test_persistent_kernel_bitwise_equals_streaming(obj, n, d, kw, monkeypatch):
    """k_step_persist (a whole pso_step call per cooperative launch; every CTA
    streams a fixed set of rows through the TMA ring for every iteration, the
    gbest settled by a grid barrier and a candidate-row pull) against the
    per-iteration streaming kernel: X, V, PB, pf, the gbest index and G bitwise
    after calls of 1, 2, 5 and 3 iterations, across a set_state, and with fewer
    rows than CTAs (n = 60: most CTAs own no row).  (The narrow TMA shapes only:
    rows of up to 512 float4.)"""
    lo, hi = DOMAINS[obj]
    bk = {}
    if kw.get("bounds"):
        bk["bounds"] = _dim_bounds(d, 7)
    monkeypatch.setenv("PSO_PERSIST", "1")
    g = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 99, device=0, **bk)
    monkeypatch.setenv("PSO_PERSIST", "0")
    monkeypatch.setenv("PSO_RESIDENT", "0")
    e = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 99, device=0, **bk)
    assert g.info()["resident"] == 3 and e.info()["resident"] == 0
    assert g.info()["lazy_pb"] == e.info()["lazy_pb"]
    for k in (1, 2, 5, 3):
        g.step(k)
        e.step(k)
        for x, y, nm in zip(g.get_state(), e.get_state(), "X V PB pf t".split()):
            if nm == "t":
                assert x == y
            else:
                assert_bitwise(x, y, f"persistent vs streaming {nm}")
        gf, gi, G = g.gbest()
        ef, ei, EG = e.gbest()
        assert (gf, gi) == (ef, ei)
        assert_bitwise(G, EG, "G")
    X, V, PB, pf, t = e.get_state()
    rng = np.random.default_rng(5)
    pf = (pf * rng.choice([0.5, 2.0], size=n)).astype(np.float32)  # both pbest branches
    g.set_state(X, V, PB, pf, t=t)
    e.set_state(X, V, PB, pf, t=t)
    g.step(4)
    e.step(4)
    for x, y, nm in zip(g.get_state()[:4], e.get_state()[:4], "X V PB pf".split()):
        assert_bitwise(x, y, f"after set_state {nm}")
    assert g.gbest()[:2] == e.gbest()[:2]
    # one step launch per call instead of one per iteration (15 iterations in 5 calls)
    assert g.info()["launches"] <= e.info()["launches"] - 10


def test_persistent_kernel_matches_the_oracle(monkeypatch):
    """C3's shape at a tenth of its rows through k_step_persist against the
    oracle run from the same seed: X bit-exact after 1 + 4 iterations, the
    gbest index and fitness."""
    monkeypatch.setenv("PSO_PERSIST", "1")
    n, d, obj = 1000, 1000, ROSENBROCK
    g = gpu_swarm(n, d, obj, seed=17)
    assert g.info()["resident"] == 3
    c = cpu_swarm(n, d, obj, seed=17)
    for k in (1, 4):
        g.step(k)
        c.step(k)
        X, V, PB, pf, t = g.get_state()
        assert_bitwise(X, c.X, "X vs oracle")
        assert_bitwise(V, c.V, "V vs oracle")
        assert_fitness_close(obj, c.PB, pf, c.pf, "pf")
        gf, gi, G = g.gbest()
        assert gi == c.gi
        assert_bitwise(G, PB[gi], "G == PB[gi]")


# ------------------------------------------------------------------ wide rows (NEXT-3)
WIDE = [(5, 8193), (3, 10000), (4, 16384), (2, 65536)]


@pytest.mark.parametrize("obj", [SPHERE, RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY])
@pytest.mark.parametrize("n,d", WIDE)
def test_wide_rows_cluster_path(obj, n, d, monkeypatch):
    """d > 8192: each row is split in column blocks over a thread-block cluster
    (DSMEM partials, CTA 0 decides); init bit-exact, one step bit-exact in X/V.
    Above PSO_D_AUTO_COLSPLIT a single GPU picks the column split, so the
    cluster is requested there (PSO_CLUSTER)."""
    if d > fp.PSO_D_AUTO_COLSPLIT:
        monkeypatch.setenv("PSO_CLUSTER", "4" if d <= 16384 else "16")
    g = gpu_swarm(n, d, obj, seed=d + obj)
    assert g.info()["cluster"] >= 2
    c = cpu_swarm(n, d, obj, seed=d + obj)
    X, V, PB, pf, _ = g.get_state()
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    assert_fitness_close(obj, c.X, pf, c.pf, "pf0")
    _step_and_compare(obj, n, d, seed=5000 + d, pf_mode="mixed", t0=2)
    _step_and_compare(obj, n, d, seed=5100 + d, pf_mode="inf", t0=0)


@pytest.mark.parametrize("d", [9217, 12000, 16385, 40000, 65536])
def test_single_gpu_wide_rows_pick_the_column_split(d):
    """One GPU, d > PSO_D_AUTO_COLSPLIT: the column split is chosen (it beats
    8- and 16-CTA clusters); results as the oracle's (init bit-exact, one step
    bit-exact in X / V)."""
    g = gpu_swarm(3, d, RASTRIGIN, seed=d)
    assert g.info()["column_split"] == 1 and g.info()["cluster"] == 0
    c = cpu_swarm(3, d, RASTRIGIN, seed=d)
    X, V, PB, pf, _ = g.get_state()
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    _step_and_compare(RASTRIGIN, 3, d, seed=5200 + d, pf_mode="mixed", t0=2)
    assert gpu_swarm(3, fp.PSO_D_AUTO_COLSPLIT, RASTRIGIN).info()["column_split"] == 0


@pytest.mark.parametrize("C", [2, 4, 8, 16])
@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 40, 1000), (ROSENBROCK, 33, 2001),
                                     (GRIEWANK, 20, 999), (ACKLEY, 17, 4096)])
def test_forced_cluster_split_matches_oracle(C, obj, n, d, monkeypatch):
    monkeypatch.setenv("PSO_CLUSTER", str(C))
    g, _ = _step_and_compare(obj, n, d, seed=6000 + C + d, pf_mode="mixed", t0=7)
    assert g.info()["cluster"] == C
    # several iterations: invariants and G == PB[gi]
    lo, hi = DOMAINS[obj]
    g.step(5)
    X, V, PB, pf, _ = g.get_state()
    gf, gi, G = g.gbest()
    assert (X >= np.float32(lo)).all() and (X <= np.float32(hi)).all()
    assert gf == pf.min() and gi == int(np.argmin(pf))
    assert_bitwise(G, PB[gi], "G == PB[gi]")


def test_wide_rows_with_bounds_and_lockstep(monkeypatch):
    n, d, obj = 6, 12000, ROSENBROCK
    b = _dim_bounds(d, 3)
    lo, hi = DOMAINS[obj]
    g = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 21, device=0, bounds=b)
    c = orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 21, bounds=b)
    for _ in range(4):
        X, V, PB, pf, t = g.get_state()
        c.set_state(X, V, PB, pf, t=t)
        g.step(1)
        c.step(1)
        X2, V2, _, pf2, _ = g.get_state()
        assert_bitwise(X2, c.X, "X")
        assert_bitwise(V2, c.V, "V")
        assert_fitness_close(obj, c.PB, pf2, c.pf, "pf")


@pytest.mark.parametrize("obj,n,d", [(RASTRIGIN, 300, 1000), (GRIEWANK, 50, 13),
                                     (ROSENBROCK, 6, 10000)])
def test_nvlink_peer_exchange_single_rank(obj, n, d, monkeypatch):
    """The NVLink peer exchange (records stored into every rank's receive buffer
    by the step kernel's last CTA, iteration tags acquired by the next step's
    prologue) on a 1-rank communicator: bitwise the single-GPU results, one
    kernel per iteration."""
    import torch  # noqa: F401
    monkeypatch.setenv("PSO_FORCE_EXCHANGE", "1")
    keep_cluster(monkeypatch, d)
    comm = fp.nccl_comm_init(1, fp.nccl_unique_id(), 0, 0)
    try:
        g = gpu_swarm(n, d, obj, seed=8, nccl_comm=comm)
        h, off = g.p2p_handle()
        assert len(h) == 64 and off > 0
        g.p2p_connect([h], [off]).p2p_enable(True)
        ref = gpu_swarm(n, d, obj, seed=8)
        g.reset_counters()
        g.step(15)
        ref.step(15)
        assert g.info()["launches"] == 16  # 15 step kernels + the final fold
        for x, y in zip(g.get_state()[:4], ref.get_state()[:4]):
            assert_bitwise(x, y, "p2p exchange state")
        assert g.gbest()[:2] == ref.gbest()[:2]
        X, V, PB, pf, t = g.get_state()
        g.set_state(X, V, PB, pf, t=t)
        ref.set_state(X, V, PB, pf, t=t)
        g.step(4)
        ref.step(4)
        gf, gi, G = g.gbest()
        rf, ri, RG = ref.gbest()
        assert (gf, gi) == (rf, ri)
        assert_bitwise(G, RG, "G")
        g.close()
    finally:
        fp.nccl_comm_destroy(comm)


def test_switch_to_nvlink_after_set_state(monkeypatch):
    """Records all-gathered over NCCL carry the same (epoch, iteration) tag as
    NVLink records: a handle that runs set_state (a new epoch) on the NCCL
    exchange and only then switches to NVLink finds its last records instead
    of waiting for a tag that never comes."""
    import torch  # noqa: F401
    monkeypatch.setenv("PSO_FORCE_EXCHANGE", "1")
    comm = fp.nccl_comm_init(1, fp.nccl_unique_id(), 0, 0)
    try:
        g = gpu_swarm(200, 1000, RASTRIGIN, seed=12, nccl_comm=comm)
        ref = gpu_swarm(200, 1000, RASTRIGIN, seed=12)
        g.step(3)
        ref.step(3)
        X, V, PB, pf, t = g.get_state()
        g.set_state(X, V, PB, pf, t=t)
        ref.set_state(X, V, PB, pf, t=t)
        g.step(2)
        ref.step(2)
        h, off = g.p2p_handle()
        g.p2p_connect([h], [off]).p2p_enable(True)
        g.step(3)
        ref.step(3)
        for x, y in zip(g.get_state()[:4], ref.get_state()[:4]):
            assert_bitwise(x, y, "state after the switch")
        assert g.gbest()[:2] == ref.gbest()[:2]
        g.close()
    finally:
        fp.nccl_comm_destroy(comm)


# ------------------------------------------------------------------ lazy pbest rows
@pytest.mark.parametrize("obj,n,d", [(GRIEWANK, 300, 2000), (RASTRIGIN, 301, 1000),
                                     (ROSENBROCK, 5, 12000)])
def test_lazy_pbest_rows_lockstep(obj, n, d, monkeypatch):
    """Streaming TMA / cluster kernels keep a row's pbest implicit while it equals
    x (no pb load, no pb store) and write it when the row stops improving.  Over
    several iterations with both transitions, PB (materialised by get_state),
    pf and X/V equal the oracle's and the eager kernel's bit for bit."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    keep_cluster(monkeypatch, d)
    g = gpu_swarm(n, d, obj, seed=77)
    assert g.info()["lazy_pb"] == 1
    monkeypatch.setenv("PSO_LAZY_PB", "0")
    e = gpu_swarm(n, d, obj, seed=77)
    assert e.info()["lazy_pb"] == 0
    c = cpu_swarm(n, d, obj, seed=77)
    for k in (1, 1, 3, 1, 6):
        g.step(k)
        e.step(k)
        c.step(k)
        gs, es = g.get_state(), e.get_state()
        for x, y, nm in zip(gs[:4], es[:4], "X V PB pf".split()):
            assert_bitwise(x, y, f"lazy vs eager {nm}")
        assert_bitwise(gs[0], c.X, "X vs oracle")
        assert_bitwise(gs[2], c.PB, "PB vs oracle")
        assert g.gbest()[:2] == e.gbest()[:2]
    info = g.info()
    assert info["pb_loads"] < e.info()["pb_loads"]  # flagged rows skipped their pb load


@pytest.mark.parametrize("w,c1,c2", [(0.0, 2.0, 0.0), (0.0, -1.5, 2.0), (0.5, 0.0, 2.0),
                                     (0.9, -2.0, 2.0), (0.0, 0.0, 0.0)])
@pytest.mark.parametrize("obj,n,d,kw", [(GRIEWANK, 300, 2000, {}), (SPHERE, 64, 1000, {}),
                                        (ROSENBROCK, 5, 12000, {}),
                                        (GRIEWANK, 9, 999, {"column_split": True})])
def test_lazy_rows_skip_r1_signed_zeros(w, c1, c2, obj, n, d, kw, monkeypatch):
    """A lazy row (PB == X) does not draw R1: (c1 r1)(pb - x) is copysign(0, c1)
    for any r1.  The velocity must still be rounded as Eq. 1 rounds it: with
    w = 0 a negative v gives a = -0, and -0 + (+0) = +0 must not become -0 when
    c = 0 (c2 = 0, or g == x).  Negative and zero c1 give b = -0 / +0.  Lazy and
    eager kernels and the oracle agree bit for bit (signs of zero included)."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    if not kw:
        keep_cluster(monkeypatch, d)
    g = gpu_swarm(n, d, obj, seed=5, w=w, c1=c1, c2=c2, **kw)
    c = cpu_swarm(n, d, obj, seed=5, w=w, c1=c1, c2=c2)
    if not kw:
        assert g.info()["lazy_pb"] == 1
        monkeypatch.setenv("PSO_LAZY_PB", "0")
        e = gpu_swarm(n, d, obj, seed=5, w=w, c1=c1, c2=c2)
        assert e.info()["lazy_pb"] == 0
    for k in (1, 1, 2, 1):
        g.step(k)
        c.step(k)
        gs = g.get_state()
        assert_bitwise(gs[0], c.X, "X vs oracle")
        assert_bitwise(gs[1], c.V, "V vs oracle")
        assert_bitwise(gs[2], c.PB, "PB vs oracle")
        if not kw:
            e.step(k)
            for x, y, nm in zip(gs[:4], e.get_state()[:4], "X V PB pf".split()):
                assert_bitwise(x, y, f"lazy vs eager {nm}")


@pytest.mark.parametrize("obj,n,d", [(ROSENBROCK, 301, 1000), (GRIEWANK, 300, 2000),
                                     (RASTRIGIN, 7, 12000), (SPHERE, 5000, 600),
                                     (GRIEWANK, 1200, 4096), (RASTRIGIN, 100, 2000)])
def test_row_order_is_invisible(obj, n, d, monkeypatch):
    """Serpentine row order (odd iterations walk the rows backwards for L2
    reuse), the L2 prefetch and the dynamic row claims (a CTA takes its next
    row from a counter the iteration's last CTA resets) change no bit: state,
    pf and gbest equal the forward, prefetch-free, round-robin run after every
    call (many rows per CTA, the wide 512-thread kernel at d = 4096, fewer rows
    than CTAs, the cluster kernel at d = 12000)."""
    monkeypatch.setenv("PSO_RESIDENT", "0")
    keep_cluster(monkeypatch, d)
    monkeypatch.setenv("PSO_SERP", "1")
    monkeypatch.setenv("PSO_L2PF_ALL", "1")
    monkeypatch.setenv("PSO_DYN_ROWS", "3")  # claims on every streaming path, the cluster too
    g = gpu_swarm(n, d, obj, seed=12)
    monkeypatch.setenv("PSO_SERP", "0")
    monkeypatch.setenv("PSO_L2PF", "0")
    monkeypatch.setenv("PSO_L2PF_ALL", "0")
    monkeypatch.setenv("PSO_DYN_ROWS", "0")
    e = gpu_swarm(n, d, obj, seed=12)
    for k in (1, 2, 3, 1):
        g.step(k)
        e.step(k)
        for x, y, nm in zip(g.get_state()[:4], e.get_state()[:4], "X V PB pf".split()):
            assert_bitwise(x, y, f"serpentine vs forward {nm}")
        assert g.gbest()[:2] == e.gbest()[:2]
    assert g.info()["launches"] == e.info()["launches"]


def test_async_gbest_single_rank_is_synchronous(monkeypatch):
    """With one rank the asynchronous split has nobody to lag behind: bitwise
    the synchronous single-GPU run."""
    import torch  # noqa: F401
    monkeypatch.setenv("PSO_FORCE_EXCHANGE", "1")
    comm = fp.nccl_comm_init(1, fp.nccl_unique_id(), 0, 0)
    try:
        lo, hi = DOMAINS[RASTRIGIN]
        g = fp.Swarm(300, 1000, 0.9, 2.0, 2.0, lo, hi, RASTRIGIN, 9, device=0, nccl_comm=comm,
                     async_gbest=True)
        ref = gpu_swarm(300, 1000, RASTRIGIN, seed=9)
        for k in (1, 6, 3):
            g.step(k)
            ref.step(k)
            assert g.gbest()[:2] == ref.gbest()[:2]
        for x, y in zip(g.get_state()[:4], ref.get_state()[:4]):
            assert_bitwise(x, y, "async 1-rank state")
        g.close()
    finally:
        fp.nccl_comm_destroy(comm)


# ------------------------------------------------------------------ column split (NEXT-3)
def _col_tiles(d):
    nv = (d + 3) // 4
    t = min(max((nv + 7) // 8, 32), 512, nv)
    return -(-nv // t)


@pytest.mark.parametrize("obj", OBJS)
@pytest.mark.parametrize("n,d", [(20, 13), (33, 999), (9, 2049), (6, 5000), (4, 40001)])
def test_column_split_single_gpu_matches_oracle(obj, n, d):
    """PSO_FLAG_COLUMN_SPLIT on one GPU: rows cut into column tiles, tile
    partials combined by k_col_decide.  Init bit-exact; one step from injected
    state bit-exact in X / V, decisions as the oracle's; pf within tolerance."""
    g = gpu_swarm(n, d, obj, seed=d + 3 * obj, column_split=True)
    info = g.info()
    assert info["column_split"] == 1 and info["col_begin"] == 0 and info["d_local"] == d
    assert info["col_tiles"] == _col_tiles(d)
    c = cpu_swarm(n, d, obj, seed=d + 3 * obj)
    X, V, PB, pf, t = g.get_state()
    assert t == 0
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    assert_bitwise(PB, c.PB, "PB0")
    assert_fitness_close(obj, c.X, pf, c.pf, "pf0")
    gf, gi, G = g.gbest()
    assert_bitwise(G, PB[gi], "G == PB[gi]")
    assert gf == pf.min() and gi == int(np.argmin(pf))
    _step_and_compare(obj, n, d, seed=7000 + d, pf_mode="mixed", t0=3, column_split=True)
    _step_and_compare(obj, n, d, seed=7100 + d, pf_mode="inf", t0=0, column_split=True)


@pytest.mark.parametrize("obj,n,d", [(ROSENBROCK, 5, 9000), (GRIEWANK, 7, 3001),
                                     (RASTRIGIN, 3, 70001), (ROSENBROCK, 2, 65537)])
def test_column_split_lockstep_and_wide_rows(obj, n, d):
    """Several iterations in lockstep with the oracle (the lazy pbest rows of
    the split: position / pbest slots, the plain layout restored by get_state); d > PSO_D_MAX_ROW
    selects the column split automatically."""
    kw = {} if d > fp.PSO_D_MAX_ROW else {"column_split": True}
    g = gpu_swarm(n, d, obj, seed=31, **kw)
    assert g.info()["column_split"] == 1
    c = cpu_swarm(n, d, obj, seed=31, create=False)
    for _ in range(4):
        X, V, PB, pf, t = g.get_state()
        c.set_state(X, V, PB, pf, t=t)
        g.step(1)
        c.step(1)
        X2, V2, PB2, pf2, _ = g.get_state()
        assert_bitwise(X2, c.X, "X")
        assert_bitwise(V2, c.V, "V")
        assert_fitness_close(obj, c.PB, pf2, c.pf, "pf")
        gf, gi, G = g.gbest()
        assert gf == pf2.min() and gi == int(np.argmin(pf2))
        assert_bitwise(G, PB2[gi], "G == PB[gi]")
    info = g.info()
    assert info["launches"] >= 2 + 2 * 4


@pytest.mark.parametrize("obj,n,d,vmax", [(GRIEWANK, 48, 3001, 40.0), (ROSENBROCK, 24, 5003, 0.3),
                                          (SPHERE, 40, 2049, 2.0), (RASTRIGIN, 6, 20001, 0.5)])
def test_column_split_position_slots_lockstep(obj, n, d, vmax):
    """The column split keeps a row's position and pbest in two slots (the X
    and PB arrays, pbx bit 1) and never copies a pbest: a lazy row (improved
    in the last decision) stores x' into the other slot, so its old x stays
    as the pbest.  Step by step against the oracle with the state read by
    get_rows, which resolves the slots without restoring the plain layout, so
    every slot transition (plain -> lazy -> swapped -> lazy in the other slot
    ...) runs on the device over several iterations; get_state (which
    restores the plain layout) then returns the same bits, and a twin run
    that was never read equals the read one after further steps."""
    seed = 900 + d
    g = gpu_swarm(n, d, obj, seed=seed, vmax=vmax, column_split=True)
    twin = gpu_swarm(n, d, obj, seed=seed, vmax=vmax, column_split=True)
    assert g.info()["column_split"] == 1
    c = cpu_swarm(n, d, obj, seed=seed, vmax=vmax, create=False)
    idx = np.arange(n)
    imps, T = 0, 8
    for it in range(T):
        X, V, PB, pf = g.get_rows(idx)
        c.set_state(X, V, PB, pf, t=it)
        g.step(1)
        c.step(1)
        X2, V2, PB2, pf2 = g.get_rows(idx)
        assert_bitwise(X2, c.X, f"X, iteration {it + 1}")
        assert_bitwise(V2, c.V, f"V, iteration {it + 1}")
        tol = fit_tol(obj, c.X, c.f)
        amb = np.abs(c.f.astype(np.float64) - pf.astype(np.float64)) <= tol
        c_imp = c.f < pf
        g_imp = (pf2.view(np.uint32) != pf.view(np.uint32)) | (PB2 != PB).any(axis=1)
        assert ((g_imp == c_imp) | amb).all()
        agree = (g_imp == c_imp) & ~amb
        assert_bitwise(PB2[agree], c.PB[agree], f"PB, iteration {it + 1}")
        assert_fitness_close(obj, c.X[agree & c_imp], pf2[agree & c_imp], c.pf[agree & c_imp], "pf")
        gf, gi, G = g.gbest()
        assert_bitwise(G, PB2[gi], "G == PB[gi]")
        imps += int(c_imp.sum())
    assert 0 < imps < n * T  # both pbest branches, so lazy rows turn plain and plain rows lazy
    twin.step(T)
    Xr, Vr, PBr, pfr = g.get_rows(idx)
    for a, b in zip(twin.get_rows(idx), (Xr, Vr, PBr, pfr)):
        assert_bitwise(a, b, "a run read with get_rows equals one that was not")
    X, V, PB, pf, t = g.get_state()
    for a, b in zip((X, V, PB, pf), (Xr, Vr, PBr, pfr)):
        assert_bitwise(a, b, "get_state (plain layout) equals get_rows (slots)")
    g.step(3)
    twin.step(3)
    for a, b in zip(g.get_state()[:4], twin.get_state()[:4]):
        assert_bitwise(a, b, "stepping after the layout was restored")
    assert_bitwise(g.gbest()[2], twin.gbest()[2], "G")


@pytest.mark.parametrize("n,d,forced", [(6, 6001, True), (3, 20001, False)])
def test_column_split_with_bounds_lockstep(n, d, forced):
    """Per-dimension bounds through the column split, forced (d = 6001) or
    chosen automatically on one GPU (d > PSO_D_AUTO_COLSPLIT)."""
    obj = ROSENBROCK
    b = _dim_bounds(d, 5)
    lo, hi = DOMAINS[obj]
    g = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 23, device=0, bounds=b, column_split=forced)
    assert g.info()["column_split"] == 1 and g.info()["bounds"] == 1
    c = orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 23, bounds=b)
    X, V, PB, pf, _ = g.get_state()
    assert_bitwise(X, c.X, "X0")
    assert_bitwise(V, c.V, "V0")
    for _ in range(3):
        X, V, PB, pf, t = g.get_state()
        c.set_state(X, V, PB, pf, t=t)
        g.step(1)
        c.step(1)
        X2, V2, _, pf2, _ = g.get_state()
        assert_bitwise(X2, c.X, "X")
        assert_bitwise(V2, c.V, "V")
        assert_fitness_close(obj, c.PB, pf2, c.pf, "pf")


def test_column_split_end_to_end_c1_gbest():
    """C1 (Sphere 32 x 10, 100 iterations) through the column split: gbest
    within relative 1e-4 of the oracle (north_star)."""
    w = WORKLOADS["C1"]
    g = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax,
                 device=0, column_split=True)
    c = orc.OracleSwarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax)
    g.step(w.iters)
    c.step(w.iters)
    gf, _, _ = g.gbest()
    assert abs(gf - c.gf) <= 1e-4 * abs(c.gf) + 1e-30


@pytest.mark.parametrize("obj", [RASTRIGIN, GRIEWANK])
def test_maximum_dimension(obj):
    """d = PSO_D_MAX (2^24, the column split on one GPU, 4096 tiles per row):
    init and two steps equal the oracle -- X, V, PB bitwise, fitness within the
    tolerance (Griewank: the product of 16.7M factors), gbest as the oracle's."""
    n, d = 2, fp.PSO_D_MAX
    g = gpu_swarm(n, d, obj, seed=77)
    assert g.info()["column_split"] == 1
    c = cpu_swarm(n, d, obj, seed=77)
    for k in (0, 1, 1):
        g.step(k)
        c.step(k)
        X, V, PB, pf, t = g.get_state()
        assert t == c.t
        assert_bitwise(X, c.X, f"X t={t}")
        assert_bitwise(V, c.V, f"V t={t}")
        assert_bitwise(PB, c.PB, f"PB t={t}")
        assert_fitness_close(obj, c.PB, pf, c.pf, f"pf t={t}")
        gf, gi, G = g.gbest()
        assert gi == c.gi
        assert_bitwise(G, PB[gi], "G == PB[gi]")
