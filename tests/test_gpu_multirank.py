"""Ranks of the particle split as 2-8 processes on ONE GPU, with
the NVLink peer exchange (CUDA IPC mappings between the processes): every
iteration each rank's step kernel stores its gbest record into every rank's
receive buffer and the next step kernel acquires the tags -- the real
multi-rank protocol (slot rotation, epoch tags, merge order), not a 1-rank
stand-in.  Every call's result is checked against the oracle run as `world`
virtual shards, and the whole run against a single-process run bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as orc
import paper_conf_icpp_liuwc21_b200 as fp
from pso_testutil import assert_bitwise, oracle_lockstep
from synth import DOMAINS, GRIEWANK, RASTRIGIN, ROSENBROCK, SPHERE, random_state, row_range

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _snap(s):
    X, V, PB, pf, t = s.get_state()
    f, i, G = s.gbest()
    return dict(X=X, V=V, PB=PB, pf=pf, t=t, f=f, i=i, G=G)


def _run_ops(s, ops, rows=None, cols=None):
    """Apply ops to a handle; a snapshot after create / init and after each op.
    ("step", k); ("restore", None): set_state with the handle's own state (a new
    epoch: records of the previous state must never match); ("set_state",
    (X, V, PB, pf, t)) with the whole swarm, of which this rank takes its rows
    (particle split) or its column block (column split)."""
    snaps = [_snap(s)]
    for op, arg in ops:
        if op == "step":
            s.step(arg)
        elif op == "restore":
            X, V, PB, pf, t = s.get_state()
            s.set_state(X, V, PB, pf, t=t)
        else:
            X, V, PB, pf, t = arg
            if rows is not None:
                b, e = rows
                X, V, PB, pf = X[b:e], V[b:e], PB[b:e], pf[b:e]
            if cols is not None:
                b, e = cols
                X, V, PB = X[:, b:e], V[:, b:e], PB[:, b:e]
            s.set_state(np.ascontiguousarray(X), np.ascontiguousarray(V), np.ascontiguousarray(PB),
                        pf, t=t)
        snaps.append(_snap(s))
    return snaps


def _save(out_dir, tag, rank, snaps, **extra):
    flat = {f"{k}{j}": np.asarray(v) for j, sn in enumerate(snaps) for k, v in sn.items()}
    np.savez(os.path.join(out_dir, f"{tag}{rank}.npz"), nsnap=len(snaps), **flat, **extra)


def _load(path):
    z = np.load(path)
    out = []
    for j in range(int(z["nsnap"])):
        sn = {k: z[f"{k}{j}"] for k in ("X", "V", "PB", "pf", "G")}
        sn.update(t=int(z[f"t{j}"]), f=float(z[f"f{j}"]), i=int(z[f"i{j}"]))
        out.append(sn)
    return out, z


def _worker(rank, world, port, n, d, obj, seed, ops, out_dir, params=(0.9, 2.0, 2.0, None),
            bounds=None, column_split=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    w, c1, c2, dom = params
    lo, hi = dom or DOMAINS[obj]
    s = fp.Swarm(n, d, w, c1, c2, lo, hi, obj, seed, device=0, world=world, rank=rank,
                 defer_init=True, bounds=bounds, column_split=column_split)
    assert connect_p2p(s)
    s.init()
    info = s.info()
    if column_split:
        snaps = _run_ops(s, ops, cols=(info["col_begin"], info["col_begin"] + info["d_local"]))
    else:
        snaps = _run_ops(s, ops, rows=row_range(n, rank, world))
    _save(out_dir, "r", rank, snaps, launches=info["launches"])
    s.close()
    dist.barrier()
    dist.destroy_process_group()


def _gathered(tmp_path, tag, world, axis=0):
    per_rank = [_load(tmp_path / f"{tag}{r}.npz")[0] for r in range(world)]
    out = []
    for j in range(len(per_rank[0])):
        sn = dict(per_rank[0][j])
        for k in ("X", "V", "PB"):
            sn[k] = np.concatenate([pr[j][k] for pr in per_rank], axis=axis)
        if axis == 0:
            sn["pf"] = np.concatenate([pr[j]["pf"] for pr in per_rank])
        else:
            sn["G"] = np.concatenate([pr[j]["G"] for pr in per_rank])
            for pr in per_rank[1:]:  # every rank holds all n pf and the same gbest
                assert_bitwise(pr[j]["pf"], sn["pf"], f"pf rank-identical, snapshot {j}")
        for pr in per_rank[1:]:  # the gbest is bitwise identical on every rank
            assert (pr[j]["f"], pr[j]["i"], pr[j]["t"]) == (sn["f"], sn["i"], sn["t"])
            if axis == 0:
                assert_bitwise(pr[j]["G"], sn["G"], f"G rank-identical, snapshot {j}")
        out.append(sn)
    return out


def _oracle_ops(ops, snaps):
    """The ops as the oracle replays them (restore = set_state of the previous snapshot)."""
    out = []
    for k, (op, arg) in enumerate(ops):
        if op == "restore":
            p = snaps[k]
            arg = (p["X"], p["V"], p["PB"], p["pf"], p["t"])
            op = "set_state"
        out.append((op, arg))
    return out


def _injected_state(n, d, t):
    """A random injected state: every pbest above every fitness (all rows
    improve) and a NaN pbest at row 0 (read as +inf)."""
    lo, hi = DOMAINS[RASTRIGIN]
    X, V, PB, pf = random_state(n, d, lo, hi, 1.0, 99 + n, pf_mode="rand")
    pf = (pf + np.float32(5e4)).astype(np.float32)
    pf[0] = np.nan
    return X, V, PB, pf, t


WORLDS = [(2, RASTRIGIN, 300, 1000), (2, GRIEWANK, 41, 13), (2, ROSENBROCK, 6, 10000),
          (3, RASTRIGIN, 7, 2000), (4, GRIEWANK, 9, 999), (8, RASTRIGIN, 203, 1000),
          (8, GRIEWANK, 37, 2001), (3, SPHERE, 2, 300)]


@pytest.mark.parametrize("world,obj,n,d", WORLDS)
def test_processes_nvlink_exchange_match_the_oracle(tmp_path, world, obj, n, d, monkeypatch):
    """Each rank's shard after every call equals the oracle run as `world`
    virtual particle shards (X, V, PB bitwise, pf within the
    fitness tolerance, (gi, G) the oracle's), replayed call by call from the
    gathered GPU state; the gbest is bitwise identical on every rank; and the
    whole run equals a single-process run bit for bit (world invariance).
    (3, SPHERE, 2, 300): rank 0 owns no particle (n < world)."""
    seed = 4242
    ops = [("step", 1), ("step", 4), ("step", 3), ("restore", None), ("step", 2)]
    if obj == RASTRIGIN:
        ops += [("set_state", _injected_state(n, d, t=17)), ("step", 1), ("step", 2)]
    mp.spawn(_worker, args=(world, _free_port(), n, d, obj, seed, ops, str(tmp_path)),
             nprocs=world, join=True)
    snaps = _gathered(tmp_path, "r", world)
    lo, hi = DOMAINS[obj]

    def make_oracle(create):
        return orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, nshards=world,
                               create=create)

    skip_state, skip_g = oracle_lockstep(make_oracle, obj, snaps, _oracle_ops(ops, snaps),
                                         f"world={world}")
    assert skip_state <= 1 and skip_g <= 2, (skip_state, skip_g)
    # world invariance: the single-process run of the same ops (on the ranks'
    # row kernel: one GPU alone would take the column split above d = 9216)
    monkeypatch.setenv("PSO_COLSPLIT", "0")
    ref = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, device=0)
    rsnaps = _run_ops(ref, ops)
    for j, (a, b) in enumerate(zip(snaps, rsnaps)):
        for k in ("X", "V", "PB", "pf", "G"):
            assert_bitwise(a[k], b[k], f"snapshot {j} {k} vs 1 process")
        assert (a["f"], a["i"], a["t"]) == (b["f"], b["i"], b["t"])


@pytest.mark.parametrize("case", ["ties", "zero", "minf"])
@pytest.mark.parametrize("world", [3, 8])
def test_processes_decisions_across_ranks(tmp_path, world, case):
    """The decision pins (readings 9-11) with the rows of the case in different
    ranks (row 1 on rank 0, row n - 2 on the last rank): equal fitness in two
    ranks goes to the lower global index through the NVLink merge, -0 ties +0
    across ranks, a -inf pbest on the last rank wins everywhere.  Frozen swarm,
    so every value is exact: compared with the oracle bit for bit."""
    from pso_testutil import crafted_expect, crafted_state
    n, d = 48, 1000
    obj, lo, hi, X, V, PB, pf, a, b = crafted_state(case, n, d)
    assert row_range(n, 0, world)[1] > a and row_range(n, world - 1, world)[0] <= b
    ops = [("set_state", (X, V, PB, pf, 5)), ("step", 1), ("step", 1),
           ("set_state", (X, V, PB, pf, 8)), ("step", 2)]
    mp.spawn(_worker, args=(world, _free_port(), n, d, obj, 7, ops, str(tmp_path),
                            (0.0, 0.0, 0.0, (lo, hi))), nprocs=world, join=True)
    snaps = _gathered(tmp_path, "r", world)
    c = orc.OracleSwarm(n, d, 0.0, 0.0, 0.0, lo, hi, obj, 7, nshards=world, create=False)
    expect_steps = [None, 0, 1, 2, 0, 2]
    for j, (op, arg) in enumerate(ops, start=1):
        if op == "set_state":
            c.set_state(*arg[:4], t=arg[4])
        else:
            c.step(arg)
        sn = snaps[j]
        for k, ref in (("X", c.X), ("V", c.V), ("PB", c.PB), ("pf", c.pf), ("G", c.G)):
            assert_bitwise(sn[k], ref, f"{case} world={world} snapshot {j}: {k}")
        assert (sn["i"], sn["t"]) == (c.gi, c.t) and sn["f"] == c.gf
        assert (sn["i"], sn["f"]) == crafted_expect(case, n, d, expect_steps[j])


def _async_worker(rank, world, port, n, d, obj, steps, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    lo, hi = DOMAINS[obj]
    s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 777, device=0, world=world, rank=rank,
                 defer_init=True, async_gbest=True)
    assert connect_p2p(s)
    s.init()
    views = []
    for n_call, k in enumerate(steps):
        if n_call == len(steps) - 1:  # restore mid-run: synchronous re-selection, lag restarts
            s.set_state(*s.get_state())
        s.step(k)
        views.append(s.gbest()[:2])
    X, V, PB, pf, t = s.get_state()
    f, i, G = s.gbest()
    np.savez(os.path.join(out_dir, f"a{rank}.npz"), X=X, V=V, PB=PB, pf=pf, G=G, t=t,
             views=np.array(views, dtype=np.float64))
    s.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,obj,n,d", [(2, RASTRIGIN, 40, 300), (3, GRIEWANK, 30, 13),
                                           (2, ROSENBROCK, 4, 9000), (3, SPHERE, 2, 300),
                                           (8, RASTRIGIN, 50, 1000)])
def test_async_split_matches_the_async_oracle(tmp_path, world, obj, n, d):
    """NEXT-4: each rank adopts its own candidates at once and its peers' one
    iteration late (merging records of t - 2 over NVLink); set_state mid-run
    re-selects synchronously and restarts the lag.  Per-rank state and the host
    view equal the oracle's asynchronous split model."""
    from oracle.async_model import AsyncSplitSwarm
    from pso_testutil import assert_bitwise, assert_fitness_close
    steps = (2, 3, 4)
    mp.spawn(_async_worker, args=(world, _free_port(), n, d, obj, steps, str(tmp_path)),
             nprocs=world, join=True)
    lo, hi = DOMAINS[obj]
    model = AsyncSplitSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 777, k=world)
    views = []
    for n_call, k in enumerate(steps):
        if n_call == len(steps) - 1:
            model.set_state([model.state(r)[:4] for r in range(world)], t=model.t)
        model.step(k)
        views.append(model.view(0)[:2])
    for r in range(world):
        z = np.load(tmp_path / f"a{r}.npz")
        X, V, PB, pf, t = model.state(r)
        assert int(z["t"]) == t
        assert_bitwise(z["X"], X, f"X rank {r}")
        assert_bitwise(z["V"], V, f"V rank {r}")
        assert_bitwise(z["PB"], PB, f"PB rank {r}")
        assert_fitness_close(obj, PB, z["pf"], pf, f"pf rank {r}")
        for (gf, gi), (mf, mi) in zip(z["views"], views):
            assert int(gi) == mi
            assert abs(gf - mf) <= 1e-5 * abs(mf) + 1e-6


def _col_worker(rank, world, port, n, d, obj, seed, ops, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    lo, hi = DOMAINS[obj]
    s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, device=0, world=world, rank=rank,
                 defer_init=True, column_split=True)
    assert connect_p2p(s)
    s.init()
    info = s.info()
    snaps = _run_ops(s, ops, cols=(info["col_begin"], info["col_begin"] + info["d_local"]))
    _save(out_dir, "c", rank, snaps, col_begin=info["col_begin"], d_local=info["d_local"])
    s.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,obj,n,d", [(2, ROSENBROCK, 50, 6000), (3, GRIEWANK, 17, 9001),
                                           (4, RASTRIGIN, 64, 4096), (2, ROSENBROCK, 3, 70001),
                                           (8, RASTRIGIN, 40, 8192)])
def test_column_split_processes_match_the_oracle(tmp_path, world, obj, n, d):
    """NEXT-3 across ranks ("tile matrix"): each rank process owns a
    block of column tiles of every row; tile partials travel by NVLink peer
    stores, every rank decides pbest / gbest from the same partial table.  The
    blocks tile the row in rank order; the gathered state after every call
    equals the oracle (replayed call by call), pf and the gbest are identical
    on every rank, and the run equals the single-GPU column split bit for bit."""
    seed = 99
    ops = [("step", 1), ("step", 3), ("step", 1), ("restore", None), ("step", 2), ("step", 1)]
    mp.spawn(_col_worker, args=(world, _free_port(), n, d, obj, seed, ops, str(tmp_path)),
             nprocs=world, join=True)
    covered = 0
    for r in range(world):
        z = np.load(tmp_path / f"c{r}.npz")
        assert int(z["col_begin"]) == covered  # blocks tile the row in rank order
        covered += int(z["d_local"])
    assert covered == d
    snaps = _gathered(tmp_path, "c", world, axis=1)
    lo, hi = DOMAINS[obj]

    def make_oracle(create):
        return orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, create=create)

    skip_state, skip_g = oracle_lockstep(make_oracle, obj, snaps, _oracle_ops(ops, snaps),
                                         f"colsplit world={world}")
    assert skip_state <= 1 and skip_g <= 2, (skip_state, skip_g)
    ref = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, device=0, column_split=True)
    rsnaps = _run_ops(ref, ops)
    for j, (a, b) in enumerate(zip(snaps, rsnaps)):
        for k in ("X", "V", "PB", "pf", "G"):
            assert_bitwise(a[k], b[k], f"snapshot {j} {k} vs 1 process")
        assert (a["f"], a["i"], a["t"]) == (b["f"], b["i"], b["t"])


@pytest.mark.parametrize("split,world,obj,n,d", [("particle", 3, RASTRIGIN, 40, 1000),
                                                 ("particle", 2, ROSENBROCK, 9, 2001),
                                                 ("column", 3, RASTRIGIN, 12, 6001),
                                                 ("column", 2, GRIEWANK, 7, 9000)])
def test_processes_with_per_dimension_bounds_match_the_oracle(tmp_path, split, world, obj, n, d):
    """NEXT-2's per-dimension velocity bounds and domains (Eq. 5's
    lower/upper_bound_j) across rank processes: the particle split
    (every rank holds the whole bounds table) and the column split (each rank
    its block of it) equal the oracle call by call."""
    rng = np.random.default_rng(d)
    xlo = rng.uniform(-5, -0.5, d).astype(np.float32)
    xhi = (xlo + rng.uniform(0.5, 6, d)).astype(np.float32)
    vhi = rng.uniform(0.05, 2, d).astype(np.float32)
    vlo = (-rng.uniform(0.05, 2, d)).astype(np.float32)
    bounds = np.stack([vlo, vhi, xlo, xhi])
    seed = 31
    ops = [("step", 1), ("step", 3), ("restore", None), ("step", 2)]
    lo, hi = DOMAINS[obj]
    mp.spawn(_worker, args=(world, _free_port(), n, d, obj, seed, ops, str(tmp_path),
                            (0.9, 2.0, 2.0, None), bounds, split == "column"),
             nprocs=world, join=True)
    snaps = _gathered(tmp_path, "r", world, axis=1 if split == "column" else 0)

    def make_oracle(create):
        return orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, seed, create=create, bounds=bounds,
                               nshards=world if split == "particle" else 1)

    skip_state, skip_g = oracle_lockstep(make_oracle, obj, snaps, _oracle_ops(ops, snaps),
                                         f"{split} bounds world={world}")
    assert skip_state <= 1 and skip_g <= 2, (skip_state, skip_g)


def _dead_peer_worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["PSO_PEER_TIMEOUT_S"] = "2"
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import time
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    s = fp.Swarm(64, 300, 0.9, 2.0, 2.0, -5.12, 5.12, RASTRIGIN, 5, device=0, world=world,
                 rank=rank, defer_init=True)
    assert connect_p2p(s)
    s.init()
    if rank == 0:  # rank 1 never steps: the second iteration's prologue waits for its record
        t0 = time.time()
        status, msg = -1, ""
        try:
            s.step(3)
            s.gbest()
        except fp.PsoError as e:
            status, msg = e.status, str(e)
        try:
            s.gbest()
        except fp.PsoError as e:
            msg += " | then: " + str(e)
        with open(os.path.join(out_dir, "dead_peer.txt"), "w") as fh:
            fh.write(f"{status}\n{time.time() - t0:.2f}\n{msg}\n")
    dist.barrier()  # rank 1 stays alive (its memory mapped) until rank 0 has seen the failure
    os._exit(0)


def test_dead_peer_traps_and_poisons_instead_of_hanging(tmp_path):
    """A rank that stops delivering its records (here: it never steps) makes
    the waiting step kernel trap after the peer timeout (PSO_PEER_TIMEOUT_S=2)
    -- the handle reports PSO_ERR_CUDA and is poisoned, nothing hangs."""
    mp.spawn(_dead_peer_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    status, secs, msg = open(tmp_path / "dead_peer.txt").read().split("\n")[:3]
    assert int(status) == 3, msg  # PSO_ERR_CUDA
    assert 1.5 < float(secs) < 30, secs
    assert "POISONED" in msg, msg
