"""Ranks of the particle split as 2-4 processes on ONE GPU, with
the NVLink peer exchange (CUDA IPC mappings between the processes): every
iteration each rank's step kernel stores its gbest record into both ranks'
receive buffers and the next step kernel acquires both tags — the real
multi-rank protocol (parity double-buffering, epoch tags, merge order), not a
1-rank stand-in.  Results must equal a single-process run bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_icpp_liuwc21_b200 as fp
from synth import DOMAINS, GRIEWANK, RASTRIGIN, ROSENBROCK, row_range

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, n, d, obj, steps, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    lo, hi = DOMAINS[obj]
    s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 4242, device=0, world=world, rank=rank,
                 defer_init=True)
    assert connect_p2p(s)
    s.init()
    for k in steps:
        s.step(k)
    X, V, PB, pf, t = s.get_state()
    f, i, G = s.gbest()
    # set_state starts a new epoch: records of the previous state must never match
    s.set_state(X, V, PB, pf, t=t)
    s.step(2)
    X2, V2, PB2, pf2, t2 = s.get_state()
    f2, i2, G2 = s.gbest()
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), X=X, V=V, PB=PB, pf=pf, G=G, f=f, i=i, t=t,
             X2=X2, PB2=PB2, pf2=pf2, G2=G2, f2=f2, i2=i2, launches=s.info()["launches"])
    s.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,obj,n,d", [(2, RASTRIGIN, 300, 1000), (2, GRIEWANK, 41, 13),
                                           (2, ROSENBROCK, 6, 10000), (3, RASTRIGIN, 7, 2000),
                                           (4, GRIEWANK, 9, 999)])
def test_processes_nvlink_exchange_matches_single_gpu(tmp_path, world, obj, n, d):
    steps = (1, 4, 3)
    mp.spawn(_worker, args=(world, _free_port(), n, d, obj, steps, str(tmp_path)), nprocs=world,
             join=True)
    lo, hi = DOMAINS[obj]
    ref = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 4242, device=0)
    for k in steps:
        ref.step(k)
    RX, RV, RPB, Rpf, Rt = ref.get_state()
    rf, ri, RG = ref.gbest()
    ref.set_state(RX, RV, RPB, Rpf, t=Rt)
    ref.step(2)
    RX2, _, RPB2, Rpf2, _ = ref.get_state()
    rf2, ri2, RG2 = ref.gbest()
    for r in range(world):
        z = np.load(tmp_path / f"r{r}.npz")
        b, e = row_range(n, r, world)
        for name, full in (("X", RX), ("V", RV), ("PB", RPB), ("pf", Rpf), ("X2", RX2),
                           ("PB2", RPB2), ("pf2", Rpf2)):
            assert np.array_equal(z[name].view(np.uint32), full[b:e].view(np.uint32)), (r, name)
        assert int(z["t"]) == Rt
        assert (float(z["f"]), int(z["i"])) == (rf, ri)
        assert (float(z["f2"]), int(z["i2"])) == (rf2, ri2)
        assert np.array_equal(z["G"].view(np.uint32), RG.view(np.uint32))
        assert np.array_equal(z["G2"].view(np.uint32), RG2.view(np.uint32))


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
                                           (2, ROSENBROCK, 4, 9000)])
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


def _col_worker(rank, world, port, n, d, obj, steps, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    lo, hi = DOMAINS[obj]
    s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 99, device=0, world=world, rank=rank,
                 defer_init=True, column_split=True)
    assert connect_p2p(s)
    s.init()
    for k in steps:
        s.step(k)
    X, V, PB, pf, t = s.get_state()
    f, i, G = s.gbest()
    s.set_state(X, V, PB, pf, t=t)  # new epoch: stale tags never match
    s.step(2)
    X2, _, PB2, pf2, _ = s.get_state()
    f2, i2, G2 = s.gbest()
    info = s.info()
    np.savez(os.path.join(out_dir, f"c{rank}.npz"), X=X, V=V, PB=PB, pf=pf, G=G, f=f, i=i, t=t,
             X2=X2, PB2=PB2, pf2=pf2, G2=G2, f2=f2, i2=i2, col_begin=info["col_begin"],
             d_local=info["d_local"])
    s.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,obj,n,d", [(2, ROSENBROCK, 50, 6000), (3, GRIEWANK, 17, 9001),
                                           (4, RASTRIGIN, 64, 4096), (2, ROSENBROCK, 3, 70001)])
def test_column_split_processes_match_single_gpu(tmp_path, world, obj, n, d):
    """NEXT-3 across ranks ("tile matrix"): each rank process owns a
    block of column tiles of every row; tile partials travel by NVLink peer
    stores, every rank decides pbest / gbest from the same partial table.  The
    tiling depends on d only, so the ranks' blocks, pf and gbest equal the
    single-GPU column split bit for bit."""
    steps = (1, 3, 2)
    mp.spawn(_col_worker, args=(world, _free_port(), n, d, obj, steps, str(tmp_path)),
             nprocs=world, join=True)
    lo, hi = DOMAINS[obj]
    ref = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 99, device=0, column_split=True)
    for k in steps:
        ref.step(k)
    RX, RV, RPB, Rpf, Rt = ref.get_state()
    rf, ri, RG = ref.gbest()
    ref.set_state(RX, RV, RPB, Rpf, t=Rt)
    ref.step(2)
    RX2, _, RPB2, Rpf2, _ = ref.get_state()
    rf2, ri2, RG2 = ref.gbest()
    covered = 0
    for r in range(world):
        z = np.load(tmp_path / f"c{r}.npz")
        b = int(z["col_begin"])
        e = b + int(z["d_local"])
        assert b == covered  # blocks tile the row in rank order
        covered = e
        for name, full in (("X", RX), ("V", RV), ("PB", RPB), ("X2", RX2), ("PB2", RPB2)):
            assert np.array_equal(z[name].view(np.uint32), full[:, b:e].view(np.uint32)), (r, name)
        for name, full in (("pf", Rpf), ("pf2", Rpf2)):
            assert np.array_equal(z[name].view(np.uint32), full.view(np.uint32)), (r, name)
        assert np.array_equal(z["G"].view(np.uint32), RG[b:e].view(np.uint32))
        assert np.array_equal(z["G2"].view(np.uint32), RG2[b:e].view(np.uint32))
        assert (float(z["f"]), int(z["i"])) == (rf, ri)
        assert (float(z["f2"]), int(z["i2"])) == (rf2, ri2)
        assert int(z["t"]) == Rt
    assert covered == d
