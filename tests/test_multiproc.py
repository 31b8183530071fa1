"""World-size-2 tests of the particle-split path (made synchronous) on CPU
with the gloo backend: the shard/merge protocol the GPUs run (each rank
steps its rows, all ranks all-gather (key, candidate row) records, every rank
selects the same winner) reproduces the single-process run bitwise; the NCCL
unique id travels over torch.distributed; the row partition matches the ABI."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as orc
from synth import DOMAINS, RASTRIGIN, ROSENBROCK, row_range


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _shard_worker(rank, world, port, n, d, obj, T, out_dir):
    _init(rank, world, port)
    lo, hi = DOMAINS[obj]
    b, e = row_range(n, rank, world)
    s = orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 77, row_begin=b, nrows=e - b,
                        create=False)

    def exchange(cand, is_init):
        recs = [None] * world
        dist.all_gather_object(recs, cand)
        s.merge([r[0] for r in recs], [r[1] for r in recs], [r[2] for r in recs],
                np.stack([r[3] for r in recs]), is_init)

    exchange(s.init_local(), True)
    for _ in range(T):
        exchange(s.step_local(), False)
    np.savez(os.path.join(out_dir, f"rank{rank}.npz"), X=s.X, V=s.V, PB=s.PB, pf=s.pf, G=s.G,
             gf=s.gf, gi=s.gi, t=s.t, b=b, e=e)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n,d,obj,world", [(37, 9, RASTRIGIN, 2), (5, 4, ROSENBROCK, 2),
                                           (2, 3, RASTRIGIN, 3)])
def test_particle_split_matches_single_process(tmp_path, n, d, obj, world):
    T = 15
    mp.spawn(_shard_worker, args=(world, _free_port(), n, d, obj, T, str(tmp_path)), nprocs=world,
             join=True)
    lo, hi = DOMAINS[obj]
    ref = orc.OracleSwarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 77)
    ref.step(T)
    for r in range(world):
        z = np.load(tmp_path / f"rank{r}.npz")
        b, e = int(z["b"]), int(z["e"])
        for name in ("X", "V", "PB"):
            assert np.array_equal(z[name].view(np.uint32), getattr(ref, name)[b:e].view(np.uint32))
        assert np.array_equal(z["pf"].view(np.uint32), ref.pf[b:e].view(np.uint32))
        assert np.array_equal(z["G"].view(np.uint32), ref.G.view(np.uint32))  # replicated gbest
        assert float(z["gf"]) == ref.gf and int(z["gi"]) == ref.gi
        assert int(z["t"]) == T


def _uid_worker(rank, world, port, out_dir):
    _init(rank, world, port)
    from paper_conf_icpp_liuwc21_b200.distributed import broadcast_unique_id
    uid = broadcast_unique_id()
    with open(os.path.join(out_dir, f"uid{rank}.bin"), "wb") as fh:
        fh.write(uid)
    dist.barrier()
    dist.destroy_process_group()


def test_nccl_unique_id_broadcast_over_gloo(tmp_path):
    mp.spawn(_uid_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    a = (tmp_path / "uid0.bin").read_bytes()
    b = (tmp_path / "uid1.bin").read_bytes()
    assert len(a) == 128 and a == b and any(a)


@pytest.mark.parametrize("n", [1, 2, 7, 100_000, 2**32 - 1])
@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_row_partition_covers_every_row_once(n, world):
    from paper_conf_icpp_liuwc21_b200.distributed import row_range as lib_row_range
    spans = [row_range(n, r, world) for r in range(world)]
    assert spans == [lib_row_range(n, r, world) for r in range(world)]
    assert spans[0][0] == 0 and spans[-1][1] == n
    for (b0, e0), (b1, e1) in zip(spans, spans[1:]):
        assert e0 == b1 and b0 <= e0
    sizes = [e - b for b, e in spans]
    assert max(sizes) - min(sizes) <= 1
