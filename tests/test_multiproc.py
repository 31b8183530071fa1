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


class _FakeSwarm:
    """The four p2p calls of a handle, scripted per rank (no GPU): connect_p2p's
    collective decision logic is what is under test."""

    def __init__(self, rank, fail_connect=False, fail_probe=False):
        self.rank, self.fail_connect, self.fail_probe = rank, fail_connect, fail_probe
        self.enabled = False
        self.calls = []

    def p2p_handle(self):
        return bytes([self.rank]) * 64, 4096 + self.rank

    def p2p_connect(self, handles, offsets):
        from paper_conf_icpp_liuwc21_b200 import PsoError
        self.calls.append(("connect", [h[0] for h in handles], list(offsets)))
        if self.fail_connect:
            raise PsoError(3, "pso_p2p_connect", "cudaIpcOpenMemHandle failed (scripted)")

    def p2p_probe(self, phase):
        self.calls.append(("probe", phase))
        return not self.fail_probe

    def p2p_enable(self, on=True):
        self.enabled = bool(on)


def _connect_worker(rank, world, port, fail_connect_rank, fail_probe_rank, out_dir):
    _init(rank, world, port)
    os.environ["PSO_QUIET"] = "1"
    from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
    s = _FakeSwarm(rank, fail_connect=rank == fail_connect_rank, fail_probe=rank == fail_probe_rank)
    on = connect_p2p(s)
    import json
    with open(os.path.join(out_dir, f"c{rank}.json"), "w") as fh:
        json.dump({"on": on, "enabled": s.enabled, "calls": s.calls}, fh)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,fail_connect,fail_probe", [(2, -1, -1), (3, 1, -1), (2, -1, 0),
                                                           (3, -1, 2)])
def test_connect_p2p_is_all_or_nothing(tmp_path, world, fail_connect, fail_probe):
    """The NVLink exchange is switched on only if every rank mapped its peers
    AND every rank's probe saw every token; otherwise no rank enables it (all
    stay on the NCCL exchange).  Handles and offsets reach every rank in rank
    order; a failed mapping skips the probe on every rank."""
    import json
    mp.spawn(_connect_worker, args=(world, _free_port(), fail_connect, fail_probe, str(tmp_path)),
             nprocs=world, join=True)
    res = [json.load(open(tmp_path / f"c{r}.json")) for r in range(world)]
    expect = fail_connect < 0 and fail_probe < 0
    for r in res:
        assert r["on"] == expect and r["enabled"] == expect
        connect = [c for c in r["calls"] if c[0] == "connect"][0]
        assert connect[1] == list(range(world)) and connect[2] == [4096 + k for k in range(world)]
        probes = [c[1] for c in r["calls"] if c[0] == "probe"]
        assert probes == ([] if fail_connect >= 0 else [0, 1])
