"""Process-group plumbing for the particle-split multi-GPU path.

One process per GPU.  torch.distributed (any backend) only carries
out-of-band setup data: the 128-byte NCCL unique id, and the CUDA IPC handles
of the NVLink peer exchange.  Per iteration the gbest exchange runs inside the
step kernels (NVLink peer stores of each rank's record, merged by the next
kernel's prologue); the NCCL all-gather of the same records (+ a select
kernel at the end of each pso_step call) is the fallback when a rank cannot
map or probe its peers.
"""
from __future__ import annotations

import os
import sys

from . import nccl_comm_destroy, nccl_comm_init, nccl_unique_id


def env_rank_world() -> tuple[int, int, int]:
    """(rank, world, local_rank) from the torchrun environment (defaults: 0, 1, 0)."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    return rank, world, local


def row_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Rows owned by `rank`: [floor(n r / k), floor(n (r+1) / k)) (include/fastpso.h)."""
    return (n * rank) // world, (n * (rank + 1)) // world


def broadcast_unique_id(uid_factory=nccl_unique_id, group=None) -> bytes:
    """Rank 0 creates the id; every rank receives it over torch.distributed."""
    import torch.distributed as dist
    obj = [uid_factory() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return bytes(obj[0])


def init_comm(device: int, group=None) -> int:
    """Create the library's NCCL communicator over the ranks of `group`."""
    import torch.distributed as dist
    uid = broadcast_unique_id(group=group)
    return nccl_comm_init(dist.get_world_size(group), uid, dist.get_rank(group), device)


def destroy_comm(comm: int) -> None:
    if comm:
        nccl_comm_destroy(comm)


def _log(msg: str) -> None:
    if os.environ.get("PSO_QUIET", "0") in ("", "0"):
        print(f"[fastpso] {msg}", file=sys.stderr, flush=True)


def connect_p2p(swarm, group=None) -> bool:
    """Switch `swarm` to the NVLink peer exchange: all-gather every rank's CUDA
    IPC handle + receive-buffer offset over torch.distributed, map the peers'
    buffers, then PROBE the mapped path (every rank stores a token into every
    peer with a system-scope release; after a barrier every rank checks it
    received all of them).  The mode is enabled only if every rank mapped and
    probed successfully; otherwise every rank stays on the NCCL all-gather (a
    handle with a communicator) and the reason is logged to stderr.  Returns
    whether the peer exchange is on.  Collective."""
    import torch.distributed as dist
    from . import PsoError
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    mine = swarm.p2p_handle()
    everyone = [None] * world
    dist.all_gather_object(everyone, mine, group=group)
    why = ""
    try:
        swarm.p2p_connect([h for h, _ in everyone], [o for _, o in everyone])
    except PsoError as e:
        why = f"rank {rank}: peer mapping failed: {e}"
    votes = [None] * world
    dist.all_gather_object(votes, why, group=group)
    reasons = [v for v in votes if v]
    if not reasons:
        probe_ok = False
        try:
            swarm.p2p_probe(0)
            dist.barrier(group=group)
            probe_ok = swarm.p2p_probe(1)
        except PsoError as e:
            why = f"rank {rank}: probe failed: {e}"
        if not probe_ok and not why:
            why = f"rank {rank}: probe tokens missing"
        votes = [None] * world
        dist.all_gather_object(votes, why, group=group)
        reasons = [v for v in votes if v]
    if not reasons:
        swarm.p2p_enable(True)
        if rank == 0:
            _log(f"gbest exchange: NVLink peer stores, {world} ranks mapped and probed")
        return True
    if rank == 0:
        _log("gbest exchange: falling back to the NCCL all-gather (" + "; ".join(reasons) + ")")
    return False
