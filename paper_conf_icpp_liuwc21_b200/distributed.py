"""Process-group plumbing for the particle-split multi-GPU path.

One process per GPU.  torch.distributed (any backend) only carries the
128-byte NCCL unique id from rank 0 to the others; the per-iteration exchange
(one ncclAllGather of the (key, candidate row) records + a select kernel)
runs inside the C library on the handle's stream.
"""
from __future__ import annotations

import os

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


def connect_p2p(swarm, group=None) -> bool:
    """Switch `swarm` (created with a communicator) to the NVLink peer exchange:
    all-gather every rank's CUDA IPC handle + receive-buffer offset over
    torch.distributed, map the peers' buffers, and enable the mode only if every
    rank succeeded (else all ranks stay on the NCCL all-gather).  Returns
    whether the peer exchange is on.  Collective."""
    import torch.distributed as dist
    from . import PsoError
    mine = swarm.p2p_handle()
    everyone = [None] * dist.get_world_size(group)
    dist.all_gather_object(everyone, mine, group=group)
    ok = True
    try:
        swarm.p2p_connect([h for h, _ in everyone], [o for _, o in everyone])
    except PsoError:
        ok = False
    votes = [None] * dist.get_world_size(group)
    dist.all_gather_object(votes, ok, group=group)
    if all(votes):
        swarm.p2p_enable(True)
        return True
    return False
