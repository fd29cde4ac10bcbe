"""torch.distributed bootstrap for the edge-sharded path (plumbing only).

torch.distributed carries the 128-byte NCCL unique id from rank 0 to every
rank; the library then builds its own NCCL communicator and runs every step
(kernels and the per-round ncclAllReduce) itself.
"""
from __future__ import annotations

import torch.distributed as tdist

from . import _native


def unique_id_from_group(group=None) -> bytes:
    """Rank 0 of `group` creates the NCCL unique id; every rank returns it."""
    rank = tdist.get_rank(group)
    obj = [_native.ecl_mst_dist_unique_id() if rank == 0 else None]
    tdist.broadcast_object_list(obj, src=tdist.get_global_rank(group, 0) if group else 0, group=group)
    return obj[0]


def init_from_group(group=None):
    """Library handle for this rank (call with the rank's GPU current)."""
    uid = unique_id_from_group(group)
    return _native.ecl_mst_dist_init(uid, tdist.get_rank(group), tdist.get_world_size(group))
